"""Print parity statistics of the llama decode split (diagnostic, GPU)."""
import dataclasses
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
from oracle import llama as olm  # noqa: E402
from tests.gpu_util import DEV, bf16_tensor, to64  # noqa: E402
from tests.test_gpu_llama import _setup  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

for name in ("tiny-llama", "lm2"):
    if name == "lm2":
        cfg = dataclasses.replace(e3data.get("lm"), layers=2, ramp_layers=(0, 1), exit_profile=None, tau=(0.2, 0.2))
        ramp = e3data.make_ramp(cfg, 0)
        W = {"layers": [e3data.make_layer(cfg, 0), e3data.make_layer(cfg, 1)], "ramps": [ramp, ramp]}
    else:
        cfg = e3data.get(name)
        W = e3data.make_weights(cfg)
    B = cfg.batch
    slot_of = {i: i for i in range(B)}
    pos_of = {s: cfg.ctx for s in range(B)}
    W, kv_np, cache, model = _setup(api, cfg, B, slot_of, pos_of, B, W=W)
    X = e3data.make_inputs(cfg, range(B), seed=6)
    split = api.Split(model, api.split_desc(cfg, 0, cfg.ramp_layers[0] + 1, cfg.tau))
    x = bf16_tensor(X)
    x_out = torch.zeros_like(x)
    id_out = torch.full((B,), -9, dtype=torch.int64, device=DEV)
    n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
    ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, DEV)
    split.run(x, torch.arange(B, dtype=torch.int64, device=DEV), x_out, id_out, n_surv, ex)
    torch.cuda.synchronize()
    sample = list(range(0, B, max(1, B // 6)))
    kv_or = [np.stack([kv_np[l][0][sample], kv_np[l][1][sample]]).astype(np.float64) for l in range(cfg.layers)]
    so = {i: k for k, i in enumerate(sample)}
    po = {k: cfg.ctx for k in range(len(sample))}
    recs, surv, h, margins = olm.run_split(cfg, W, X[sample, 0], 0, cfg.ramp_layers[0] + 1, sample, kv_or, so, po,
                                           mode="bf16", )
    # brute logits for every sampled token at the first ramp
    el = ex.exit_layer.cpu().numpy()
    print(name, "gpu exits", int(ex.n_exit.item()), "of", B, "n_surv", int(n_surv.item()))
    print("  oracle exits among sample", len(recs), "of", len(sample), "margins", np.round(list(margins.values()), 4))
    lg = ex.logits.cpu().numpy()
    for r in recs:
        if el[r.id] == r.exit_layer:
            print("  id", r.id, "metric gpu/oracle", float(ex.conf[r.id]), r.metric, "max|dz|",
                  float(np.max(np.abs(lg[r.id] - r.logits))), "max|z|", float(np.max(np.abs(r.logits))),
                  "label", int(ex.label[r.id]), r.label)
    got = id_out[:int(n_surv.item())].cpu().tolist()
    for i in surv:
        if i in got:
            g, o = to64(x_out[got.index(i), 0]), h[surv.index(i)]
            print("  surv", i, "mean|dh|", float(np.mean(np.abs(g - o))), "max|dh|", float(np.max(np.abs(g - o))),
                  "mean|h|", float(np.mean(np.abs(o))))
