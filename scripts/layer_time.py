"""Graph-timed single split runs of EE-BERT-base (full batch B = 64, L2-warm).

    python scripts/layer_time.py [layers_per_split ...]
Prints the time of one split run of 1 layer + ramp + compaction, and of k layers.
"""
import sys

import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

DEV = "cuda:0"
cfg = e3data.get(sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].isdigit() else "bb")
tau = e3data.tau_for(cfg)
W = e3data.make_weights(cfg)
model = api.DeviceModel(cfg, W, DEV)
B = cfg.batch
X = api.to_bf16(e3data.make_inputs(cfg, range(B)), DEV)
ids = torch.arange(B, dtype=torch.int64, device=DEV)
for nl in [int(a) for a in sys.argv[1:] if a.isdigit()] or [1, 2, 12]:
    split = api.Split(model, api.split_desc(cfg, 0, nl, tau))
    x_out = torch.empty_like(X)
    id_out = torch.empty_like(ids)
    n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
    ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, DEV)
    for _ in range(3):
        split.run(X, ids, x_out, id_out, n_surv, ex)
    torch.cuda.synchronize()
    n = 20
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            for _ in range(n):
                split.run(X, ids, x_out, id_out, n_surv, ex)
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    print(f"{cfg.name}: split of {nl} layer(s), B={B}: {e0.elapsed_time(e1) / n * 1000:.1f} us per run "
          f"({e0.elapsed_time(e1) / n * 1000 / nl:.1f} us per layer)")
