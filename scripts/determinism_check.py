"""Run the same pipeline job several times in one process and compare the exit
records bit for bit (any difference means a race).
python scripts/determinism_check.py [cfg] [N] [reps] [per-ramp|cut6] [bf16|fp32]"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
from oracle.pipeline_sim import Plan  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "bl"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 768
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 4
plan = sys.argv[4] if len(sys.argv) > 4 else "per-ramp"
dtype = sys.argv[5] if len(sys.argv) > 5 else "bf16"
DEV = "cuda:0"
cfg = e3data.get(name)
tau = e3data.tau_for(cfg)
if cfg.arch == "llama":
    max_ctx = cfg.ctx + 1
    kv = api.KVCache(cfg, N, max_ctx, N, DEV, dtype=dtype)
    for l in range(cfg.layers):
        k, v = e3data.make_kv(cfg, l, range(N), max_ctx)
        kv.k[l].copy_(torch.from_numpy(k).to(kv.k[l].dtype))
        kv.v[l].copy_(torch.from_numpy(v).to(kv.v[l].dtype))
    kv.slot_of_id.copy_(torch.arange(N, dtype=torch.int32))
    kv.pos_of_slot.copy_(torch.tensor([cfg.ctx - (s % 5) for s in range(N)], dtype=torch.int32))
    W = {"layers": [e3data.make_layer(cfg, l) for l in range(cfg.layers)],
         "ramps": [e3data.make_ramp(cfg, 0)] * cfg.n_ramps}
    model = api.DeviceModel(cfg, W, DEV, kv=kv)
    X = torch.from_numpy(e3data.make_inputs(cfg, range(N), seed=5)).to(DEV)
else:
    model = api.DeviceModel(cfg, e3data.make_weights(cfg), DEV)
    X = torch.from_numpy(e3data.make_inputs(cfg, range(N))).to(DEV)
X = X.to(torch.bfloat16) if dtype == "bf16" else X.float()
bounds = Plan.per_ramp(cfg.ramp_layers).bounds if plan == "per-ramp" else (0, 6, cfg.layers)
pipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau, dtype=dtype))
base = None
bad = 0
for r in range(reps):
    ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, DEV)
    if cfg.test == "patience":
        ex.state.zero_()
    pipe.run(X, torch.arange(N, dtype=torch.int64, device=DEV), ex)
    torch.cuda.synchronize()
    el, lg = ex.exit_layer.cpu().numpy(), ex.logits.cpu().numpy()
    hist = [round(float((el == l).mean()), 4) for l in cfg.ramp_layers]
    if base is None:
        base = (el, lg)
        print(name, plan, dtype, "rep 0 hist", hist, flush=True)
    else:
        d_el = int((el != base[0]).sum())
        d_lg = int((lg != base[1]).any(axis=1).sum())
        bad += d_el + d_lg > 0
        print(name, f"rep {r}: exit_layer diffs {d_el}, logit rows differing {d_lg}", flush=True)
print(name, plan, dtype, "NONDETERMINISTIC" if bad else "deterministic", f"({reps} repeats)", flush=True)
