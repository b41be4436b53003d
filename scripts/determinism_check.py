"""Run the same pipeline job several times in one process and compare the exit
records bit for bit (any difference means a race).
python scripts/determinism_check.py [cfg] [N] [reps]"""
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
DEV = "cuda:0"
cfg = e3data.get(name)
tau = e3data.tau_for(cfg)
model = api.DeviceModel(cfg, e3data.make_weights(cfg), DEV)
X = torch.from_numpy(e3data.make_inputs(cfg, range(N))).to(torch.bfloat16).to(DEV)
pipe = api.Pipeline(model, api.make_plan(cfg, Plan.per_ramp(cfg.ramp_layers).bounds, tau))
base = None
for r in range(reps):
    ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, DEV)
    pipe.run(X, torch.arange(N, dtype=torch.int64, device=DEV), ex)
    torch.cuda.synchronize()
    el, lg = ex.exit_layer.cpu().numpy(), ex.logits.cpu().numpy()
    hist = [round(float((el == l).mean()), 4) for l in cfg.ramp_layers]
    if base is None:
        base = (el, lg)
        print(name, "rep 0 hist", hist, flush=True)
    else:
        d_el = int((el != base[0]).sum())
        d_lg = int((lg != base[1]).any(axis=1).sum())
        print(name, f"rep {r}: exit_layer diffs {d_el}, logit rows differing {d_lg}", hist, flush=True)
