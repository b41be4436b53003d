"""End-to-end GPU pipeline vs oracle: distribution of logit gaps and of
exit-decision mismatches as a function of the oracle margin."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
import oracle  # noqa: E402
from oracle.pipeline_sim import Plan  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

DEV = "cuda:0"
name = sys.argv[1] if len(sys.argv) > 1 else "tiny"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 256
n_or = int(sys.argv[3]) if len(sys.argv) > 3 else N
cfg = e3data.get(name)
tau = cfg.tau
if tau is None:
    from oracle.calibrate import load_tau
    tau = load_tau(cfg)
W = e3data.make_weights(cfg)
model = api.DeviceModel(cfg, W, DEV)
X = e3data.make_inputs(cfg, range(N))
ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, DEV)
pipe = api.Pipeline(model, api.make_plan(cfg, Plan.per_ramp(cfg.ramp_layers).bounds, tau))
pipe.run(api.to_bf16(X, DEV), torch.arange(N, dtype=torch.int64, device=DEV), ex)
el = ex.exit_layer.cpu().numpy()
lg = ex.logits.cpu().numpy()
print("exit hist", np.bincount(el, minlength=cfg.layers) / N)
t = time.time()
recs = oracle.run(cfg, W, X[:n_or], tau=tau, mode="bf16")
print("oracle s", time.time() - t)
margins = np.array([r.margin for r in recs])
mism = np.array([el[i] != r.exit_layer for i, r in enumerate(recs)])
gap = np.array([np.abs(lg[i] - r.logits).max() for i, r in enumerate(recs) if el[i] == r.exit_layer])
print("margin quantiles", np.quantile(margins, [0.01, 0.05, 0.1, 0.5]))
print("frac margin<=1e-3", np.mean(margins <= 1e-3), "<=1e-2", np.mean(margins <= 1e-2))
print("mismatches", mism.sum(), "margins of mismatches", np.sort(margins[mism])[:20])
print("logit gap quantiles", np.quantile(gap, [0.5, 0.9, 0.99, 1.0]))
recs64 = oracle.run(cfg, W, X[:min(n_or, 64)], tau=tau, mode="fp64")
gap64 = np.array([np.abs(lg[i] - r.logits).max() for i, r in enumerate(recs64) if el[i] == r.exit_layer])
print("vs fp64 logit gap quantiles", np.quantile(gap64, [0.5, 0.9, 0.99, 1.0]))
