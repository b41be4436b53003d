"""Run EE-BERT-base splits on full batches (for ncu captures of each kernel).

    python scripts/prof_split.py [n_runs] [layers_per_split]
"""
import sys

import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

n_runs = int(sys.argv[1]) if len(sys.argv) > 1 else 3
nl = int(sys.argv[2]) if len(sys.argv) > 2 else 1
DEV = "cuda:0"
cfg = e3data.get("bb")
tau = e3data.tau_for(cfg)
W = e3data.make_weights(cfg)
model = api.DeviceModel(cfg, W, DEV)
B = cfg.batch
X = api.to_bf16(e3data.make_inputs(cfg, range(B)), DEV)
ids = torch.arange(B, dtype=torch.int64, device=DEV)
split = api.Split(model, api.split_desc(cfg, 0, nl, tau))
x_out = torch.empty_like(X)
id_out = torch.empty_like(ids)
n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, DEV)
for _ in range(n_runs):
    split.run(X, ids, x_out, id_out, n_surv, ex)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20):
    split.run(X, ids, x_out, id_out, n_surv, ex)
e1.record()
torch.cuda.synchronize()
print(f"split of {nl} layer(s), B={B}: {e0.elapsed_time(e1) / 20 * 1000:.1f} us per run")
