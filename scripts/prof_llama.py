"""One EE-Llama-7B-shaped split (layers [0, n)) on a full batch of 64 tokens
(for ncu captures of the decode kernels).

    python scripts/prof_llama.py [n_runs] [layers]
"""
import dataclasses
import sys

import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

n_runs = int(sys.argv[1]) if len(sys.argv) > 1 else 3
nl = int(sys.argv[2]) if len(sys.argv) > 2 else 2
DEV = "cuda:0"
cfg = dataclasses.replace(e3data.get("lm"), layers=nl, ramp_layers=(nl - 1,), exit_profile=None, tau=(0.5,))
B = cfg.batch
ramp = e3data.make_ramp(cfg, 0)
kv = api.KVCache(cfg, B, cfg.ctx + 1, B, DEV)
for t in kv.k + kv.v:
    t[:, :, :cfg.ctx].normal_()
kv.slot_of_id.copy_(torch.arange(B, dtype=torch.int32))
model = api.DeviceModel(cfg, {"layers": (e3data.make_layer(cfg, l) for l in range(nl)), "ramps": [ramp]}, DEV, kv=kv)
X = api.to_bf16(e3data.make_inputs(cfg, range(B)), DEV)
ids = torch.arange(B, dtype=torch.int64, device=DEV)
split = api.Split(model, api.split_desc(cfg, 0, nl, cfg.tau))
x_out = torch.empty_like(X)
id_out = torch.empty_like(ids)
n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, DEV)
for _ in range(n_runs):
    split.run(X, ids, x_out, id_out, n_surv, ex)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    split.run(X, ids, x_out, id_out, n_surv, ex)
e1.record()
torch.cuda.synchronize()
print(f"llama split of {nl} layer(s), B={B}: {e0.elapsed_time(e1) / 10 * 1000:.1f} us per run")
