"""Kernel timeline of the BB pipeline itself (e3_debug_timeline around one
e3_pipeline_run; the buffer holds the first 32768 CTA records, ~30 split runs).

    python scripts/pipeline_timeline.py [config] [inputs] [first_run] [n_runs]

Prints, for n_runs consecutive split runs starting at first_run, every kernel
instance in order of its last CTA's release: CTAs, entry / release / end of
the first and last CTA relative to the window start (us), and the per-run
period (QKV GEMM release to the next one).  Run it with and without
E3_NO_TAIL_OVERLAP=1 to see where the last ramp + compaction land.
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import _lib, api  # noqa: E402

NAMES = {3: "layernorm", 4: "ramp(all CTAs)", 5: "ramp decision", 6: "ln_compact", 7: "gemm_ln (O+LN1)",
         9: "ramp_vit", 74: "ramp2", 70: "ramp+compact (fused)"}


def name(k):
    if k in NAMES:
        return NAMES[k]
    if 1000 <= k < 2000:
        return "gemm<BN=%d,epi=%d>" % ((k - 1000) // 64 * 64, (k - 1000) % 64)
    if 2000 <= k < 3000:
        return "attention<%d>" % (k - 2000)
    return str(k)


DEV = "cuda:0"
args = sys.argv[1:]
cfg = e3data.get(args[0] if args and not args[0].isdigit() else "bb")
nums = [int(a) for a in args if a.isdigit()]
n = nums[0] if nums else 4096
first = nums[1] if len(nums) > 1 else 8
nruns = nums[2] if len(nums) > 2 else 6
tau = e3data.tau_for(cfg)
model = api.DeviceModel(cfg, e3data.make_weights(cfg), DEV)
X = api.to_bf16(e3data.make_inputs(cfg, range(n)), DEV)
ids = torch.arange(n, dtype=torch.int64, device=DEV)
bounds = (0,) + tuple(l + 1 for l in cfg.ramp_layers)
pipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau))
ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV, logits=False)
for _ in range(2):
    pipe.run(X, ids, ex)
torch.cuda.synchronize()
buf = torch.zeros(1 + 4 * 32768, dtype=torch.int64, device=DEV)
_lib.lib.e3_debug_timeline(buf.data_ptr())
pipe.run(X, ids, ex)
torch.cuda.synchronize()
_lib.lib.e3_debug_timeline(None)
b = buf.cpu().numpy()
cnt = min(int(b[0]), 32768)
r = b[1:1 + 4 * cnt].reshape(cnt, 4)
kid = (r[:, 0] & 0xFFFF).astype(int)
t = r[:, 1:].astype(np.float64)
t = (t - t.min()) / 1000.0
inst = []
for k in np.unique(kid):
    sel = np.where(kid == k)[0]
    sel = sel[np.argsort(t[sel, 0])]
    start = 0
    for i in range(1, len(sel) + 1):
        if i == len(sel) or t[sel[i], 0] - t[sel[i - 1], 0] > 3.0:
            inst.append((k, sel[start:i]))
            start = i
inst.sort(key=lambda p: np.max(t[p[1], 1]))
# the QKV GEMM is the encoder layer's only bias-only (epilogue 0) GEMM
qkv = [i for i, (k, _) in enumerate(inst) if 1000 <= k < 2000 and (k - 1000) % 64 == 0 and len(_) >= 64]
if len(qkv) < first + nruns + 1:
    first = max(0, len(qkv) - nruns - 1)
lo, hi = qkv[first], qkv[min(first + nruns, len(qkv) - 1)]
t0 = np.max(t[inst[lo][1], 1])
print(f"{cfg.name}: pipeline run of {n} inputs, split runs {first}..{first + nruns - 1} "
      f"(tail overlap {'off' if os.environ.get('E3_NO_TAIL_OVERLAP') else 'on'}); us from the window start")
print("%-24s %5s %8s %8s %8s %8s %8s" % ("kernel", "CTAs", "entry0", "rel0", "rel_last", "end0", "end_last"))
for k, sel in inst[lo:hi]:
    e, rl, en = t[sel, 0] - t0, t[sel, 1] - t0, t[sel, 2] - t0
    print("%-24s %5d %8.2f %8.2f %8.2f %8.2f %8.2f" % (name(k), len(sel), e.min(), rl.min(), rl.max(), en.min(),
                                                        en.max()))
per = [np.max(t[inst[qkv[i + 1]][1], 1]) - np.max(t[inst[qkv[i]][1], 1]) for i in range(first, first + nruns)
       if i + 1 < len(qkv)]
print("period per split run (QKV release to QKV release): " + " ".join("%.1f" % p for p in per) +
      "  mean %.2f us" % np.mean(per))
