"""Kernel timeline of graph-replayed EE-BERT split runs (e3_debug_timeline).

    python scripts/timeline.py [config] [layers_per_split] [runs]

For every kernel launch of the middle run: when its first CTA became resident
(entry), when the first / last CTA was released by griddepcontrol.wait, and
when the first / last CTA finished, relative to the previous run's end.  The
gap between one kernel's last end and the next kernel's last release is the
dependency hand-off cost; entry -> release is the prologue that overlapped.
"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import _lib, api  # noqa: E402

NAMES = {77: "O+LN: tfull|stats|stored", 78: "O+LN: resid|pass1|rec", 79: "O+LN: pre-sync|.|rec", 9: "ramp_vit", 91: "vit ramp: ln|cls|end", 3: "layernorm", 4: "ramp(all CTAs)", 5: "ramp decision", 6: "ln_compact", 7: "gemm_ln (O+LN1)", 40: "ramp: cls ready|partials|sync", 41: "decide: synced|computed|tl5", 60: "compact: scan done", 70: "ramp+compact (fused)", 71: "fused: pdl|decided|end", 72: "fused slice: rel|rows|computed", 73: "fused decider start", 74: "ramp2", 75: "ramp2 slice: rel|computed|end", 76: "ramp2 decider: rel|computed|end"}


def name(kid):
    if kid in NAMES:
        return NAMES[kid]
    if 1000 <= kid < 2000:
        return "gemm<BN=%d,epi=%d>" % ((kid - 1000) // 64 * 64, (kid - 1000) % 64)
    if 2000 <= kid < 3000:
        return "attention<%d>" % (kid - 2000)
    return str(kid)


DEV = "cuda:0"
args = [a for a in sys.argv[1:]]
cfg = e3data.get(args[0] if args and not args[0].isdigit() else "bb")
nums = [int(a) for a in args if a.isdigit()]
nl = nums[0] if nums else 1
runs = nums[1] if len(nums) > 1 else 3
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
for _ in range(3):
    split.run(X, ids, x_out, id_out, n_surv, ex)
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    with torch.cuda.graph(g, stream=s):
        for _ in range(runs):
            split.run(X, ids, x_out, id_out, n_surv, ex)
g.replay()
torch.cuda.synchronize()
buf = torch.zeros(1 + 4 * 32768, dtype=torch.int64, device=DEV)
_lib.lib.e3_debug_timeline(buf.data_ptr())
g.replay()
torch.cuda.synchronize()
_lib.lib.e3_debug_timeline(None)
b = buf.cpu().numpy()
n = int(b[0])
r = b[1:1 + 4 * n].reshape(n, 4)
kid = (r[:, 0] & 0xFFFF).astype(int)
t = r[:, 1:].astype(np.float64)
t0 = t.min()
t = (t - t0) / 1000.0
# instances: per kernel id, split by gaps in entry time
inst = []
for k in np.unique(kid):
    sel = np.where(kid == k)[0]
    sel = sel[np.argsort(t[sel, 0])]
    start = 0
    for i in range(1, len(sel) + 1):
        if i == len(sel) or t[sel[i], 0] - t[sel[i - 1], 0] > 3.0:
            inst.append((k, sel[start:i]))
            start = i
inst.sort(key=lambda p: np.median(t[p[1], 1]))
print(f"{cfg.name}: {runs} graph-replayed split runs of {nl} layer(s), B={B}; times in us")
print("%-22s %5s %8s %8s %8s %8s %8s %8s" % ("kernel", "CTAs", "entry0", "rel0", "rel_last", "end0", "end_last",
                                            "busy"))
prev_end = None
for k, sel in inst:
    e, rl, en = t[sel, 0], t[sel, 1], t[sel, 2]
    busy = en.max() - rl.max()
    print("%-22s %5d %8.2f %8.2f %8.2f %8.2f %8.2f %8.2f%s" % (
        name(k), len(sel), e.min(), rl.min(), rl.max(), en.min(), en.max(), en.max() - rl.min(),
        "" if prev_end is None else "   handoff %.2f" % (rl.max() - prev_end)))
    prev_end = en.max()
print("total span %.2f us, per run %.2f us" % (t.max(), t.max() / runs))
