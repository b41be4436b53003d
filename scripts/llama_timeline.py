"""Kernel timeline of graph-replayed Llama-7B decode split runs (T = 64
tokens, 513 cache positions, a 4-layer split ending in the LM-head ramp):
every kernel instance in order, with its CTA count, first entry, last release
and last end (us), and the idle gap before it.

    python scripts/llama_timeline.py [layers]
"""
import dataclasses
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import _lib, api  # noqa: E402

DEV = "cuda:0"
nl = int(sys.argv[1]) if len(sys.argv) > 1 else 4
cfg = dataclasses.replace(e3data.get("lm"), layers=nl, ramp_layers=(nl - 1,), exit_profile=None, tau=(0.5,))
B = cfg.batch
layers = [e3data.make_layer(cfg, l) for l in range(nl)]
W = {"layers": layers, "ramps": [e3data.make_ramp(cfg, 0)]}
max_ctx = cfg.ctx + 1
cache = api.KVCache(cfg, B, max_ctx, B, DEV)
cache.slot_of_id.copy_(torch.arange(B, dtype=torch.int32))
cache.pos_of_slot.copy_(torch.full((B,), cfg.ctx, dtype=torch.int32))
model = api.DeviceModel(cfg, W, DEV, kv=cache)
split = api.Split(model, api.split_desc(cfg, 0, nl, cfg.tau))
x = api.to_bf16(e3data.make_inputs(cfg, range(B), seed=6), DEV)
ids = torch.arange(B, dtype=torch.int64, device=DEV)
x_out = torch.zeros_like(x)
id_out = torch.zeros_like(ids)
n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, DEV)
run = lambda: split.run(x, ids, x_out, id_out, n_surv, ex)
for _ in range(2):
    run()
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    with torch.cuda.graph(g, stream=s):
        run()
        run()
g.replay()
torch.cuda.synchronize()
buf = torch.zeros(1 + 4 * 32768, dtype=torch.int64, device=DEV)
_lib.lib.e3_debug_timeline(buf.data_ptr())
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
g.replay()
e1.record()
torch.cuda.synchronize()
_lib.lib.e3_debug_timeline(None)
b = buf.cpu().numpy()
n = min(int(b[0]), 32768)
r = b[1:1 + 4 * n].reshape(n, 4)
kid = (r[:, 0] & 0xFFFF).astype(int)
t = r[:, 1:].astype(np.float64)
keep = (kid == 8600) | (kid == 8700) | (kid == 8710) | ((kid >= 8100) & (kid < 8200))
kid, t = kid[keep], t[keep]
t = (t - t.min()) / 1000.0
NAMES = {8600: "attn_dec", 8700: "rmsnorm", 8710: "reduce+rmsnorm", 8105: "gemm PARTIAL (O/down)", 8100: "gemm STORE", 8101: "gemm RESID (O/down)", 8102: "gemm SWIGLU",
         8103: "gemm QKV+RoPE", 8104: "gemm LM head"}
inst = []
for k in np.unique(kid):
    sel = np.where(kid == k)[0]
    sel = sel[np.argsort(t[sel, 0])]
    start = 0
    for i in range(1, len(sel) + 1):
        # a new instance when the entry jumps past the previous instance's end
        if i == len(sel) or t[sel[i], 0] > t[sel[start:i], 2].max() + 0.2 and t[sel[i], 1] > t[sel[start:i], 2].max():
            inst.append((k, sel[start:i]))
            start = i
inst.sort(key=lambda p: np.max(t[p[1], 2]))
print(f"Llama-7B decode split of {nl} layers, B={B}, graph time {e0.elapsed_time(e1) * 1000 / 2:.1f} us per run")
print("%-22s %6s %8s %8s %8s %8s %7s" % ("kernel", "CTAs", "entry0", "rel_last", "end_last", "busy", "gap"))
prev = None
tot = {}
for k, sel in inst:
    e, rl, en = t[sel, 0], t[sel, 1], t[sel, 2]
    busy = en.max() - (rl.max() if prev is None else max(prev, rl.min()))
    gap = 0.0 if prev is None else rl.min() - prev
    print("%-22s %6d %8.2f %8.2f %8.2f %8.2f %7.2f" % (NAMES.get(k, str(k)), len(sel), e.min(), rl.max(), en.max(),
                                                       en.max() - (prev if prev is not None else rl.min()), gap))
    tot[NAMES.get(k, str(k))] = tot.get(NAMES.get(k, str(k)), 0) + en.max() - (prev if prev is not None else rl.min())
    prev = en.max()
print("per kind (end-to-end share of the timeline):", {k: round(v, 1) for k, v in tot.items()})
