"""Per-segment phases of the stream-K decode GEMM (one call after a flush):
for each CTA, the SM it ran on, when its mainloop finished, and for each
segment the accumulator-ready -> partial published (ticket) -> reduced ->
epilogue-end times.

    python scripts/dec_segments.py [qkv|gate_up|lm_head]
"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import _lib, api  # noqa: E402

DEV = "cuda:0"
T = 64
SH = {"qkv": (12288, 4096, "store"), "o": (4096, 4096, "resid"), "gate_up": (11008, 4096, "swiglu"),
      "down": (4096, 11008, "resid"), "lm_head": (32000, 4096, "store")}
for name in (sys.argv[1:] or ["qkv", "gate_up"]):
    N, K, epi = SH[name]
    X = torch.randn(T, K, device=DEV).to(torch.bfloat16)
    W = torch.randn(N, K, device=DEV).to(torch.bfloat16)
    W2 = torch.randn(N, K, device=DEV).to(torch.bfloat16) if epi == "swiglu" else None
    R = torch.randn(T, N, device=DEV).to(torch.bfloat16)
    out = torch.empty(T, N, device=DEV, dtype=torch.bfloat16)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=DEV)
    run = lambda: api.ops.dec_gemm(X, W, epi, W2=W2, resid=R if epi == "resid" else None, out=out)
    for _ in range(3):
        run()
    flush.zero_()
    torch.cuda.synchronize()
    buf = torch.zeros(1 + 4 * 32768, dtype=torch.int64, device=DEV)
    _lib.lib.e3_debug_timeline(buf.data_ptr())
    run()
    torch.cuda.synchronize()
    _lib.lib.e3_debug_timeline(None)
    b = buf.cpu().numpy()
    n = int(b[0])
    r = b[1:1 + 4 * n].reshape(n, 4)
    kid = (r[:, 0] & 0xFFFF).astype(int)
    bid = ((r[:, 0] >> 16) & 0xFFFFFFFF).astype(int)
    sm = (r[:, 0] >> 48).astype(int)
    t = r[:, 1:].astype(np.float64)
    t0 = t[(kid >= 8100) & (kid < 8200), 0].min()
    t = (t - t0) / 1000
    M = (kid >= 8000) & (kid < 8100)
    print(f"{name}: {M.sum()} CTAs")
    for lab, k0 in (("partial only", 8300), ("reduced", 8400), ("whole", 8500)):
        s = (kid >= k0) & (kid < k0 + 100)
        if s.sum():
            d1 = t[s, 1] - t[s, 0]
            d2 = t[s, 2] - t[s, 1]
            print(f"  {lab:12s} segments {s.sum():4d}: acc->{'ticket' if k0 == 8300 else 'reduced':7s} "
                  f"p50 {np.median(d1):5.2f} max {d1.max():5.2f} | ->end p50 {np.median(d2):5.2f} max {d2.max():5.2f}")
    last = t[M, 1]
    end = t[M, 2]
    print(f"  mainloop done p0/p50/p100 {np.percentile(last, [0, 50, 100]).round(2)}  end {np.percentile(end, [0, 50, 100]).round(2)}")
    o = np.argsort(last)
    print("  fastest (sm, bid, done):", [(int(sm[M][i]), int(bid[M][i]), round(last[i], 1)) for i in o[:8]])
    print("  slowest (sm, bid, done):", [(int(sm[M][i]), int(bid[M][i]), round(last[i], 1)) for i in o[-8:]])
    smm = sm[M]
    for lo, hi in ((0, 74), (74, 148)):
        sel = (smm >= lo) & (smm < hi)
        print(f"  SMs {lo}-{hi - 1}: mainloop done median {np.median(last[sel]):.2f} max {last[sel].max():.2f}")
    # per-CTA: mainloop done vs the CTA's segment structure
    seg = {}
    for k0, lab in ((8300, "P"), (8400, "R"), (8500, "W")):
        s_ = (kid >= k0) & (kid < k0 + 100)
        for b_, tt in zip(bid[s_], t[s_, 0]):
            seg.setdefault(int(b_), []).append((round(tt, 1), lab))
    rows_ = sorted(zip(last, bid[M], sm[M]))
    print("  CTA (mainloop done, bid, sm, segments acc-ready/kind):")
    for L_, b_, s_ in rows_[:4] + rows_[len(rows_) // 2 - 2:len(rows_) // 2 + 2] + rows_[-6:]:
        print("    %6.2f %4d %4d %s" % (L_, b_, s_, sorted(seg.get(int(b_), []))))
