"""Back-to-back decode GEMM calls (graph-replayed, 4 weight copies so every
call streams from HBM) with the per-CTA timeline: for each call, CTA entry,
release from griddepcontrol.wait, first / last accumulator ready and end
(min / median / max, us from the first call's first entry).

    python scripts/dec_timeline_seq.py [qkv|o|gate_up|down|lm_head]
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
CALLS = 4
for name in (sys.argv[1:] or ["o", "qkv"]):
    N, K, epi = SH[name]
    X = torch.randn(T, K, device=DEV).to(torch.bfloat16)
    Ws = [torch.randn(N, K, device=DEV).to(torch.bfloat16) for _ in range(CALLS)]
    W2s = [torch.randn(N, K, device=DEV).to(torch.bfloat16) for _ in range(CALLS)] if epi == "swiglu" else None
    R = torch.randn(T, N, device=DEV).to(torch.bfloat16)
    out = torch.empty(T, N, device=DEV, dtype=torch.bfloat16)

    def run():
        for i in range(CALLS):
            api.ops.dec_gemm(X, Ws[i], epi, W2=W2s[i] if W2s else None, resid=R if epi == "resid" else None, out=out)

    run()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
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
    n = int(b[0])
    r = b[1:1 + 4 * n].reshape(n, 4)
    kid = (r[:, 0] & 0xFFFF).astype(int)
    bid = ((r[:, 0] >> 16) & 0xFFFFFFFF).astype(int)
    t = r[:, 1:].astype(np.float64)
    A = np.where((kid >= 8100) & (kid < 8200))[0]
    M = np.where((kid >= 8000) & (kid < 8100))[0]
    t0 = t[A, 0].min()
    G = len(A) // CALLS
    # pair the j-th 8100 record of a CTA index with its j-th 8000 record
    rows = []
    for c in np.unique(bid[A]):
        a_ = A[bid[A] == c]
        m_ = M[bid[M] == c]
        a_ = a_[np.argsort(t[a_, 0])]
        m_ = m_[np.argsort(t[m_, 2])]
        for j in range(min(len(a_), len(m_))):
            rows.append((j, t[a_[j], 0], t[a_[j], 1], t[m_[j], 0], t[m_[j], 1], t[m_[j], 2]))
    rows = np.array(rows)
    f = lambda v: "%6.2f/%6.2f/%6.2f" % tuple(np.percentile((v - t0) / 1000, [0, 50, 100]))
    print(f"{name}: {CALLS} calls, {G} CTAs each, graph time {e0.elapsed_time(e1) * 1000 / CALLS:.2f} us per call")
    for j in range(CALLS):
        s = rows[rows[:, 0] == j]
        print(f"  call {j}: entry {f(s[:, 1])} rel {f(s[:, 2])} first acc {f(s[:, 3])} last acc {f(s[:, 4])} "
              f"end {f(s[:, 5])}")
