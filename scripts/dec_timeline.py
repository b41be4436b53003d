"""Per-CTA phase timeline of the decode GEMMs (e3_debug_timeline): entry,
release from griddepcontrol.wait, first / last accumulator ready (mainloop),
end of the epilogue, for the Llama-7B decode shapes at T = 64.

    python scripts/dec_timeline.py
"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import _lib, api  # noqa: E402

DEV = "cuda:0"
T = 64
shapes = [("qkv", 12288, 4096, "store"), ("o", 4096, 4096, "resid"), ("gate_up", 11008, 4096, "swiglu"),
          ("down", 4096, 11008, "resid"), ("lm_head", 32000, 4096, "store")]
for name, N, K, epi in shapes:
    X = torch.randn(T, K, device=DEV).to(torch.bfloat16)
    W = torch.randn(N, K, device=DEV).to(torch.bfloat16)
    W2 = torch.randn(N, K, device=DEV).to(torch.bfloat16) if epi == "swiglu" else None
    R = torch.randn(T, N, device=DEV).to(torch.bfloat16)
    out = torch.empty(T, N, device=DEV, dtype=torch.bfloat16)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=DEV)

    def run():
        api.ops.dec_gemm(X, W, epi, W2=W2, resid=R if epi == "resid" else None, out=out)

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
    t = r[:, 1:].astype(np.float64)
    a = t[(kid >= 8100) & (kid < 8200)]
    m = t[(kid >= 8000) & (kid < 8100)]
    red = t[kid >= 8200]
    t0 = a[:, 0].min()
    f = lambda v: "%6.2f/%6.2f/%6.2f" % tuple(np.percentile((v - t0) / 1000, [0, 50, 100]))
    print(f"{name:8s} CTAs {len(a)}  entry {f(a[:, 0])}  released {f(a[:, 1])}  first acc {f(m[:, 0])}  "
          f"last acc {f(m[:, 1])}  end {f(m[:, 2])}  (us, min/median/max)")
    if len(red):
        print(f"         {len(red)} tile reductions: start {f(red[:, 0])}  end {f(red[:, 2])}  "
              f"duration median {np.median(red[:, 2] - red[:, 0]) / 1000:.2f} us")
    if name == "o" or "-v" in sys.argv:
        bid = ((r[:, 0] >> 16) & 0xFFFFFFFF).astype(int)
        mm = (kid >= 8000) & (kid < 8100)
        order = np.argsort(-t[mm][:, 2])[:8]
        rb = bid[kid >= 8200]
        for i in order:
            b_ = bid[mm][i]
            tt = (t[mm][i] - t0) / 1000
            rr = [(x - t0) / 1000 for x in t[(kid >= 8200) & (bid == b_)][:, [0, 2]].ravel()]
            print(f"   CTA {b_:3d}: first acc {tt[0]:6.2f} last acc {tt[1]:6.2f} end {tt[2]:6.2f} reductions "
                  + " ".join(f"{v:6.2f}" for v in rr))
