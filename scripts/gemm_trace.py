"""Per-tile timeline of the layer GEMM (e3_debug_gemm_trace): MMA vs epilogue, per CTA.

    python scripts/gemm_trace.py M N K epi
"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import _lib, api  # noqa: E402

M, N, K = (int(v) for v in sys.argv[1:4])
epi = sys.argv[4] if len(sys.argv) > 4 else "bias"
dev = "cuda:0"
A = torch.randn(M, K, device=dev).to(torch.bfloat16)
W = (torch.randn(N, K, device=dev) * K ** -0.5).to(torch.bfloat16)
bias = torch.randn(N, device=dev).to(torch.bfloat16)
R = torch.randn(M, N, device=dev).to(torch.bfloat16)
C = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
buf = torch.zeros(148 * 16 * 6 + 296 * 8 * 6, dtype=torch.int64, device=dev)
run = lambda: api.ops.gemm(A, W, bias, epi, resid=R if epi == "bias_resid" else None, out=C)  # noqa: E731
for _ in range(3):
    run()
torch.cuda.synchronize()
_lib.lib.e3_debug_gemm_trace(buf.data_ptr())
run()
torch.cuda.synchronize()
_lib.lib.e3_debug_gemm_trace(None)
t = buf.cpu().numpy()[: 148 * 16 * 6].reshape(148, 16, 6).astype(np.float64)
valid = t[:, :, 2] > 0
has_mma = t[:, :, 1] > 0
t0 = t[t > 0].min()
t = (t - t0) / 1000.0   # us
end = np.where(valid, np.maximum(t[:, :, 3], t[:, :, 5]), 0).max()
print(f"{M}x{N}x{K} {epi}: kernel span (first MMA start .. last epilogue end) {end:.2f} us")
for cta in (0, 1, 2, 3, 146, 147):
    print(f"CTA {cta}:")
    for i in range(16):
        if not valid[cta, i]:
            break
        r = t[cta, i]
        mma = f"mma {r[0]:6.2f}-{r[1]:6.2f}" if has_mma[cta, i] else "mma (peer)       "
        print(f"  tile {i:2d}: {mma}  epi4 {r[2]:6.2f}-{r[3]:6.2f} ({r[3] - r[2]:5.2f})  "
              f"epi11 {r[4]:6.2f}-{r[5]:6.2f} ({r[5] - r[4]:5.2f})")
ep = np.where(valid, t[:, :, 3] - t[:, :, 2], np.nan)
mm = np.where(valid & has_mma, t[:, :, 1] - t[:, :, 0], np.nan)
print(f"median epilogue (warp 4) per tile {np.nanmedian(ep):.2f} us; median MMA issue span per tile "
      f"{np.nanmedian(mm):.2f} us")
