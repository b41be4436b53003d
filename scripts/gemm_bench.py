"""Time the layer GEMM shapes of EE-BERT-base: our tcgen05 kernel (e3_op_gemm)
vs torch.matmul (cuBLAS) on the same shapes, CUDA events, L2-warm."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

dev = "cuda:0"
M = 64 * 128
shapes = [("qkv", 2304, 768, "bias"), ("o", 768, 768, "bias_resid"), ("ffn1", 3072, 768, "bias_gelu"),
          ("ffn2", 768, 3072, "bias_resid")]
if len(sys.argv) > 1:
    M = int(sys.argv[1])


def timeit(fn, n=50):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1000


for name, N, K, epi in shapes:
    A = torch.randn(M, K, device=dev).to(torch.bfloat16)
    W = (torch.randn(N, K, device=dev) * K ** -0.5).to(torch.bfloat16)
    bias = torch.randn(N, device=dev).to(torch.bfloat16)
    R = torch.randn(M, N, device=dev).to(torch.bfloat16)
    C = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
    t_ours = timeit(lambda: api.ops.gemm(A, W, bias, epi, resid=R if epi == "bias_resid" else None, out=C))
    t_cublas = timeit(lambda: torch.matmul(A, W.t(), out=C))
    fl = 2 * M * N * K
    print(f"{name:5s} M={M} N={N} K={K}: ours {t_ours:7.1f} us ({fl / t_ours / 1e6:6.0f} TF/s)   "
          f"cuBLAS (no epilogue) {t_cublas:7.1f} us ({fl / t_cublas / 1e6:6.0f} TF/s)")
