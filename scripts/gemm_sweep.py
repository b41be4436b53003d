"""GEMM diagnostics: epilogue cost and wave quantization of e3_op_gemm vs cuBLAS (graph-timed, L2-warm)."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402


def timeit(fn, n=50):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(n):
            fn()
    g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    g.replay()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1000


dev = "cuda:0"
cases = [(8192, 3072, 768, "bias"), (8192, 3072, 768, "bias_gelu"),
         (8192, 768, 3072, "bias"), (8192, 768, 3072, "bias_resid"),
         (8192, 768, 768, "bias"), (8192, 768, 768, "bias_resid"),
         (18944, 768, 3072, "bias"), (18944, 768, 768, "bias"),   # 296 tiles of 256x192: 4 full waves
         (9472, 768, 3072, "bias"), (9472, 3072, 768, "bias"), (8192, 2304, 768, "bias")]
if len(sys.argv) > 1:   # e.g. 8192,3072,768,bias_gelu
    cases = [tuple(int(v) if v.isdigit() else v for v in a.split(',')) for a in sys.argv[1:]]
for M, N, K, epi in cases:
    A = torch.randn(M, K, device=dev).to(torch.bfloat16)
    W = (torch.randn(N, K, device=dev) * K ** -0.5).to(torch.bfloat16)
    bias = torch.randn(N, device=dev).to(torch.bfloat16)
    R = torch.randn(M, N, device=dev).to(torch.bfloat16)
    C = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
    t_ours = timeit(lambda: api.ops.gemm(A, W, bias, epi, resid=R if epi == "bias_resid" else None, out=C))
    t_cublas = timeit(lambda: torch.matmul(A, W.t(), out=C))
    fl = 2 * M * N * K
    print(f"M={M:6d} N={N:5d} K={K:5d} {epi:11s}: ours {t_ours:7.1f} us ({fl / t_ours / 1e6:6.0f} TF/s)   "
          f"cuBLAS {t_cublas:7.1f} us ({fl / t_cublas / 1e6:6.0f} TF/s)")
