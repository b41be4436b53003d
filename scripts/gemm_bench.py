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
    """Device time per call: n calls in one CUDA graph (the op API encodes
    tensor maps on the host per call; the split path precomputes them)."""
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

# fused O projection + residual + LayerNorm vs the two kernels it replaces
H = 768
A = torch.randn(M, H, device=dev).to(torch.bfloat16)
W = (torch.randn(H, H, device=dev) * H ** -0.5).to(torch.bfloat16)
bias = torch.randn(H, device=dev).to(torch.bfloat16)
R = torch.randn(M, H, device=dev).to(torch.bfloat16)
g = torch.ones(H, device=dev).to(torch.bfloat16)
bb = torch.zeros(H, device=dev).to(torch.bfloat16)
Y = torch.empty(M, H, device=dev, dtype=torch.bfloat16)
X1 = torch.empty(M, H, device=dev, dtype=torch.bfloat16)
t_f = timeit(lambda: api.ops.gemm_ln(A, W, bias, R, g, bb, 1e-12, out=X1))
t_o = timeit(lambda: api.ops.gemm(A, W, bias, "bias_resid", resid=R, out=Y))
t_ln = timeit(lambda: api.ops.layernorm(Y, g, bb, 1e-12, out=X1))
print(f"O+LN1 M={M} H={H}: fused {t_f:6.1f} us | gemm {t_o:6.1f} + layernorm {t_ln:6.1f} = {t_o + t_ln:6.1f} us")
for K in (64, 256, 768, 1536):
    A = torch.randn(M, K, device=dev).to(torch.bfloat16)
    W = (torch.randn(H, K, device=dev) * K ** -0.5).to(torch.bfloat16)
    t_f = timeit(lambda: api.ops.gemm_ln(A, W, bias, R, g, bb, 1e-12, out=X1))
    print(f"  fused O+LN K={K}: {t_f:6.1f} us ({2 * M * H * K / t_f / 1e6:6.0f} TF/s)")
