"""Time the fused O projection + LayerNorm (e3_op_gemm_ln) at a layer shape,
CUDA-graph replayed (device time only).  E3_LN_SINGLE=1 selects the 1-SM
cluster-of-2 variant instead of the CTA-pair cluster-of-4 one.

    python scripts/gemm_ln_bench.py [M N K]     (default EE-BERT-base: 8192 768 768)
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

M, N, K = (int(v) for v in sys.argv[1:4]) if len(sys.argv) > 3 else (8192, 768, 768)
g = torch.Generator(device="cuda").manual_seed(0)
A = torch.randn(M, K, device="cuda", generator=g).to(torch.bfloat16)
W = (torch.randn(N, K, device="cuda", generator=g) * K ** -0.5).to(torch.bfloat16)
b = torch.zeros(N, device="cuda", dtype=torch.bfloat16)
R = torch.randn(M, N, device="cuda", generator=g).to(torch.bfloat16)
gam = torch.ones(N, device="cuda", dtype=torch.bfloat16)
out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
for _ in range(5):
    api.ops.gemm_ln(A, W, b, R, gam, b, 1e-12, out=out)
torch.cuda.synchronize()
n = 50
graph = torch.cuda.CUDAGraph()
with torch.cuda.graph(graph):
    for _ in range(n):
        api.ops.gemm_ln(A, W, b, R, gam, b, 1e-12, out=out)
graph.replay()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
graph.replay()
e1.record()
torch.cuda.synchronize()
t = e0.elapsed_time(e1) / n * 1000
print(f"gemm_ln M={M} N={N} K={K} ({'1-SM' if os.environ.get('E3_LN_SINGLE') else 'pair'}): {t:.2f} us "
      f"{2 * M * N * K / t / 1e6:.0f} TFLOP/s")
