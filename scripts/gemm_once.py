"""Run one layer GEMM of ours and cuBLAS's a few times, eagerly (an ncu target):
python scripts/gemm_once.py M N K epi [reps]."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

M, N, K, epi = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 3
dev = "cuda:0"
A = torch.randn(M, K, device=dev).to(torch.bfloat16)
W = (torch.randn(N, K, device=dev) * K ** -0.5).to(torch.bfloat16)
bias = torch.randn(N, device=dev).to(torch.bfloat16)
R = torch.randn(M, N, device=dev).to(torch.bfloat16)
C = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
for _ in range(reps):
    api.ops.gemm(A, W, bias, epi, resid=R if epi == "bias_resid" else None, out=C)
    torch.matmul(A, W.t(), out=C)
torch.cuda.synchronize()
