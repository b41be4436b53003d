"""One call of our decode GEMM on one Llama-7B shape (for ncu captures).

    python scripts/dec_one.py gate_up
"""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

T = 64
SH = {"qkv": (12288, 4096, "store"), "o": (4096, 4096, "resid"), "gate_up": (11008, 4096, "swiglu"),
      "down": (4096, 11008, "resid"), "lm_head": (32000, 4096, "store")}
N, K, epi = SH[sys.argv[1] if len(sys.argv) > 1 else "gate_up"]
X = torch.randn(T, K, device="cuda").to(torch.bfloat16)
W = torch.randn(N, K, device="cuda").to(torch.bfloat16)
W2 = torch.randn(N, K, device="cuda").to(torch.bfloat16) if epi == "swiglu" else None
R = torch.randn(T, N, device="cuda").to(torch.bfloat16)
out = torch.empty(T, N, device="cuda", dtype=torch.bfloat16)
for _ in range(2):
    api.ops.dec_gemm(X, W, epi, W2=W2, resid=R if epi == "resid" else None, out=out)
torch.cuda.synchronize()
