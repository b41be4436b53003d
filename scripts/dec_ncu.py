"""One call each of our decode GEMM and cuBLAS on the Llama-7B O and QKV
shapes (T = 64), for an ncu capture:

    ncu --set full -k regex:'gemm_dec|nvjet|xmma|gemm' python scripts/dec_ncu.py
"""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

DEV = "cuda:0"
T = 64
for name, N, K, epi in [("o", 4096, 4096, "resid"), ("qkv", 12288, 4096, "store")]:
    X = torch.randn(T, K, device=DEV).to(torch.bfloat16)
    W = torch.randn(N, K, device=DEV).to(torch.bfloat16)
    R = torch.randn(T, N, device=DEV).to(torch.bfloat16)
    out = torch.empty(T, N, device=DEV, dtype=torch.bfloat16)
    api.ops.dec_gemm(X, W, epi, resid=R if epi == "resid" else None, out=out)
    y = X @ W.t()
    torch.cuda.synchronize()
    print(name, "done", flush=True)
