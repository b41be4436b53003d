"""Decode GEMM bandwidth vs cuBLAS on the Llama-7B shapes (T = 64 tokens).

    python scripts/dec_bench.py
"""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

DEV = "cuda:0"
T = 64
shapes = [("qkv", 12288, 4096, "store"), ("o", 4096, 4096, "resid"), ("gate_up", 11008, 4096, "swiglu"),
          ("down", 4096, 11008, "resid"), ("lm_head", 32000, 4096, "store")]


def timeit(fn, n=20):
    """Device time per call: n calls captured in one CUDA graph (the host-side
    tensor-map encoding and scratch allocation of the op API are not timed)."""
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(n):
            fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1000


for name, N, K, epi in shapes:
    X = torch.randn(T, K, device=DEV).to(torch.bfloat16)
    # several weight copies round-robin so every call streams from HBM, not L2
    copies = max(2, int(400e6 // (N * K * 2 * (2 if epi == "swiglu" else 1))))
    Ws = [torch.randn(N, K, device=DEV).to(torch.bfloat16) for _ in range(copies)]
    W2s = [torch.randn(N, K, device=DEV).to(torch.bfloat16) for _ in range(copies)] if epi == "swiglu" else None
    R = torch.randn(T, N, device=DEV).to(torch.bfloat16)
    out = torch.empty(T, N, device=DEV, dtype=torch.bfloat16)
    it = [0]

    def ours():
        i = it[0] % copies
        it[0] += 1
        api.ops.dec_gemm(X, Ws[i], "swiglu" if epi == "swiglu" else ("resid" if epi == "resid" else "store"),
                         W2=W2s[i] if W2s else None, resid=R if epi == "resid" else None, out=out)

    def cublas():
        i = it[0] % copies
        it[0] += 1
        y = X @ Ws[i].t()
        if W2s:
            y = torch.nn.functional.silu(y) * (X @ W2s[i].t())

    bytes_ = N * K * 2 * (2 if epi == "swiglu" else 1)
    t1 = timeit(ours)
    t2 = timeit(cublas)
    print(f"{name:8s} N={N:6d} K={K:6d}: ours {t1:7.1f} us {bytes_ / t1 / 1e3:6.0f} GB/s | "
          f"torch/cuBLAS {t2:7.1f} us {bytes_ / t2 / 1e3:6.0f} GB/s")
