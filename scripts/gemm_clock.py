"""FFN1-shaped GEMM with and without the GELU epilogue, 2 s each, with nvidia-smi SM clock and power sampled."""
import subprocess
import sys
import time

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

dev = "cuda:0"
M, N, K = 8192, 3072, 768
A = torch.randn(M, K, device=dev).to(torch.bfloat16)
W = (torch.randn(N, K, device=dev) * K ** -0.5).to(torch.bfloat16)
bias = torch.randn(N, device=dev).to(torch.bfloat16)
C = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
for epi in ("bias", "bias_gelu", "bias", "bias_gelu"):
    fn = lambda: api.ops.gemm(A, W, bias, epi, out=C)  # noqa: E731
    for _ in range(5):
        fn()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(100):
            fn()
    torch.cuda.synchronize()
    p = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,power.draw", "--format=csv,noheader,nounits",
                          "-lms", "100"], stdout=subprocess.PIPE, text=True)
    t0 = time.time()
    n = 0
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    while time.time() - t0 < 2.0:
        g.replay()
        n += 1
        torch.cuda.synchronize()
    e1.record()
    torch.cuda.synchronize()
    p.terminate()
    rows = [r.split(",") for r in p.stdout.read().strip().splitlines() if r.strip()]
    clk = sorted(float(r[0]) for r in rows)
    pw = sorted(float(r[1]) for r in rows)
    us = e0.elapsed_time(e1) * 1000 / (n * 100)
    print(f"{epi:10s}: {us:6.1f} us per GEMM, SM clock median {clk[len(clk) // 2]:.0f} MHz, power median {pw[len(pw) // 2]:.0f} W")
