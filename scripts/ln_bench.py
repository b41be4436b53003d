"""LayerNorm op vs torch's layer_norm and a plain copy on the VT / BB row
counts (graph-timed): python scripts/ln_bench.py [rows] [H]"""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402
from gemm_sweep_util import timeit  # noqa: E402

rows = int(sys.argv[1]) if len(sys.argv) > 1 else 256 * 197
H = int(sys.argv[2]) if len(sys.argv) > 2 else 768
x = torch.randn(rows, H, device="cuda").to(torch.bfloat16)
g = torch.randn(H, device="cuda").to(torch.bfloat16)
b = torch.randn(H, device="cuda").to(torch.bfloat16)
y = torch.empty_like(x)
nb = 2 * rows * H * 2
for name, fn in [("ours", lambda: api.ops.layernorm(x, g, b, 1e-6, out=y)),
                 ("torch layer_norm", lambda: torch.nn.functional.layer_norm(x, (H,), g, b, 1e-6)),
                 ("copy", lambda: y.copy_(x))]:
    t = timeit(fn, 20)
    print(f"{name:18s} rows={rows} H={H}: {t:7.1f} us  {nb / t / 1e3:6.0f} GB/s")
