"""Time e3_op_attention on the EE-BERT-base shape (B=64, S=128, H=768, 12 heads), L2-warm."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

B, S, H, nh = 64, 128, 768, 12
if len(sys.argv) > 1:
    B, S, H, nh = (int(v) for v in sys.argv[1:5])
qkv = torch.randn(B * S, 3 * H, device="cuda").to(torch.bfloat16)
out = torch.empty(B * S, H, device="cuda", dtype=torch.bfloat16)
for _ in range(5):
    api.ops.attention(qkv, B, S, H, nh, out=out)
torch.cuda.synchronize()
n = 50
g = torch.cuda.CUDAGraph()            # device time only (the op API encodes tensor maps per call)
with torch.cuda.graph(g):
    for _ in range(n):
        api.ops.attention(qkv, B, S, H, nh, out=out)
g.replay()
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
g.replay()
b.record()
torch.cuda.synchronize()
t = a.elapsed_time(b) / n * 1000
fl = 4 * B * S * S * H
print(f"attention B={B} S={S} H={H}: {t:.1f} us  {fl / t / 1e6:.0f} TFLOP/s")
