"""Per-item phase timeline of the encoder attention kernel (e3_debug_gemm_trace)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import _lib, api  # noqa: E402

B, S, H, nh = 64, 128, 768, 12
if len(sys.argv) > 1:
    B, S, H, nh = (int(v) for v in sys.argv[1:5])
qkv = torch.randn(B * S, 3 * H, device="cuda").to(torch.bfloat16)
out = torch.empty(B * S, H, device="cuda", dtype=torch.bfloat16)
for _ in range(5):
    api.ops.attention(qkv, B, S, H, nh, out=out)
torch.cuda.synchronize()
buf = torch.zeros(148 * 16 * 6 + 296 * 8 * 6, dtype=torch.int64, device="cuda")
_lib.lib.e3_debug_gemm_trace(buf.data_ptr())
api.ops.attention(qkv, B, S, H, nh, out=out)
torch.cuda.synchronize()
_lib.lib.e3_debug_gemm_trace(None)
t = buf.cpu().numpy()[148 * 16 * 6:].reshape(296, 8, 6).astype(np.float64)
t0 = t[t > 0].min()
print("phases per item (us): loads landed, S ready, P ready, O ready, stored")
for c in (0, 1, 2, 148, 149, 295):
    print("CTA", c)
    for j in range(8):
        if t[c, j, 0] <= 0:
            break
        print("  ", " ".join(f"{(v - t0) / 1000:6.2f}" for v in t[c, j, :5]))
v = t[:, :, :5]
ok = (v > 0).all(axis=2)
d = np.diff(v, axis=2)[ok] / 1000
print("median phase durations (us): load->S %.2f, S->P %.2f, P->O %.2f, O->stored %.2f" % tuple(np.median(d, axis=0)))
print("kernel span %.2f us" % ((t[t > 0].max() - t0) / 1000))
