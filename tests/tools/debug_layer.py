"""Step-by-step GPU vs oracle (bf16-emulate) diagnostics for one encoder layer."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import e3data  # noqa: E402
from oracle import encoder as E  # noqa: E402
from oracle.numerics import bf16_rne  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

DEV = "cuda:0"
cfg = e3data.get(sys.argv[1] if len(sys.argv) > 1 else "tiny")
W = e3data.make_weights(cfg)
B = 4
X = e3data.make_inputs(cfg, range(B))
L = {k: v.astype(np.float64) for k, v in W["layers"][0].items()}
Lt = {k: api.to_bf16(v, DEV) for k, v in W["layers"][0].items()}
H, F, S = cfg.hidden, cfg.ffn, cfg.seq


def t64(t):
    return t.float().cpu().numpy().astype(np.float64)


def report(name, got, ref):
    d = np.abs(got - ref)
    print(f"{name:8s} max {d.max():.3e} mean {d.mean():.3e} frac_diff {np.mean(got != ref):.4f} "
          f"|ref| {np.abs(ref).mean():.3e}")


x = api.to_bf16(X.reshape(B * S, H), DEV)
x64 = X.reshape(B * S, H).astype(np.float64)
qkv = api.ops.gemm(x, Lt["w_qkv"], Lt["b_qkv"], "bias")
report("qkv", t64(qkv), bf16_rne(E.linear(x64, L["w_qkv"], L["b_qkv"])))
q64 = t64(qkv)
ctx = api.ops.attention(qkv, B, S, H, cfg.heads)
report("ctx", t64(ctx).reshape(B, S, H), E.attention(q64.reshape(B, S, 3 * H), cfg.heads, "bf16"))
c64 = t64(ctx)
y = api.ops.gemm(ctx, Lt["w_o"], Lt["b_o"], "bias_resid", resid=x)
report("y1", t64(y), bf16_rne(E.linear(c64, L["w_o"], L["b_o"]) + x64))
y64 = t64(y)
x1 = api.ops.layernorm(y, Lt["ln1_g"], Lt["ln1_b"], cfg.norm_eps)
report("x1", t64(x1), bf16_rne(E.layer_norm(y64, L["ln1_g"], L["ln1_b"], cfg.norm_eps)))
x164 = t64(x1)
h = api.ops.gemm(x1, Lt["w_1"], Lt["b_1"], "bias_gelu")
report("h", t64(h), bf16_rne(E.gelu(E.linear(x164, L["w_1"], L["b_1"]))))
h64 = t64(h)
y2 = api.ops.gemm(h, Lt["w_2"], Lt["b_2"], "bias_resid", resid=x1)
report("y2", t64(y2), bf16_rne(E.linear(h64, L["w_2"], L["b_2"]) + x164))
out = api.ops.layernorm(y2, Lt["ln2_g"], Lt["ln2_b"], cfg.norm_eps)
report("x2", t64(out), bf16_rne(E.layer_norm(t64(y2), L["ln2_g"], L["ln2_b"], cfg.norm_eps)))
full = E.bert_layer(X.astype(np.float64), L, cfg.heads, cfg.norm_eps, "bf16").reshape(B * S, H)
report("layer", t64(out), full)
fp = E.bert_layer(X.astype(np.float64), L, cfg.heads, cfg.norm_eps, "fp64").reshape(B * S, H)
report("vs fp64", t64(out), fp)
report("emu-fp64", full, fp)
