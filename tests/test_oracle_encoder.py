"""Pins for oracle.encoder: torch.nn.TransformerEncoderLayer (float64, CPU) and
closed-form special cases."""
import numpy as np
import pytest
import torch

import e3data
from e3data.configs import ModelConfig
from oracle import encoder
from oracle.numerics import bf16_rne


def _cfg(arch, H=64, nh=4, F=256, S=9, eps=1e-12):
    return ModelConfig(name="t", arch=arch, layers=1, hidden=H, heads=nh, ffn=F, seq=S,
                       classes=2, norm_eps=eps, ramp_layers=(0,), batch=4, test="maxprob")


def _torch_layer(W, H, nh, F, eps, norm_first):
    L = torch.nn.TransformerEncoderLayer(d_model=H, nhead=nh, dim_feedforward=F, dropout=0.0,
                                         activation="gelu", layer_norm_eps=eps,
                                         batch_first=True, norm_first=norm_first)
    L = L.double().eval()
    t = lambda a: torch.tensor(np.asarray(a, dtype=np.float64))
    with torch.no_grad():
        L.self_attn.in_proj_weight.copy_(t(W["w_qkv"]))
        L.self_attn.in_proj_bias.copy_(t(W["b_qkv"]))
        L.self_attn.out_proj.weight.copy_(t(W["w_o"]))
        L.self_attn.out_proj.bias.copy_(t(W["b_o"]))
        L.linear1.weight.copy_(t(W["w_1"]))
        L.linear1.bias.copy_(t(W["b_1"]))
        L.linear2.weight.copy_(t(W["w_2"]))
        L.linear2.bias.copy_(t(W["b_2"]))
        L.norm1.weight.copy_(t(W["ln1_g"]))
        L.norm1.bias.copy_(t(W["ln1_b"]))
        L.norm2.weight.copy_(t(W["ln2_g"]))
        L.norm2.bias.copy_(t(W["ln2_b"]))
    return L


@pytest.mark.parametrize("arch,norm_first,eps", [("bert", False, 1e-12), ("vit", True, 1e-6)])
def test_layer_matches_torch_transformer_encoder_layer(arch, norm_first, eps):
    cfg = _cfg(arch, eps=eps)
    W = {k: v.astype(np.float64) for k, v in e3data.make_layer(cfg, 0, seed=3).items()}
    X = e3data.make_inputs(cfg, range(5), seed=4).astype(np.float64)
    ours = encoder.encoder_layer(cfg, X, W, mode="fp64")
    L = _torch_layer(W, cfg.hidden, cfg.heads, cfg.ffn, eps, norm_first)
    with torch.no_grad():
        ref = L(torch.tensor(X)).numpy()
    assert np.max(np.abs(ours - ref)) < 1e-11


def test_single_token_attention_is_v_projection():
    rng = np.random.default_rng(1)
    qkv = rng.standard_normal((3, 1, 3 * 32))
    out = encoder.attention(qkv, heads=4, mode="fp64")
    assert np.allclose(out, qkv[..., 64:], atol=0, rtol=0)


def test_attention_key_permutation_invariance():
    rng = np.random.default_rng(2)
    S, H = 11, 32
    qkv = rng.standard_normal((S, 3 * H))
    perm = rng.permutation(S)
    permuted = qkv.copy()
    permuted[:, H:] = qkv[perm, H:]          # permute key/value rows together
    a = encoder.attention(qkv, heads=2, mode="fp64")
    b = encoder.attention(permuted, heads=2, mode="fp64")
    assert np.max(np.abs(a - b)) < 1e-13


def test_attention_matches_explicit_softmax_formula():
    # two-key closed form: weight on key 0 is sigmoid((s0 - s1))
    q = np.array([[1.0, 0.0]]); k = np.array([[2.0, 0.0], [0.0, 1.0]]); v = np.array([[1.0, 3.0], [5.0, 7.0]])
    qkv = np.concatenate([np.repeat(q, 2, 0), k, v], axis=1)   # S=2, H=2, 1 head
    out = encoder.attention(qkv, heads=1, mode="fp64")
    s0, s1 = 2.0 / np.sqrt(2), 0.0
    w0 = 1 / (1 + np.exp(s1 - s0))
    assert np.allclose(out[0], w0 * v[0] + (1 - w0) * v[1], rtol=1e-14)


def test_zero_weights_give_double_layernorm():
    cfg = _cfg("bert")
    W = {k: np.zeros_like(v, dtype=np.float64) for k, v in e3data.make_layer(cfg, 0).items()}
    W["ln1_g"][:] = 1.0
    W["ln2_g"][:] = 1.0
    X = e3data.make_inputs(cfg, range(2)).astype(np.float64)
    out = encoder.bert_layer(X, W, cfg.heads, cfg.norm_eps)
    ln = lambda x: (x - x.mean(-1, keepdims=True)) / np.sqrt(x.var(-1, keepdims=True) + cfg.norm_eps)
    assert np.max(np.abs(out - ln(ln(X)))) < 1e-12


def test_gelu_and_layernorm_definitions():
    from scipy.stats import norm
    x = np.linspace(-6, 6, 101)
    assert np.allclose(encoder.gelu(x), x * norm.cdf(x), rtol=1e-13, atol=1e-15)
    y = np.random.default_rng(0).standard_normal((4, 16))
    g = np.full(16, 2.0); b = np.full(16, 0.5)
    z = encoder.layer_norm(y, g, b, 0.0)
    assert np.allclose(z.mean(-1), 0.5) and np.allclose(z.std(-1), 2.0)


def test_bf16_mode_outputs_are_bf16():
    cfg = _cfg("bert")
    W = e3data.make_layer(cfg, 0)
    X = e3data.make_inputs(cfg, range(2))
    out = encoder.bert_layer(X.astype(np.float64), W, cfg.heads, cfg.norm_eps, mode="bf16")
    assert np.array_equal(bf16_rne(out), out)
    ref = encoder.bert_layer(X.astype(np.float64), W, cfg.heads, cfg.norm_eps, mode="fp64")
    assert np.max(np.abs(out - ref)) < 0.1      # same function up to bf16 rounding
