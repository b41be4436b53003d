"""Pins of the oracle's bf16-emulate STORAGE POINTS (DESIGN.md §3 "Rounding
contract").

Two kinds of pin:

1. Hand-computed tiny cases whose result changes distinctly if any one
   rounding point is dropped, moved or added (the expected numbers are
   derived in the comments, by hand, from the contract -- not by calling
   the oracle).  bf16 keeps 8 significant bits: on [2^e, 2^(e+1)) the spacing
   is 2^(e-7); ties go to the even mantissa.

2. Dataflow pins: the oracle's `store` is wrapped by a recorder, and every
   recorded storage point is checked to be computed from the ROUNDED values
   of the storage points before it, in the contract's order, with nothing
   else rounded (an extra rounding -- e.g. of the softmax normaliser l -- or a
   missing one shows up as a wrong call count or a failed relation).
"""
import numpy as np
import pytest

import e3data
from e3data.configs import ModelConfig
from oracle import encoder, llama
from oracle import numerics
from oracle.numerics import bf16_rne


# ------------------------------------------------------------ hand cases --

def test_attention_rounds_p_not_the_normaliser():
    """1 head, d = 1, S = 2; rows [q, k, v] = [1, 0, 0] and [0, -1, 1].
    Query 0: s = (q0 k0, q0 k1) = (0, -1); p = (1, e^-1 = 0.36787944...).
      bf16(e^-1): 0.36787944 / 2^-9 = 188.35 -> 188 * 2^-9 = 0.3671875.
      l = 1 + e^-1 = 1.36787944 (UNROUNDED p).
      numerator = bf16(p) . v = 0.3671875.
      ctx = 0.3671875 / 1.36787944 = 0.26843557 -> / 2^-9 = 137.44 -> 137
          -> 0.267578125.
      Had l been rounded (1.3671875): 0.26857143 -> 137.51 -> 138 -> 0.26953125;
      had p not been rounded: 0.26894142 -> 137.70 -> 138 -> 0.26953125.
    Query 1: q = 0 -> s = (0, 0), p = (1, 1), l = 2, ctx = 1/2 = 0.5.
    fp64 mode: ctx0 = e^-1 / (1 + e^-1) = 1 / (1 + e)."""
    qkv = np.array([[[1.0, 0.0, 0.0], [0.0, -1.0, 1.0]]])
    out = encoder.attention(qkv, 1, "bf16")
    assert out[0, 0, 0] == 0.267578125
    assert out[0, 1, 0] == 0.5
    out64 = encoder.attention(qkv, 1, "fp64")
    assert abs(out64[0, 0, 0] - 1.0 / (1.0 + np.e)) < 1e-15


def _zero_layer(H, F, heads):
    z = lambda *s: np.zeros(s)
    return {"w_qkv": z(3 * H, H), "b_qkv": z(3 * H), "w_o": z(H, H), "b_o": z(H),
            "ln1_g": np.ones(H), "ln1_b": z(H), "w_1": z(F, H), "b_1": z(F), "w_2": z(H, F), "b_2": z(H),
            "ln2_g": np.ones(H), "ln2_b": z(H)}


def test_bert_layer_rounds_y1_before_ln_and_x1_before_ln2():
    """H = 4, 1 head, S = 1, F = 4; every weight zero except b_o = (2, 0, 0, 0),
    LN gamma = 1, beta = 0, eps = 1e-12.  x = (255, 255, 254, 250) (bf16).
      qkv = 0 -> ctx = 0;  y1 = x + b_o = (257, 255, 254, 250).
      bf16(y1): 257 lies midway between 256 and 258 (spacing 2 on [256, 512))
        -> tie to even -> 256;  y1 = (256, 255, 254, 250).
      LN1: mean 253.75, var (2.25^2 + 1.25^2 + 0.25^2 + 3.75^2)/4 = 5.1875,
        x1 = (0.98787834, 0.54882130, 0.10976426, -1.64646390)
        -> bf16: 252.90 * 2^-8 -> 0.98828125; 140.50 * 2^-9 -> 0.546875
           (140.498 < 140.5); 224.80 * 2^-11 -> 0.10986328125;
           210.75 * 2^-7 -> -1.6484375.
      FFN: W_1 = 0 -> h = GELU(0) = 0;  y2 = 0 + x1 (bf16 already).
      LN2 of the ROUNDED x1: mean -0.0008544921875, var 1.0012963265,
        x2 = (0.98849524, 0.54737482, 0.11064608, -1.64651614)
        -> bf16: 0.98828125, 0.546875, 226.60 * 2^-11 -> 0.11083984375, -1.6484375.
    Variants: y1 not rounded -> x2 = (1.1796875, 0.390625, -0.00048828125,
    -1.5703125); x1 not rounded -> LN2(LN1(y1)) = LN1(y1) -> third element
    0.10986328125."""
    H = 4
    W = _zero_layer(H, 4, 1)
    W["b_o"] = np.array([2.0, 0.0, 0.0, 0.0])
    x = np.array([[[255.0, 255.0, 254.0, 250.0]]])
    out = encoder.bert_layer(x, W, 1, 1e-12, "bf16")
    assert out[0, 0].tolist() == [0.98828125, 0.546875, 0.11083984375, -1.6484375]


def test_vit_layer_rounds_n1_and_y1():
    """Pre-LN (ViT), H = 4, 1 head, S = 1, zero weights except b_o, eps 1e-6:
      n1 = bf16(LN1(x)) feeds only the (zero) QKV -> ctx = 0;
      y1 = bf16(x + b_o), x = (255, 255, 254, 250), b_o = (2, 0, 0, 0)
         -> (257 -> 256, 255, 254, 250);
      n2 = bf16(LN2(y1)) feeds only the (zero) MLP -> h = 0;
      x2 = bf16(0 + b_2 + y1) = y1 = (256, 255, 254, 250).
    Had y1 been kept unrounded and only x2 rounded, x2 would still be 256 in
    the first element; so add b_2 = (1, 0, 0, 0): x2 = bf16(256 + 1) = 256 (tie
    to even) with rounded y1, but bf16(257 + 1) = 258 with an unrounded y1."""
    H = 4
    W = _zero_layer(H, 4, 1)
    W["b_o"] = np.array([2.0, 0.0, 0.0, 0.0])
    W["b_2"] = np.array([1.0, 0.0, 0.0, 0.0])
    x = np.array([[[255.0, 255.0, 254.0, 250.0]]])
    out = encoder.vit_layer(x, W, 1, 1e-6, "bf16")
    assert out[0, 0].tolist() == [256.0, 255.0, 254.0, 250.0]


def test_llama_decode_rounds_the_layer_output():
    """Llama decode, H = 2 (1 head, d = 2), position 0, RMSNorm eps 0, all
    weights zero except W_gate[0,0] = W_up[0,0] = W_down[0,0] = 1; x = (255, 250).
      q = k = v = 0 -> a = 0 -> h = bf16(x) = (255, 250).
      n2 = RMSNorm(h): rms = sqrt((255^2 + 250^2)/2) = 252.51238;
        n2 = (1.0098509, 0.9902459) -> bf16: 129.26 * 2^-7 -> 1.0078125,
        253.50 * 2^-8 -> 253 (253.4959) -> 0.98828125.
      act_0 = bf16(SiLU(1.0078125) * 1.0078125) = bf16(0.74408330)
            -> 190.49 * 2^-8 -> 190 -> 0.7421875;  act_1 = 0.
      x' = bf16(h + act W_down^T) = (bf16(255.7421875), 250) = (256, 250)
        (spacing 1 on [128, 256); 255.74 rounds up to 256).
    An unrounded x' would be 255.7421875."""
    cfg = ModelConfig(name="t", arch="llama", layers=1, hidden=2, heads=1, ffn=2, seq=1, classes=2,
                      norm_eps=0.0, ramp_layers=(0,), batch=1, test="maxprob", kv_heads=1, ctx=0)
    z = lambda *s: np.zeros(s)
    W = {"ln1_g": np.ones(2), "ln2_g": np.ones(2), "w_qkv": z(6, 2), "w_o": z(2, 2),
         "w_gate": z(2, 2), "w_up": z(2, 2), "w_down": z(2, 2)}
    W["w_gate"][0, 0] = 1.0
    W["w_up"][0, 0] = 1.0
    W["w_down"][0, 0] = 1.0
    K = np.zeros((1, 1, 1, 2))
    V = np.zeros((1, 1, 1, 2))
    x = np.array([[255.0, 250.0]])
    out = llama.decode_layer(cfg, x, W, K, V, [0], "bf16")
    assert out[0].tolist() == [256.0, 250.0]
    # fp64: x'_0 = 255 + SiLU(n2_0) n2_0 with the exact n2_0 = 255 / 252.5124
    n20 = 255.0 / np.sqrt((255.0 ** 2 + 250.0 ** 2) / 2)
    out64 = llama.decode_layer(cfg, x, W, K, V, [0], "fp64")
    assert abs(out64[0, 0] - (255.0 + n20 * n20 / (1 + np.exp(-n20)))) < 1e-12
    # the hand value of act: n2 rounded then SiLU * up, rounded to bf16
    assert bf16_rne(1.0078125 / (1 + np.exp(-1.0078125)) * 1.0078125) == 0.7421875


# --------------------------------------------------------- dataflow pins --

class _Recorder:
    def __init__(self):
        self.calls = []

    def __call__(self, x, mode):
        x = np.asarray(x, dtype=np.float64)
        out = numerics.store(x, mode)
        self.calls.append((x.copy(), out))
        return out


def _rand_layer(rng, H, F):
    r = lambda *s: bf16_rne(rng.standard_normal(s) * 0.3)
    return {"w_qkv": r(3 * H, H), "b_qkv": r(3 * H), "w_o": r(H, H), "b_o": r(H), "ln1_g": 1 + r(H) * 0.1,
            "ln1_b": r(H) * 0.1, "w_1": r(F, H), "b_1": r(F), "w_2": r(H, F), "b_2": r(H),
            "ln2_g": 1 + r(H) * 0.1, "ln2_b": r(H) * 0.1}


def _attn_check(calls, qkv_r, heads, k0):
    """calls[k0 .. k0+heads-1] = p per head from the ROUNDED qkv; calls[k0+heads]
    = ctx = (bf16(p) v) / l with l from the UNROUNDED p."""
    H = qkv_r.shape[-1] // 3
    d = H // heads
    ctx = np.empty(qkv_r.shape[:-1] + (H,))
    for h in range(heads):
        q, k, v = (qkv_r[..., j * H + h * d: j * H + (h + 1) * d] for j in range(3))
        s = q @ np.swapaxes(k, -1, -2) / np.sqrt(d)
        p = np.exp(s - s.max(-1, keepdims=True))
        assert np.allclose(calls[k0 + h][0], p, rtol=1e-13, atol=0)
        ctx[..., h * d:(h + 1) * d] = calls[k0 + h][1] @ v / p.sum(-1, keepdims=True)
    assert np.allclose(calls[k0 + heads][0], ctx, rtol=1e-12, atol=1e-14)
    return calls[k0 + heads][1]


def test_bert_layer_storage_dataflow(monkeypatch):
    rng = np.random.default_rng(0)
    S, H, F, heads, eps = 5, 8, 16, 2, 1e-12
    W = _rand_layer(rng, H, F)
    x = bf16_rne(rng.standard_normal((1, S, H)))
    rec = _Recorder()
    monkeypatch.setattr(encoder, "store", rec)
    out = encoder.bert_layer(x, W, heads, eps, "bf16")
    c = rec.calls
    assert len(c) == 7 + heads        # qkv, p x heads, ctx, y1, x1, h, y2, x2
    LN = lambda y, g, b: encoder.layer_norm(y, g, b, eps)
    close = lambda a, b: np.allclose(a, b, rtol=1e-12, atol=1e-13)
    assert close(c[0][0], x @ W["w_qkv"].T + W["b_qkv"])
    ctx = _attn_check(c, c[0][1], heads, 1)
    k = 2 + heads
    assert close(c[k][0], ctx @ W["w_o"].T + W["b_o"] + x)                       # y1 from rounded ctx
    assert close(c[k + 1][0], LN(c[k][1], W["ln1_g"], W["ln1_b"]))              # x1 = LN1(rounded y1)
    assert close(c[k + 2][0], encoder.gelu(c[k + 1][1] @ W["w_1"].T + W["b_1"]))   # h from rounded x1
    assert close(c[k + 3][0], c[k + 2][1] @ W["w_2"].T + W["b_2"] + c[k + 1][1])  # y2 = rounded h, x1
    assert close(c[k + 4][0], LN(c[k + 3][1], W["ln2_g"], W["ln2_b"]))          # x2 = LN2(rounded y2)
    assert np.array_equal(out, c[k + 4][1])


def test_vit_layer_storage_dataflow(monkeypatch):
    rng = np.random.default_rng(1)
    S, H, F, heads, eps = 4, 8, 16, 2, 1e-6
    W = _rand_layer(rng, H, F)
    x = bf16_rne(rng.standard_normal((2, S, H)))
    rec = _Recorder()
    monkeypatch.setattr(encoder, "store", rec)
    out = encoder.vit_layer(x, W, heads, eps, "bf16")
    c = rec.calls
    assert len(c) == 7 + heads        # n1, qkv, p x heads, ctx, y1, n2, h, x2
    LN = lambda y, g, b: encoder.layer_norm(y, g, b, eps)
    close = lambda a, b: np.allclose(a, b, rtol=1e-12, atol=1e-13)
    assert close(c[0][0], LN(x, W["ln1_g"], W["ln1_b"]))
    assert close(c[1][0], c[0][1] @ W["w_qkv"].T + W["b_qkv"])
    ctx = _attn_check(c, c[1][1], heads, 2)
    k = 3 + heads
    assert close(c[k][0], ctx @ W["w_o"].T + W["b_o"] + x)
    assert close(c[k + 1][0], LN(c[k][1], W["ln2_g"], W["ln2_b"]))
    assert close(c[k + 2][0], encoder.gelu(c[k + 1][1] @ W["w_1"].T + W["b_1"]))
    assert close(c[k + 3][0], c[k + 2][1] @ W["w_2"].T + W["b_2"] + c[k][1])    # residual = rounded y1
    assert np.array_equal(out, c[k + 3][1])


def test_llama_decode_storage_dataflow(monkeypatch):
    cfg = e3data.get("tiny-llama")
    import dataclasses
    cfg = dataclasses.replace(cfg, hidden=256, heads=2, kv_heads=1, ffn=64)
    rng = np.random.default_rng(2)
    H, F, d, n, ctx = 256, 64, 128, 3, 6
    r = lambda *s: bf16_rne(rng.standard_normal(s) * 0.05)
    W = {"ln1_g": 1 + r(H), "ln2_g": 1 + r(H), "w_qkv": r((2 + 2) * 128, H), "w_o": r(H, H),
         "w_gate": r(F, H), "w_up": r(F, H), "w_down": r(H, F)}
    x = bf16_rne(rng.standard_normal((n, H)))
    K = bf16_rne(rng.standard_normal((n, 1, ctx + 1, d)))
    V = bf16_rne(rng.standard_normal((n, 1, ctx + 1, d)))
    pos = [ctx, ctx - 2, 1]
    rec = _Recorder()
    monkeypatch.setattr(llama, "store", rec)
    out = llama.decode_layer(cfg, x, W, K.copy(), V.copy(), pos, "bf16")
    c = rec.calls
    assert len(c) == 9                # n1, q, k, v, a, h, n2, act, x'
    close = lambda a, b: np.allclose(a, b, rtol=1e-12, atol=1e-13)
    eps = cfg.norm_eps
    assert close(c[0][0], llama.rms_norm(x, W["ln1_g"], eps))
    qkv = c[0][1] @ W["w_qkv"].T
    P = np.asarray(pos)[:, None]
    assert close(c[1][0], llama.rope(qkv[:, :256].reshape(n, 2, d), P, cfg.rope_theta))
    assert close(c[2][0], llama.rope(qkv[:, 256:384].reshape(n, 1, d), P, cfg.rope_theta))
    assert close(c[3][0], qkv[:, 384:].reshape(n, 1, d))
    # attention from the ROUNDED q, k, v (k, v written into the cache first)
    q, k, v = c[1][1], c[2][1], c[3][1]
    a = np.empty((n, 2, d))
    for i in range(n):
        Ki, Vi = K[i, 0].copy(), V[i, 0].copy()
        Ki[pos[i]], Vi[pos[i]] = k[i, 0], v[i, 0]
        for h in range(2):
            s = Ki[:pos[i] + 1] @ q[i, h] / np.sqrt(d)
            w = np.exp(s - s.max())
            a[i, h] = w @ Vi[:pos[i] + 1] / w.sum()
    assert close(c[4][0], a.reshape(n, H))
    assert close(c[5][0], x + c[4][1] @ W["w_o"].T)                      # h from rounded a
    assert close(c[6][0], llama.rms_norm(c[5][1], W["ln2_g"], eps))        # n2 = RMSNorm(rounded h)
    g, u = c[6][1] @ W["w_gate"].T, c[6][1] @ W["w_up"].T
    assert close(c[7][0], llama.silu(g) * u)                              # act from rounded n2
    assert close(c[8][0], c[5][1] + c[7][1] @ W["w_down"].T)               # x' = rounded h + act
    assert np.array_equal(out, c[8][1])
    # the ramp rounds its normalised row (R23) and nothing after it
    rec.calls.clear()
    R = {"ln_g": 1 + r(H), "w_c": r(10, H)}
    z = llama.ramp_logits(cfg, out, R, "bf16")
    assert len(rec.calls) == 1 and close(rec.calls[0][0], llama.rms_norm(out, R["ln_g"], eps))
    assert close(z, rec.calls[0][1] @ R["w_c"].T)
