"""Encoder layers of the early-exit transformer — TEST INFRASTRUCTURE ONLY.

The paper runs stock BERT-BASE / DeeBERT
and never writes the layer out; the readings used here are DESIGN.md R11
(= SURVEY §8(c) C11): BERT is post-LN with LN eps 1e-12, exact erf-GELU,
scale 1/sqrt(d), no attention mask; ViT is the pre-LN variant with eps 1e-6.

``mode`` selects the arithmetic:
  "fp64"  every operation in float64 (the plain definition);
  "bf16"  float64 arithmetic, RNE-rounded to bf16 at the storage points of
          DESIGN.md "Rounding contract" (numerics.store).

Pins (tests/test_oracle_encoder.py): in fp64 mode both layers equal
``torch.nn.TransformerEncoderLayer`` (norm_first False / True, gelu, batch
first, dropout 0) in float64 on CPU to ~1e-12; S = 1 reduces attention to the
V projection; zero weights with gamma = 1, beta = 0 give LN(LN(x)); the
attention is invariant to permuting key/value rows.
"""
from __future__ import annotations

import numpy as np
from scipy.special import erf

from .numerics import store


def layer_norm(x, g, b, eps):
    """LN over the last axis, biased variance (Ba et al.; C11)."""
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * g + b


def gelu(x):
    """Exact GELU: x * Phi(x) = 0.5 x (1 + erf(x / sqrt 2)) (C11)."""
    return 0.5 * x * (1.0 + erf(x / np.sqrt(2.0)))


def attention(qkv, heads, mode):
    """Multi-head self-attention over one or more sequences.

    qkv: [..., S, 3H] laid out [q | k | v], head h owning columns h*d:(h+1)*d
    of each third.  Per head: softmax(q k^T / sqrt(d)) v.
    bf16 mode: p = exp(s - max s) unrounded for the normaliser l = sum p,
    bf16(p) for the product with v, output bf16((bf16(p) v) / l).
    """
    H = qkv.shape[-1] // 3
    d = H // heads
    out = np.empty(qkv.shape[:-1] + (H,), dtype=np.float64)
    for h in range(heads):
        q = qkv[..., h * d:(h + 1) * d]
        k = qkv[..., H + h * d:H + (h + 1) * d]
        v = qkv[..., 2 * H + h * d:2 * H + (h + 1) * d]
        s = np.matmul(q, np.swapaxes(k, -1, -2)) / np.sqrt(d)
        p = np.exp(s - s.max(axis=-1, keepdims=True))
        l = p.sum(axis=-1, keepdims=True)
        out[..., h * d:(h + 1) * d] = np.matmul(store(p, mode), v) / l
    return store(out, mode)


def linear(x, w, b):
    """x W^T + b with W in nn.Linear layout [out, in]."""
    return np.matmul(x, w.T) + b


def bert_layer(x, W, heads, eps, mode="fp64"):
    """BERT post-LN encoder layer:
        qkv = x W_qkv^T + b_qkv
        x1  = LN1(x + attn(qkv) W_o^T + b_o)
        x2  = LN2(x1 + GELU(x1 W_1^T + b_1) W_2^T + b_2)
    """
    qkv = store(linear(x, W["w_qkv"], W["b_qkv"]), mode)
    ctx = attention(qkv, heads, mode)
    y1 = store(linear(ctx, W["w_o"], W["b_o"]) + x, mode)
    x1 = store(layer_norm(y1, W["ln1_g"], W["ln1_b"], eps), mode)
    h = store(gelu(linear(x1, W["w_1"], W["b_1"])), mode)
    y2 = store(linear(h, W["w_2"], W["b_2"]) + x1, mode)
    return store(layer_norm(y2, W["ln2_g"], W["ln2_b"], eps), mode)


def vit_layer(x, W, heads, eps, mode="fp64"):
    """ViT pre-LN encoder layer (C11):
        x1 = x + attn(LN1(x) W_qkv^T + b_qkv) W_o^T + b_o
        x2 = x1 + GELU(LN2(x1) W_1^T + b_1) W_2^T + b_2
    """
    n1 = store(layer_norm(x, W["ln1_g"], W["ln1_b"], eps), mode)
    qkv = store(linear(n1, W["w_qkv"], W["b_qkv"]), mode)
    ctx = attention(qkv, heads, mode)
    x1 = store(linear(ctx, W["w_o"], W["b_o"]) + x, mode)
    n2 = store(layer_norm(x1, W["ln2_g"], W["ln2_b"], eps), mode)
    h = store(gelu(linear(n2, W["w_1"], W["b_1"])), mode)
    return store(linear(h, W["w_2"], W["b_2"]) + x1, mode)


def encoder_layer(cfg, x, W, mode="fp64"):
    if cfg.arch == "bert":
        return bert_layer(x, W, cfg.heads, cfg.norm_eps, mode)
    if cfg.arch == "vit":
        return vit_layer(x, W, cfg.heads, cfg.norm_eps, mode)
    raise NotImplementedError(cfg.arch)
