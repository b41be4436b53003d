"""Seeded synthetic weights and inputs, shared by the oracle and the CUDA path.

This module holds NO arithmetic of the method: it only draws numbers and rounds
them to bf16 (the storage format both sides consume).  Recipe (SURVEY.md §8(d),
stated again in DESIGN.md "Input recipe"):

* one NumPy PCG64 stream per (seed, tensor kind, layer, name), so any tensor
  or any single input can be regenerated alone;
* linear weights W ~ N(0, 1/fan_in), biases N(0, 0.02^2),
  LayerNorm gamma = 1 + N(0, 0.02^2), beta ~ N(0, 0.02^2);
* ramp pooler W_p ~ N(0, 1/H); ramp classifier W_c ~ N(0, g^2/H) (gain g);
* inputs X0[i] ~ N(0, 1), one stream per (seed, input id);
* every value is rounded to bf16 (round-to-nearest-even) and handed out as
  float32 holding a bf16-representable value (``bf16_bits`` gives the bits).

Weight layout is the nn.Linear convention ``[out_features, in_features]``.
"""
from __future__ import annotations

import os
import zlib
from typing import Dict, Iterable

import numpy as np

from .configs import ModelConfig

_KIND_WEIGHT = 0x57
_KIND_INPUT = 0xD47A


def bf16_round(x: np.ndarray) -> np.ndarray:
    """float -> nearest bf16 value (ties to even), returned as float32.

    uint32 arithmetic cannot wrap for finite inputs (max 0xFF7FFFFF + 0x8000)."""
    u = np.array(x, dtype=np.float32, copy=True).view(np.uint32)
    u += np.uint32(0x7FFF) + ((u >> np.uint32(16)) & np.uint32(1))
    u &= np.uint32(0xFFFF0000)
    return u.view(np.float32)


def bf16_bits(x: np.ndarray) -> np.ndarray:
    """bf16 bit patterns (uint16) of float32 values that are bf16-representable."""
    u = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32)
    return (u >> 16).astype(np.uint16)


def _rng(seed: int, kind: int, *keys: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, kind, *keys])))


def _normal(seed, layer, name, shape, std, mean=0.0):
    g = _rng(seed, _KIND_WEIGHT, layer, zlib.crc32(name.encode()))
    v = g.standard_normal(size=shape, dtype=np.float32) * np.float32(std)
    if mean:
        v = v + np.float32(mean)
    return bf16_round(v)


def layer_tensor_specs(cfg: ModelConfig):
    """(name, shape, std, mean) of one encoder layer's tensors."""
    H, F = cfg.hidden, cfg.ffn
    if cfg.arch in ("bert", "vit"):
        return [
            ("w_qkv", (3 * H, H), H ** -0.5, 0.0),
            ("b_qkv", (3 * H,), 0.02, 0.0),
            ("w_o", (H, H), H ** -0.5, 0.0),
            ("b_o", (H,), 0.02, 0.0),
            ("ln1_g", (H,), 0.02, 1.0),
            ("ln1_b", (H,), 0.02, 0.0),
            ("w_1", (F, H), H ** -0.5, 0.0),
            ("b_1", (F,), 0.02, 0.0),
            ("w_2", (H, F), F ** -0.5, 0.0),
            ("b_2", (H,), 0.02, 0.0),
            ("ln2_g", (H,), 0.02, 1.0),
            ("ln2_b", (H,), 0.02, 0.0),
        ]
    raise NotImplementedError(cfg.arch)


def ramp_tensor_specs(cfg: ModelConfig):
    H, C = cfg.hidden, cfg.classes
    if cfg.arch == "bert":   # DeeBERT ramp: pooler + (dropout) + FC
        return [
            ("w_p", (H, H), H ** -0.5, 0.0),
            ("b_p", (H,), 0.02, 0.0),
            ("w_c", (C, H), cfg.cls_gain * H ** -0.5, 0.0),
            ("b_c", (C,), 0.02, 0.0),
        ]
    if cfg.arch == "vit":    # LN + linear head on the CLS token
        return [
            ("ln_g", (H,), 0.02, 1.0),
            ("ln_b", (H,), 0.02, 0.0),
            ("w_c", (C, H), cfg.cls_gain * H ** -0.5, 0.0),
            ("b_c", (C,), 0.02, 0.0),
        ]
    raise NotImplementedError(cfg.arch)


def make_layer(cfg: ModelConfig, layer: int, seed: int = 0) -> Dict[str, np.ndarray]:
    return {n: _normal(seed, layer, f"L.{n}", s, sd, mu)
            for (n, s, sd, mu) in layer_tensor_specs(cfg)}


def make_ramp(cfg: ModelConfig, ramp: int, seed: int = 0) -> Dict[str, np.ndarray]:
    return {n: _normal(seed, 10_000 + ramp, f"R.{n}", s, sd, mu)
            for (n, s, sd, mu) in ramp_tensor_specs(cfg)}


def make_weights(cfg: ModelConfig, seed: int = 0):
    """{"layers": [dict per layer], "ramps": [dict per ramp]} (float32, bf16-valued)."""
    return {
        "layers": [make_layer(cfg, l, seed) for l in range(cfg.layers)],
        "ramps": [make_ramp(cfg, r, seed) for r in range(cfg.n_ramps)],
    }


def make_inputs(cfg: ModelConfig, ids: Iterable[int], seed: int = 1, threads: int = 0) -> np.ndarray:
    """Embedded inputs X0[i] of shape [n, S, H] (C16: embeddings are upstream).

    Input i is drawn from its own stream (seed, i): any subset regenerates
    identically.  Large requests are filled by a thread pool (NumPy releases
    the GIL while filling)."""
    ids = [int(i) for i in ids]
    out = np.empty((len(ids), cfg.seq, cfg.hidden), dtype=np.float32)

    def fill(lo, hi):
        for k in range(lo, hi):
            g = _rng(seed, _KIND_INPUT, ids[k])
            g.standard_normal(size=(cfg.seq, cfg.hidden), dtype=np.float32, out=out[k])
            out[k] = bf16_round(out[k])

    n = len(ids)
    nt = threads or min(32, len(os.sched_getaffinity(0)))
    if n * cfg.seq * cfg.hidden < (1 << 22) or nt <= 1:
        fill(0, n)
    else:
        from concurrent.futures import ThreadPoolExecutor
        step = (n + nt - 1) // nt
        with ThreadPoolExecutor(nt) as ex:
            list(ex.map(lambda lo: fill(lo, min(n, lo + step)), range(0, n, step)))
    return out
