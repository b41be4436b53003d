"""Early-exit LLM decode step — TEST INFRASTRUCTURE ONLY.

PAPER.md evaluates early-exit LLMs where "we replicate the final layer as the
exit ramp", checks exits only at split ends because of the
vocabulary-sized ramp, and restricts itself to one-token outputs
because KV handling for exited tokens "is an open problem".  The
readings (R22-R24):

  decode layer (Llama-2 shape), one new token per sequence against its
  pre-filled KV cache, at position p = the sequence's cached length:
      n1 = RMSNorm1(x)
      q, k, v = n1 W_qkv^T split by heads;  q, k <- RoPE(q, k; p) (rotate-half, theta)
      K[p], V[p] <- k, v                    (the cache grows by this token)
      a = concat_h softmax(q_h K_{g(h)}[0..p]^T / sqrt d) V_{g(h)}[0..p]
      h = x + a W_o^T
      n2 = RMSNorm2(h)
      x' = h + (SiLU(n2 W_gate^T) * (n2 W_up^T)) W_down^T
  ramp (the model's final norm + LM head, shared by every ramp):
      z = RMSNorm_f(x') W_lm^T;  metric = max softmax z (P:1882-1884 uses a
      softmax confidence); exit iff metric > tau; the last ramp exits all.

Exited tokens write no KV for the layers they skip; nothing reads it (R24).

``mode``: "fp64" (plain) or "bf16" (float64 with RNE to bf16 at the storage
points of DESIGN.md "Rounding contract": n1, q/k (after RoPE), v, a, h, n2,
the SwiGLU product, x', and the ramp's normalised row).

Pins (tests/test_oracle_llama.py): the decode layer equals transformers'
``LlamaDecoderLayer`` in float64 applied to a whole prefix with a causal mask
(its last position = our decode step against the prefix's cache, and the
cache entry we write = its cache at that position); RoPE at position 0 is the
identity and preserves norms; attention over a single key returns V;
RMSNorm of a constant vector is sign * gamma; W_gate = 0 makes the MLP vanish;
the ramp equals ``LlamaRMSNorm`` + ``nn.Linear``; brute force over all ramps
equals the early-stopping run.
"""
from __future__ import annotations

from typing import List, Optional, Sequence

import numpy as np

from .model import ExitRecord
from .numerics import store
from .ramp import metric, passes


def rms_norm(x, g, eps):
    """x / sqrt(mean(x^2) + eps) * g over the last axis."""
    return x / np.sqrt(np.mean(x * x, axis=-1, keepdims=True) + eps) * g


def rope(v, pos, theta):
    """Rotary embedding, rotate-half convention, of v [..., d] at integer
    positions pos (broadcast over v's leading axes):
        angle_j = pos * theta^(-2j/d),  j < d/2
        out = v * [cos, cos] + [-v_hi, v_lo] * [sin, sin]."""
    d = v.shape[-1]
    inv = theta ** (-np.arange(0, d, 2, dtype=np.float64) / d)
    ang = np.asarray(pos, dtype=np.float64)[..., None] * inv
    cos = np.concatenate([np.cos(ang), np.cos(ang)], axis=-1)
    sin = np.concatenate([np.sin(ang), np.sin(ang)], axis=-1)
    rot = np.concatenate([-v[..., d // 2:], v[..., :d // 2]], axis=-1)
    return v * cos + rot * sin


def silu(x):
    return x / (1.0 + np.exp(-x))


def decode_layer(cfg, x, W, K, V, pos, mode="fp64"):
    """One decode layer for n tokens.

    x [n, H]; K, V [n, kvh, max_ctx, d] -- the caches of the tokens' sequences,
    written in place at pos[i]; pos [n] ints.  Returns x' [n, H]."""
    n, H = x.shape
    nh, d = cfg.heads, cfg.head_dim
    kvh = cfg.kv_heads or nh
    group = nh // kvh
    eps = cfg.norm_eps
    n1 = store(rms_norm(x, W["ln1_g"], eps), mode)
    qkv = n1 @ W["w_qkv"].T
    q = qkv[:, :nh * d].reshape(n, nh, d)
    k = qkv[:, nh * d:(nh + kvh) * d].reshape(n, kvh, d)
    v = qkv[:, (nh + kvh) * d:].reshape(n, kvh, d)
    pos = np.asarray(pos, dtype=np.int64)
    q = store(rope(q, pos[:, None], cfg.rope_theta), mode)
    k = store(rope(k, pos[:, None], cfg.rope_theta), mode)
    v = store(v, mode)
    a = np.empty((n, nh, d))
    for i in range(n):
        p = int(pos[i])
        K[i, :, p, :] = k[i]
        V[i, :, p, :] = v[i]
        for h in range(nh):
            g = h // group
            s = K[i, g, :p + 1, :] @ q[i, h] / np.sqrt(d)
            w = np.exp(s - s.max())
            a[i, h] = (w @ V[i, g, :p + 1, :]) / w.sum()
    a = store(a.reshape(n, nh * d), mode)
    hh = store(x + a @ W["w_o"].T, mode)
    n2 = store(rms_norm(hh, W["ln2_g"], eps), mode)
    act = store(silu(n2 @ W["w_gate"].T) * (n2 @ W["w_up"].T), mode)
    return store(hh + act @ W["w_down"].T, mode)


def ramp_logits(cfg, x, R, mode="fp64"):
    """z = RMSNorm_f(x) W_lm^T (the copied final layer)."""
    nf = store(rms_norm(x, R["ln_g"], cfg.norm_eps), mode)
    return nf @ R["w_c"].T


def _as64(W):
    return {k: np.asarray(v, dtype=np.float64) for k, v in W.items()}


def run_split(cfg, weights, X, begin: int, end: int, ids: Sequence[int], kv, slot_of_id, pos_of_slot,
              tau=None, mode: str = "fp64", inner: str = "exact", record_all: bool = False):
    """Decode layers [begin, end) (ending in a ramp) for the tokens X [n, H].

    weights["layers"][l] / weights["ramps"][r]: dicts (may be lazy sequences);
    kv[l]: array [2, n_slots, kvh, max_ctx, d] updated in place at the tokens'
    positions; slot_of_id[id] -> slot; pos_of_slot[slot] -> position of the new
    token.  Same return values as oracle.model.run_split:
    (records of the tokens exiting here, survivor ids in order, survivors'
    hidden rows [k, H], {id: min margin}).  record_all: also return every
    ramp's metric per token (brute-force pin)."""
    X = np.asarray(X, dtype=np.float64).reshape(len(ids), cfg.hidden)
    n = X.shape[0]
    ids = [int(i) for i in ids]
    tau = cfg.tau if tau is None else tau
    last = cfg.n_ramps - 1
    ramps_in = [r for r, l in enumerate(cfg.ramp_layers) if begin <= l < end]
    assert ramps_in and cfg.ramp_layers[ramps_in[-1]] == end - 1, "a split must end in a ramp"
    en = set(ramps_in) if inner == "exact" else {ramps_in[-1]}
    ramp_at = {cfg.ramp_layers[r]: r for r in ramps_in}
    slots = np.array([int(slot_of_id[i]) for i in ids], dtype=np.int64)
    pos = np.array([int(pos_of_slot[s]) for s in slots], dtype=np.int64)
    exited = {}
    alive = np.arange(n)
    margin = np.full(n, np.inf)
    h = X
    for l in range(begin, end):
        if alive.size == 0:
            break
        cache = kv[l]
        K = cache[0][slots[alive]].astype(np.float64)
        V = cache[1][slots[alive]].astype(np.float64)
        h = decode_layer(cfg, h, _as64(weights["layers"][l]), K, V, pos[alive], mode)
        cache[0][slots[alive]] = K
        cache[1][slots[alive]] = V
        r = ramp_at.get(l)
        if r is None or r not in en:
            continue
        z = ramp_logits(cfg, h, _as64(weights["ramps"][r]), mode)
        m = metric(cfg.test, z)
        if r == last:
            ok = np.ones(alive.size, dtype=bool)
        else:
            ok = passes(cfg.test, m, tau[r])
            margin[alive] = np.minimum(margin[alive], np.abs(m - np.float64(np.float32(tau[r]))))
        for j in np.nonzero(ok)[0]:
            i = alive[j]
            exited[i] = ExitRecord(ids[i], l, r, int(np.argmax(z[j])), float(m[j]), z[j].copy(),
                                   float(margin[i]))
        alive, h = alive[~ok], h[~ok]
    recs = [exited[i] for i in sorted(exited)]
    return recs, [ids[i] for i in alive], h, {ids[i]: float(margin[i]) for i in range(n)}


def run(cfg, weights, X, ids, kv, slot_of_id, pos_of_slot, tau=None, mode="fp64") -> List[ExitRecord]:
    """The whole early-exit decode step of every token (records in input order)."""
    recs, surv, _, _ = run_split(cfg, weights, X, 0, cfg.layers, ids, kv, slot_of_id, pos_of_slot, tau, mode)
    assert not surv, "a token did not exit"
    by_id = {r.id: r for r in recs}
    return [by_id[int(i)] for i in ids]


def brute_force(cfg, weights, X, ids, kv, slot_of_id, pos_of_slot, tau=None, mode="fp64"):
    """Every layer and every ramp for every token, then the first passing ramp.
    Returns (exit_layer[n], logits [n, R, V], metric [n, R])."""
    X = np.asarray(X, dtype=np.float64).reshape(len(ids), cfg.hidden)
    tau = cfg.tau if tau is None else tau
    ids = [int(i) for i in ids]
    slots = np.array([int(slot_of_id[i]) for i in ids], dtype=np.int64)
    pos = np.array([int(pos_of_slot[s]) for s in slots], dtype=np.int64)
    ramp_at = {l: r for r, l in enumerate(cfg.ramp_layers)}
    n, R = X.shape[0], cfg.n_ramps
    Z = np.zeros((n, R, cfg.classes))
    M = np.zeros((n, R))
    h = X
    for l in range(cfg.layers):
        cache = kv[l]
        K = cache[0][slots].astype(np.float64)
        V = cache[1][slots].astype(np.float64)
        h = decode_layer(cfg, h, _as64(weights["layers"][l]), K, V, pos, mode)
        cache[0][slots] = K
        cache[1][slots] = V
        if l in ramp_at:
            r = ramp_at[l]
            Z[:, r] = ramp_logits(cfg, h, _as64(weights["ramps"][r]), mode)
            M[:, r] = metric(cfg.test, Z[:, r])
    exit_layer = np.empty(n, dtype=np.int64)
    for i in range(n):
        first = R - 1
        for r in range(R - 1):
            if passes(cfg.test, M[i, r], tau[r]):
                first = r
                break
        exit_layer[i] = cfg.ramp_layers[first]
    return exit_layer, Z, M
