"""Pins for oracle.llama (the early-exit LLM decode step):
transformers' LlamaDecoderLayer / LlamaRMSNorm in float64, closed forms and
brute force."""
import dataclasses

import numpy as np
import pytest
import torch

import e3data
from oracle import llama


def _cfg(H=64, nh=2, kvh=2, F=96, V=50, ramps=(0,), L=1, eps=1e-5):
    return dataclasses.replace(e3data.get("tiny-llama"), hidden=H, heads=nh, kv_heads=kvh, ffn=F, classes=V,
                               ramp_layers=ramps, layers=L, norm_eps=eps, tau=(0.5,) * len(ramps))


def _rand_layer(cfg, rng):
    H, F, d, nh, kvh = cfg.hidden, cfg.ffn, cfg.head_dim, cfg.heads, cfg.kv_heads
    return {"w_qkv": rng.standard_normal(((nh + 2 * kvh) * d, H)) / np.sqrt(H),
            "w_o": rng.standard_normal((H, nh * d)) / np.sqrt(H),
            "w_gate": rng.standard_normal((F, H)) / np.sqrt(H),
            "w_up": rng.standard_normal((F, H)) / np.sqrt(H),
            "w_down": rng.standard_normal((H, F)) / np.sqrt(F),
            "ln1_g": 1 + 0.1 * rng.standard_normal(H), "ln2_g": 1 + 0.1 * rng.standard_normal(H)}


@pytest.mark.parametrize("nh,kvh,theta", [(2, 2, None), (2, 1, None), (4, 1, 500000.0)])
def test_decode_layer_matches_transformers_llama_layer(nh, kvh, theta):
    """(4, 1, 5e5): a group of four query heads per KV head and the Llama-3
    RoPE base, as in the Llama-3.1-8B-shaped config (e3data l8)."""
    from transformers import DynamicCache, LlamaConfig
    from transformers.models.llama import modeling_llama as ml
    cfg = _cfg(H=32 * nh, nh=nh, kvh=kvh)
    if theta is not None:
        cfg = dataclasses.replace(cfg, rope_theta=theta)
    H, nh, d, T = cfg.hidden, cfg.heads, cfg.head_dim, 7
    rng = np.random.default_rng(kvh)
    W = _rand_layer(cfg, rng)
    hc = LlamaConfig(hidden_size=H, intermediate_size=cfg.ffn, num_attention_heads=nh, num_key_value_heads=kvh,
                     head_dim=d, rms_norm_eps=cfg.norm_eps, rope_theta=cfg.rope_theta,
                     max_position_embeddings=64, attention_bias=False, mlp_bias=False)
    hc._attn_implementation = "eager"
    layer = ml.LlamaDecoderLayer(hc, layer_idx=0).double()
    rot = ml.LlamaRotaryEmbedding(hc).double()
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a))
    with torch.no_grad():
        a = layer.self_attn
        a.q_proj.weight.copy_(t(W["w_qkv"][:nh * d]))
        a.k_proj.weight.copy_(t(W["w_qkv"][nh * d:(nh + kvh) * d]))
        a.v_proj.weight.copy_(t(W["w_qkv"][(nh + kvh) * d:]))
        a.o_proj.weight.copy_(t(W["w_o"]))
        layer.mlp.gate_proj.weight.copy_(t(W["w_gate"]))
        layer.mlp.up_proj.weight.copy_(t(W["w_up"]))
        layer.mlp.down_proj.weight.copy_(t(W["w_down"]))
        layer.input_layernorm.weight.copy_(t(W["ln1_g"]))
        layer.post_attention_layernorm.weight.copy_(t(W["ln2_g"]))
        x = rng.standard_normal((1, T, H))
        pos = torch.arange(T)[None]
        # HF builds cos/sin in float32 (inv_freq.float()); the same convention
        # (emb = cat(freqs, freqs)) in float64 so the pin is not limited by it
        inv = 1.0 / (cfg.rope_theta ** (torch.arange(0, d, 2, dtype=torch.float64) / d))
        freqs = pos[0].double()[:, None] * inv[None]
        emb = torch.cat([freqs, freqs], dim=-1)[None]
        cos, sin = emb.cos(), emb.sin()
        c32, _ = rot(t(x), pos)
        assert torch.allclose(c32, cos, atol=1e-5)       # same convention as the library's
        mask = torch.full((T, T), float("-inf"), dtype=torch.float64).triu(1)[None, None]
        cache = DynamicCache(config=hc)
        out = layer(t(x), attention_mask=mask, position_ids=pos, past_key_values=cache, use_cache=True,
                    position_embeddings=(cos, sin)).numpy()
        hk, hv = cache.layers[0].keys.numpy(), cache.layers[0].values.numpy()   # [1, kvh, T, d]
    K = np.zeros((1, kvh, T, d))
    V = np.zeros((1, kvh, T, d))
    K[:, :, :T - 1], V[:, :, :T - 1] = hk[:, :, :T - 1], hv[:, :, :T - 1]
    got = llama.decode_layer(cfg, x[0, T - 1:], W, K, V, np.array([T - 1]))
    # LlamaRMSNorm normalises in float32 whatever the module dtype: agreement
    # to ~1e-7 relative; a structural slip (term, sign, index, transpose)
    # moves the output by O(0.01 .. 1)
    np.testing.assert_allclose(got[0], out[0, T - 1], rtol=1e-5, atol=1e-5)
    np.testing.assert_allclose(K[0, :, T - 1], hk[0, :, T - 1], rtol=1e-5, atol=1e-5)
    np.testing.assert_allclose(V[0, :, T - 1], hv[0, :, T - 1], rtol=1e-5, atol=1e-5)
    # the prefix's keys/values (what we attended over) are the library's own
    assert not np.allclose(got[0], x[0, T - 1], atol=1e-2)


def test_rope_identity_at_zero_and_norm_preserving():
    rng = np.random.default_rng(0)
    v = rng.standard_normal((3, 4, 128))
    assert np.array_equal(llama.rope(v, np.zeros((3, 4), dtype=np.int64), 10000.0), v)
    r = llama.rope(v, np.full((3, 4), 517), 10000.0)
    np.testing.assert_allclose(np.linalg.norm(r, axis=-1), np.linalg.norm(v, axis=-1), rtol=1e-13)
    # relative position property: <R_p q, R_s k> depends on p - s only
    q, k = v[0, 0], v[0, 1]
    dot = lambda p, s: llama.rope(q, np.array(p), 500.0) @ llama.rope(k, np.array(s), 500.0)
    assert abs(dot(9, 4) - dot(105, 100)) < 1e-9


def test_single_key_attention_returns_v_and_zero_gate_kills_mlp():
    """pos = 0 (empty cache): a = v; with W_o = I and W_gate = 0 the layer is
    x' = x + RMSNorm1(x) W_v^T exactly (SiLU(0) = 0)."""
    cfg = _cfg(H=64, nh=2, kvh=2)
    rng = np.random.default_rng(1)
    W = _rand_layer(cfg, rng)
    W["w_o"] = np.eye(64)
    W["w_gate"] = np.zeros_like(W["w_gate"])
    x = rng.standard_normal((2, 64))
    K = np.zeros((2, 2, 5, 32))
    V = np.zeros((2, 2, 5, 32))
    got = llama.decode_layer(cfg, x, W, K, V, np.array([0, 0]))
    n1 = x / np.sqrt(np.mean(x * x, axis=-1, keepdims=True) + cfg.norm_eps) * W["ln1_g"]
    v = n1 @ W["w_qkv"][128:].T
    np.testing.assert_allclose(got, x + v, rtol=1e-12, atol=1e-12)


def test_rms_norm_constant_vector():
    g = np.linspace(0.5, 2.0, 16)
    for c in (3.0, -0.25):
        np.testing.assert_allclose(llama.rms_norm(np.full(16, c), g, 1e-12), np.sign(c) * g, rtol=1e-9)


def test_ramp_matches_transformers_rmsnorm_and_linear():
    from transformers.models.llama.modeling_llama import LlamaRMSNorm
    cfg = _cfg(H=32, V=70)
    rng = np.random.default_rng(2)
    R = {"ln_g": 1 + 0.1 * rng.standard_normal(32), "w_c": rng.standard_normal((70, 32))}
    x = rng.standard_normal((5, 32)) * 3
    norm = LlamaRMSNorm(32, eps=cfg.norm_eps).double()
    lin = torch.nn.Linear(32, 70, bias=False).double()
    with torch.no_grad():
        norm.weight.copy_(torch.from_numpy(R["ln_g"]))
        lin.weight.copy_(torch.from_numpy(R["w_c"]))
        ref = lin(norm(torch.from_numpy(x))).numpy()
    np.testing.assert_allclose(llama.ramp_logits(cfg, x, R), ref, rtol=1e-5, atol=1e-5)   # float32 RMSNorm


@pytest.mark.parametrize("mode", ["fp64", "bf16"])
def test_early_exit_equals_brute_force_and_cache_writes(mode):
    cfg = e3data.get("tiny-llama")
    W = e3data.make_weights(cfg)
    N = 24
    ids = list(range(100, 100 + N))
    slot_of = {i: (i * 7) % 31 for i in ids}
    pos_of = {s: cfg.ctx - (s % 5) for s in range(31)}
    X = e3data.make_inputs(cfg, ids, seed=2)[:, 0, :]
    mk = lambda: [e3data.make_kv(cfg, l, range(31), cfg.ctx + 1).astype(np.float64) for l in range(cfg.layers)]
    kv_a, kv_b, pristine = mk(), mk(), mk()
    el, Z, M = llama.brute_force(cfg, W, X, ids, kv_a, slot_of, pos_of, mode=mode)
    recs = llama.run(cfg, W, X, ids, kv_b, slot_of, pos_of, mode=mode)
    assert [r.exit_layer for r in recs] == el.tolist()
    assert 0 < sum(e == 1 for e in el) < N                     # both ramps used
    for j, r in enumerate(recs):
        np.testing.assert_array_equal(r.logits, Z[j, cfg.ramp_layers.index(r.exit_layer)])
        # R24: the cache grows at the token's position only for the layers it ran
        s, p = slot_of[r.id], pos_of[slot_of[r.id]]
        for l in range(cfg.layers):
            wrote = not np.array_equal(kv_b[l][0][s, :, p], pristine[l][0][s, :, p])
            assert wrote == (l <= r.exit_layer), (r.id, l)
    # a split chain reproduces the whole run
    kv_c = mk()
    r0, surv, h, _ = llama.run_split(cfg, W, X, 0, 2, ids, kv_c, slot_of, pos_of, mode=mode)
    r1, surv1, _, _ = llama.run_split(cfg, W, h, 2, 4, surv, kv_c, slot_of, pos_of, mode=mode)
    assert not surv1
    by = {r.id: r for r in r0 + r1}
    for r in recs:
        assert by[r.id].exit_layer == r.exit_layer
        np.testing.assert_array_equal(by[r.id].logits, r.logits)
