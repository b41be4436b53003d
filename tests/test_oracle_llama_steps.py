"""Pins for the multi-step early-exit decode of oracle/llama.py (run_steps,
fill_kv; R27).

* transformers: greedy decode of a 2-layer model from an empty cache equals a
  causal LlamaDecoderLayer stack (float64) run over the generated sequence --
  without early exit, and WITH exits after layer 0 (for two layers, state
  propagation gives the skipped layer exactly the input the plain forward
  gives it, so the caches agree and only the exited tokens' logits come from
  the inner ramp);
* the fill rule equals the K/V the decode layer itself appends for input h;
* invariants: every token exits once per step, positions advance by one per
  step, the filled layers of a token are exactly those after its exit layer.
"""
import dataclasses

import numpy as np
import pytest
import torch

import e3data
from oracle import llama


def _cfg(L=2, ramps=(1,), tau=(1.5,), V=40, H=64, nh=2, kvh=2, F=96):
    return dataclasses.replace(e3data.get("tiny-llama"), layers=L, hidden=H, heads=nh, kv_heads=kvh, ffn=F,
                               classes=V, ramp_layers=ramps, tau=tau, ctx=0, norm_eps=1e-5)


def _weights(cfg, seed):
    rng = np.random.default_rng(seed)
    H, F, d, nh, kvh = cfg.hidden, cfg.ffn, cfg.head_dim, cfg.heads, cfg.kv_heads
    layers = [{"w_qkv": rng.standard_normal(((nh + 2 * kvh) * d, H)) / np.sqrt(H),
               "w_o": rng.standard_normal((H, nh * d)) / np.sqrt(H),
               "w_gate": rng.standard_normal((F, H)) / np.sqrt(H),
               "w_up": rng.standard_normal((F, H)) / np.sqrt(H),
               "w_down": rng.standard_normal((H, F)) / np.sqrt(F),
               "ln1_g": 1 + 0.1 * rng.standard_normal(H), "ln2_g": 1 + 0.1 * rng.standard_normal(H)}
              for _ in range(cfg.layers)]
    ramp = {"ln_g": 1 + 0.1 * rng.standard_normal(H), "w_c": 3 * rng.standard_normal((cfg.classes, H)) / np.sqrt(H)}
    embed = rng.standard_normal((cfg.classes, H))
    return {"layers": layers, "ramps": [ramp] * cfg.n_ramps}, embed


def _hf_stack(cfg, W):
    from transformers import LlamaConfig
    from transformers.models.llama import modeling_llama as ml
    H, nh, kvh, d = cfg.hidden, cfg.heads, cfg.kv_heads, cfg.head_dim
    hc = LlamaConfig(hidden_size=H, intermediate_size=cfg.ffn, num_attention_heads=nh, num_key_value_heads=kvh,
                     head_dim=d, rms_norm_eps=cfg.norm_eps, rope_theta=cfg.rope_theta,
                     max_position_embeddings=64, attention_bias=False, mlp_bias=False)
    hc._attn_implementation = "eager"
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a))
    layers = []
    with torch.no_grad():
        for l, Wl in enumerate(W["layers"]):
            m = ml.LlamaDecoderLayer(hc, layer_idx=l).double()
            a = m.self_attn
            a.q_proj.weight.copy_(t(Wl["w_qkv"][:nh * d]))
            a.k_proj.weight.copy_(t(Wl["w_qkv"][nh * d:(nh + kvh) * d]))
            a.v_proj.weight.copy_(t(Wl["w_qkv"][(nh + kvh) * d:]))
            a.o_proj.weight.copy_(t(Wl["w_o"]))
            m.mlp.gate_proj.weight.copy_(t(Wl["w_gate"]))
            m.mlp.up_proj.weight.copy_(t(Wl["w_up"]))
            m.mlp.down_proj.weight.copy_(t(Wl["w_down"]))
            m.input_layernorm.weight.copy_(t(Wl["ln1_g"]))
            m.post_attention_layernorm.weight.copy_(t(Wl["ln2_g"]))
            layers.append(m)
        norm = ml.LlamaRMSNorm(H, eps=cfg.norm_eps).double()
        norm.weight.copy_(t(W["ramps"][0]["ln_g"]))
    return layers, norm


def _hf_forward(cfg, W, seq):
    """Per-layer outputs [L][T, H] of the causal stack on the input rows seq [T, H]."""
    layers, norm = _hf_stack(cfg, W)
    T, d = seq.shape[0], cfg.head_dim
    pos = torch.arange(T)[None]
    inv = 1.0 / (cfg.rope_theta ** (torch.arange(0, d, 2, dtype=torch.float64) / d))
    emb = torch.cat([pos[0].double()[:, None] * inv[None]] * 2, dim=-1)[None]
    mask = torch.full((T, T), float("-inf"), dtype=torch.float64).triu(1)[None, None]
    h = torch.from_numpy(seq[None].copy())
    outs = []
    with torch.no_grad():
        for m in layers:
            h = m(h, attention_mask=mask, position_ids=pos, position_embeddings=(emb.cos(), emb.sin()))
            if isinstance(h, tuple):
                h = h[0]
            outs.append(h[0].numpy().copy())
    lg = lambda x: (norm(torch.from_numpy(x)).detach().numpy() @ W["ramps"][0]["w_c"].T)
    return outs, lg


def _decode(cfg, W, embed, x0, steps, n=1):
    max_ctx = steps
    kv = [np.zeros((2, n, cfg.kv_heads, max_ctx, cfg.head_dim)) for _ in range(cfg.layers)]
    slot_of = {i: i for i in range(n)}
    pos_of = {i: 0 for i in range(n)}
    recs, tokens, filled = llama.run_steps(cfg, W, x0, list(range(n)), kv, slot_of, pos_of, embed, steps)
    return recs, tokens, filled, kv, pos_of


def test_greedy_decode_without_exits_equals_transformers():
    cfg = _cfg()
    W, E = _weights(cfg, 0)
    x0 = np.random.default_rng(1).standard_normal((1, cfg.hidden))
    steps = 4
    recs, tokens, filled, kv, pos_of = _decode(cfg, W, E, x0, steps)
    assert not filled and pos_of[0] == steps
    seq = np.concatenate([x0, E[tokens[:-1, 0]]], axis=0)          # the inputs the decode consumed
    outs, lg = _hf_forward(cfg, W, seq)
    for s in range(steps):
        np.testing.assert_allclose(recs[s][0].logits, lg(outs[-1][s:s + 1])[0], rtol=1e-5, atol=1e-5)
        assert tokens[s, 0] == int(np.argmax(lg(outs[-1][s:s + 1])[0]))


def test_greedy_decode_with_exits_after_layer0_equals_transformers():
    """Ramps after both layers, a threshold that lets some steps exit after
    layer 0: the cache the next steps attend over (layer 1 filled from the
    exit state) is the plain forward's, so HF's per-layer outputs give every
    step's logits at the layer it exited."""
    cfg = _cfg(ramps=(0, 1), tau=(0.6, 0.6))
    W, E = _weights(cfg, 3)
    x0 = np.random.default_rng(4).standard_normal((1, cfg.hidden))
    steps = 8
    recs, tokens, filled, kv, _ = _decode(cfg, W, E, x0, steps)
    layers_hit = {recs[s][0].exit_layer for s in range(steps)}
    assert layers_hit == {0, 1}, layers_hit                       # both kinds of step occur
    seq = np.concatenate([x0, E[tokens[:-1, 0]]], axis=0)
    outs, lg = _hf_forward(cfg, W, seq)
    for s in range(steps):
        e = recs[s][0].exit_layer
        np.testing.assert_allclose(recs[s][0].logits, lg(outs[e][s:s + 1])[0], rtol=1e-5, atol=1e-5)
        if e == 0:
            assert filled[(s, 0)] == [1]


def test_fill_equals_the_decode_layers_own_kv_append():
    cfg = _cfg(L=1, ramps=(0,), tau=(1.5,), H=128, nh=2, kvh=1)
    W, _ = _weights(cfg, 5)
    rng = np.random.default_rng(6)
    h = rng.standard_normal((3, cfg.hidden))
    pos = np.array([0, 3, 5])
    for mode in ("fp64", "bf16"):
        K1, V1 = np.zeros((3, 1, 6, 64)), np.zeros((3, 1, 6, 64))
        K2, V2 = K1.copy(), V1.copy()
        llama.fill_kv(cfg, W["layers"][0], h, K1, V1, pos, mode)
        llama.decode_layer(cfg, h, W["layers"][0], K2, V2, pos, mode)
        assert np.array_equal(K1, K2) and np.array_equal(V1, V2)


def test_multi_step_invariants_tiny_llama():
    cfg = dataclasses.replace(e3data.get("tiny-llama"), ctx=0)
    W = e3data.make_weights(cfg)
    E = e3data.make_embed(cfg)
    n, steps = 12, 3
    X = e3data.make_inputs(cfg, range(n), seed=5)[:, 0, :]
    kv = [np.zeros((2, n, cfg.kv_heads, steps, cfg.head_dim)) for _ in range(cfg.layers)]
    pos_of = {i: 0 for i in range(n)}
    recs, tokens, filled = llama.run_steps(cfg, W, X, list(range(n)), kv, {i: i for i in range(n)}, pos_of, E,
                                           steps, mode="bf16")
    assert all(p == steps for p in pos_of.values())
    for s in range(steps):
        assert [r.id for r in recs[s]] == list(range(n))
        for r in recs[s]:
            expect = list(range(r.exit_layer + 1, cfg.layers))
            assert filled.get((s, r.id), []) == expect
            assert tokens[s, r.id] == r.label
    # every layer of every sequence has an entry at every step's position
    for l in range(cfg.layers):
        assert np.all(np.abs(kv[l]).sum(axis=-1) > 0)
