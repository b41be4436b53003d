"""-m gpu: multi-step greedy early-exit decode with the K/V of skipped layers
filled from the exit state (e3_decode_run; R27)
vs oracle.llama.run_steps.

FP32 mode against the fp64 oracle: every step's token exact wherever the
oracle's decision is clear (threshold margin and top-2 logit gap > 1e-3 at
every step of that sequence so far), and every cache entry the steps wrote --
by the layers a token ran and by the fill of the layers it skipped -- within
1e-4.  bf16: the first step's decisions exact at margin > 1e-3 (as e3_pipeline_run)
and the invariants of every step (one token per sequence per step, positions
advanced, every layer's entry written)."""
import numpy as np
import pytest
import torch

import e3data
from oracle import llama as olm
from tests.gpu_util import DEV, requires_cuda

pytestmark = [pytest.mark.gpu, requires_cuda]


@pytest.fixture(scope="module")
def api():
    from paper_conf_sosp_iyergdpgn24_b200 import api as A
    return A


def _run(api, cfg, n, steps, dtype):
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    max_ctx = cfg.ctx + steps
    kv_np = [e3data.make_kv(cfg, l, range(n), max_ctx) for l in range(cfg.layers)]
    cache = api.KVCache(cfg, n, max_ctx, n, DEV, dtype=dtype)
    for l in range(cfg.layers):
        cache.k[l].copy_(torch.from_numpy(kv_np[l][0]).to(tdt))
        cache.v[l].copy_(torch.from_numpy(kv_np[l][1]).to(tdt))
    cache.slot_of_id.copy_(torch.arange(n, dtype=torch.int32))
    cache.pos_of_slot.fill_(cfg.ctx)
    W = e3data.make_weights(cfg)
    model = api.DeviceModel(cfg, W, DEV, kv=cache)
    E = e3data.make_embed(cfg)
    X0 = e3data.make_inputs(cfg, range(n), seed=5)[:, 0, :]
    x = torch.from_numpy(X0).to(DEV).to(tdt).contiguous()
    ids = torch.arange(n, dtype=torch.int64, device=DEV)
    emb = torch.from_numpy(E).to(DEV).to(tdt)
    ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV, hidden=cfg.hidden, hidden_dtype=tdt)
    from oracle.pipeline_sim import Plan
    pipe = api.Pipeline(model, api.make_plan(cfg, Plan.per_ramp(cfg.ramp_layers).bounds, cfg.tau, dtype=dtype))
    tokens, st = pipe.decode(x, ids, steps, emb, ex)
    torch.cuda.synchronize()
    kv_or = [k.astype(np.float64) for k in kv_np]
    pos_of = {s: cfg.ctx for s in range(n)}
    mode = "fp64" if dtype == "fp32" else "bf16"
    recs, otok, filled = olm.run_steps(cfg, W, X0, list(range(n)), kv_or, {i: i for i in range(n)}, pos_of, E,
                                       steps, mode=mode)
    return tokens.cpu().numpy(), cache, kv_or, recs, otok, filled, st


def _clear(r, eps):
    z = np.sort(r.logits)
    return r.margin > eps and z[-1] - z[-2] > eps


def test_decode_fp32_tokens_and_filled_cache(api):
    cfg = e3data.get("tiny-llama")
    n, steps = 32, 4
    tok, cache, kv_or, recs, otok, filled, st = _run(api, cfg, n, steps, "fp32")
    assert st.runs > 0 and any(filled.values())           # some layers were filled
    good = np.ones(n, dtype=bool)
    checked = 0
    for s in range(steps):
        for i in range(n):
            if not good[i]:
                continue
            if not _clear(recs[s][i], 1e-3):
                good[i] = False                              # this sequence's later steps may legitimately differ
                continue
            assert tok[s, i] == otok[s, i], (s, i)
            checked += 1
    assert checked >= 0.8 * n * steps
    # every entry the steps wrote (run layers and filled layers), for the clear sequences
    for l in range(cfg.layers):
        kg, vg = cache.k[l].cpu().numpy(), cache.v[l].cpu().numpy()
        for i in np.nonzero(good)[0]:
            for p in range(cfg.ctx, cfg.ctx + steps):
                assert np.max(np.abs(kg[i, :, p] - kv_or[l][0][i, :, p])) < 1e-4, (l, i, p)
                assert np.max(np.abs(vg[i, :, p] - kv_or[l][1][i, :, p])) < 1e-4, (l, i, p)
    assert (cache.pos_of_slot.cpu().numpy() == cfg.ctx + steps).all()


def test_decode_bf16_invariants_and_first_step(api):
    cfg = e3data.get("tiny-llama")
    n, steps = 40, 3                                          # two batches of B = 32 (the second padded)
    tok, cache, kv_or, recs, otok, filled, st = _run(api, cfg, n, steps, "bf16")
    assert tok.shape == (steps, n) and (tok >= 0).all() and (tok < cfg.classes).all()
    for i in range(n):
        if _clear(recs[0][i], 1e-3):
            assert tok[0, i] == otok[0, i]
    for l in range(cfg.layers):                               # every layer has an entry at every step's position
        kg = cache.k[l].float().cpu().numpy()
        assert np.all(np.abs(kg[:, :, cfg.ctx:cfg.ctx + steps]).sum(axis=-1) > 0)
    assert (cache.pos_of_slot.cpu().numpy() == cfg.ctx + steps).all()
