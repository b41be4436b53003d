"""-m gpu: the LLaMA decode split vs oracle/llama.py.

Per split run on identical input rows and identical caches: exit decisions
exact where the margin exceeds 1e-3, logits within 2e-2 per bf16 layer
(relative above |z| = 4, R13), survivors' hidden rows close, and
the KV entries the step appends (k after RoPE, v) within bf16 rounding of
the oracle's, written only for layers a token ran (R24)."""
import dataclasses

import numpy as np
import pytest
import torch

import e3data
from oracle import llama as olm
from oracle.pipeline_sim import Plan, simulate_pipeline
from tests.gpu_util import DEV, bf16_tensor, requires_cuda, to64

pytestmark = [pytest.mark.gpu, requires_cuda]

LOGIT_TOL = 2e-2
MARGIN = 1e-3


@pytest.fixture(scope="module")
def api():
    from paper_conf_sosp_iyergdpgn24_b200 import api as A
    return A


def _setup(api, cfg, n_slots, slot_of, pos_of, id_cap, W=None):
    W = W if W is not None else e3data.make_weights(cfg)
    max_ctx = cfg.ctx + 1
    kv_np = [e3data.make_kv(cfg, l, range(n_slots), max_ctx) for l in range(cfg.layers)]
    cache = api.KVCache(cfg, n_slots, max_ctx, id_cap, DEV)
    for l in range(cfg.layers):
        cache.k[l].copy_(torch.from_numpy(kv_np[l][0]).to(torch.bfloat16))
        cache.v[l].copy_(torch.from_numpy(kv_np[l][1]).to(torch.bfloat16))
    so = np.zeros(id_cap, np.int32)
    for i, s in slot_of.items():
        so[i] = s
    cache.slot_of_id.copy_(torch.from_numpy(so))
    cache.pos_of_slot.copy_(torch.tensor([pos_of[s] for s in range(n_slots)], dtype=torch.int32))
    model = api.DeviceModel(cfg, W, DEV, kv=cache)
    return W, kv_np, cache, model


def _check_records(recs, ex, logit_tol, margin=MARGIN):
    el, lab = ex.exit_layer.cpu().numpy(), ex.label.cpu().numpy()
    conf, lg = ex.conf.cpu().numpy(), ex.logits.cpu().numpy()
    n = 0
    for r in recs:
        i = r.id
        assert el[i] >= 0
        if r.margin > margin:
            assert el[i] == r.exit_layer, (i, el[i], r.exit_layer, r.margin)
            n += 1
        if el[i] == r.exit_layer:
            tol = logit_tol * max(1.0, float(np.max(np.abs(r.logits))) / 4.0)
            assert np.max(np.abs(lg[i] - r.logits)) < tol, (i, np.max(np.abs(lg[i] - r.logits)))
            assert abs(conf[i] - r.metric) < tol
            top2 = np.sort(r.logits)[-2:]
            if top2[1] - top2[0] > 2 * tol:
                assert lab[i] == r.label
    return n


def test_llama_split_parity_and_cache_writes(api):
    """Split [0,2) on a padded batch (27 of 32 valid), then split [2,4) on the
    GPU's survivors; tokens in different slots at different positions."""
    cfg = e3data.get("tiny-llama")
    ids = list(range(5, 5 + 27))
    slot_of = {i: (3 * i) % 40 for i in ids}
    pos_of = {s: cfg.ctx - (s % 7) for s in range(40)}
    W, kv_np, cache, model = _setup(api, cfg, 40, slot_of, pos_of, 64)
    X = e3data.make_inputs(cfg, ids, seed=4)[:, 0, :]
    kv_or = [k.astype(np.float64) for k in kv_np]
    B = cfg.batch
    rows, cur_ids = X, ids
    for begin, end in ((0, 2), (2, 4)):
        xb = np.zeros((B, 1, cfg.hidden), np.float32)
        xb[:len(cur_ids), 0] = rows
        idb = np.full(B, -1, np.int64)
        idb[:len(cur_ids)] = cur_ids
        split = api.Split(model, api.split_desc(cfg, begin, end, cfg.tau))
        x = bf16_tensor(xb)
        x_out = torch.zeros_like(x)
        id_out = torch.full((B,), -9, dtype=torch.int64, device=DEV)
        n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
        ex = api.ExitBuffers(64, cfg.classes, cfg.n_ramps, DEV)
        nv = torch.tensor([len(cur_ids)], dtype=torch.int32, device=DEV)
        split.run(x, torch.from_numpy(idb).to(DEV), x_out, id_out, n_surv, ex, n_valid=nv)
        torch.cuda.synchronize()
        ns = int(n_surv.item())
        assert ns + int(ex.n_exit.item()) == len(cur_ids)
        recs, surv, h, margins = olm.run_split(cfg, W, rows, begin, end, cur_ids, kv_or, slot_of, pos_of,
                                               mode="bf16")
        _check_records(recs, ex, LOGIT_TOL * (end - begin))
        got = id_out[:ns].cpu().tolist()
        if all(m > MARGIN for m in margins.values()):
            assert got == surv
        assert torch.all(id_out[ns:] == -9)
        for i in got:
            if i in surv:
                g, o = to64(x_out[got.index(i), 0]), h[surv.index(i)]
                assert np.mean(np.abs(g - o)) < 5e-3 * max(1.0, np.mean(np.abs(o))) and np.max(np.abs(g - o)) < 0.25
        # the KV entries this split appended: GPU vs oracle, at each token's (slot, pos)
        for l in range(begin, end):
            kg, vg = to64(cache.k[l]), to64(cache.v[l])
            for i in cur_ids:
                s, p = slot_of[i], pos_of[slot_of[i]]
                ran = all(r.id != i or r.exit_layer >= l for r in recs)
                if ran:
                    ko, vo = kv_or[l][0][s, :, p], kv_or[l][1][s, :, p]
                    assert np.max(np.abs(kg[s, :, p] - ko)) < 0.05 and np.max(np.abs(vg[s, :, p] - vo)) < 0.05
                else:
                    assert np.array_equal(kg[s, :, p], kv_np[l][0][s, :, p])   # untouched (R24)
        rows = to64(x_out[:ns, 0]).astype(np.float32)
        cur_ids = got
    assert not cur_ids


def test_llama_pipeline_matches_oracle_and_simulator(api):
    cfg = e3data.get("tiny-llama")
    N = 90
    slot_of = {i: i for i in range(N)}
    pos_of = {s: cfg.ctx - (s % 3) for s in range(N)}
    W, kv_np, cache, model = _setup(api, cfg, N, slot_of, pos_of, N)
    X = e3data.make_inputs(cfg, range(N), seed=5)
    kv_or = [k.astype(np.float64) for k in kv_np]
    recs = olm.run(cfg, W, X[:, 0, :], list(range(N)), kv_or, slot_of, pos_of, mode="bf16")
    ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, DEV)
    bounds = Plan.per_ramp(cfg.ramp_layers).bounds
    pipe = api.Pipeline(model, api.make_plan(cfg, bounds, cfg.tau, lag=1, trace=True))
    pipe.run(bf16_tensor(X), torch.arange(N, dtype=torch.int64, device=DEV), ex)
    assert int(ex.n_exit.item()) == N
    n = _check_records(recs, ex, 0.1, margin=1e-2)
    assert n >= 0.8 * N
    exit_layer = {i: int(v) for i, v in enumerate(ex.exit_layer.cpu().numpy())}
    sim = simulate_pipeline(exit_layer, list(range(N)), Plan(bounds), cfg.batch, lag=1)
    assert [(r.split, r.n_valid, r.ids) for r in sim.runs] == pipe.trace()


class _LazyLayers:
    def __init__(self, cfg, n):
        self.cfg, self.n, self.cache = cfg, n, {}

    def __getitem__(self, l):
        if l not in self.cache:
            self.cache[l] = e3data.make_layer(self.cfg, l)
        return self.cache[l]

    def __len__(self):
        return self.n


@pytest.mark.parametrize("name", ["lm", "l8"])
def test_llama7b_shape_split_parity_sampled(api, name):
    """Llama-2-7B layer shapes (H 4096, 32 heads x 128, F 11008, V 32000,
    513 cache positions, B = 64) -- and the Llama-3.1-8B variant (32 query
    heads over 8 KV heads, F 14336, V 128256, RoPE base 5e5) -- on a 2-layer
    model (ramps after both): split [0,1) on a full batch, sampled tokens vs
    the oracle."""
    cfg = dataclasses.replace(e3data.get(name), layers=2, ramp_layers=(0, 1), exit_profile=None, tau=(0.2, 0.2))
    B = cfg.batch
    slot_of = {i: i for i in range(B)}
    pos_of = {s: cfg.ctx for s in range(B)}
    ramp = e3data.make_ramp(cfg, 0)
    W = {"layers": [e3data.make_layer(cfg, 0), e3data.make_layer(cfg, 1)], "ramps": [ramp, ramp]}
    W_, kv_np, cache, model = _setup(api, cfg, B, slot_of, pos_of, B, W=W)
    X = e3data.make_inputs(cfg, range(B), seed=6)
    split = api.Split(model, api.split_desc(cfg, 0, 1, cfg.tau))
    x = bf16_tensor(X)
    x_out = torch.zeros_like(x)
    id_out = torch.full((B,), -9, dtype=torch.int64, device=DEV)
    n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
    ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, DEV)
    split.run(x, torch.arange(B, dtype=torch.int64, device=DEV), x_out, id_out, n_surv, ex)
    torch.cuda.synchronize()
    ns = int(n_surv.item())
    assert ns + int(ex.n_exit.item()) == B
    sample = [0, 17, 40, 63]
    kv_or = [np.stack([kv_np[0][0][sample], kv_np[0][1][sample]]).astype(np.float64)]
    so = {i: k for k, i in enumerate(sample)}
    po = {k: cfg.ctx for k in range(len(sample))}
    recs, surv, h, margins = olm.run_split(cfg, W, X[sample, 0], 0, 1, sample, kv_or, so, po, mode="bf16")
    _check_records(recs, ex, LOGIT_TOL)
    got = id_out[:ns].cpu().tolist()
    for i in sample:
        if margins[i] > MARGIN:
            assert (i in got) == (i in surv)
    kg = to64(cache.k[0])
    for k, i in enumerate(sample):
        assert np.max(np.abs(kg[i, :, cfg.ctx] - kv_or[0][0][k, :, cfg.ctx])) < 0.05


def test_llama_multi_ramp_split_skips_kv_of_exited_tokens(api):
    """One split holding both ramps (layers [0,4), inner EXACT): a token that
    exits at the inner ramp (layer 1) writes no K/V at layers 2 and 3 (R15,
    ADVICE r01), while the tokens that run on append theirs; results equal
    the per-ramp plan bitwise."""
    cfg = e3data.get("tiny-llama")
    N = 32
    slot_of = {i: i for i in range(N)}
    pos_of = {s: cfg.ctx - (s % 4) for s in range(N)}
    W, kv_np, cache, model = _setup(api, cfg, N, slot_of, pos_of, N)
    X = e3data.make_inputs(cfg, range(N), seed=8)
    ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, DEV)
    split = api.Split(model, api.split_desc(cfg, 0, 4, cfg.tau))
    x_out = torch.zeros_like(bf16_tensor(X))
    id_out = torch.full((N,), -9, dtype=torch.int64, device=DEV)
    n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
    split.run(bf16_tensor(X), torch.arange(N, dtype=torch.int64, device=DEV), x_out, id_out, n_surv, ex)
    torch.cuda.synchronize()
    el = ex.exit_layer.cpu().numpy()
    assert int(n_surv.item()) == 0 and (el >= 0).all()
    early = [i for i in range(N) if el[i] == 1]
    late = [i for i in range(N) if el[i] == 3]
    assert early and late, el
    for l in (2, 3):
        kg, vg = to64(cache.k[l]), to64(cache.v[l])
        for i in early:
            p = pos_of[i]
            assert np.array_equal(kg[i, :, p], kv_np[l][0][i, :, p])
            assert np.array_equal(vg[i, :, p], kv_np[l][1][i, :, p])
        for i in late:
            p = pos_of[i]
            assert not np.array_equal(kg[i, :, p], kv_np[l][0][i, :, p])
    # per-ramp plan on a fresh cache: identical exits and logits
    W2, _, cache2, model2 = _setup(api, cfg, N, slot_of, pos_of, N, W=W)
    ex2 = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, DEV)
    api.Pipeline(model2, api.make_plan(cfg, (0, 2, 4), cfg.tau)).run(
        bf16_tensor(X), torch.arange(N, dtype=torch.int64, device=DEV), ex2)
    assert torch.equal(ex2.exit_layer, ex.exit_layer) and torch.equal(ex2.logits, ex.logits)
    for l in range(cfg.layers):
        assert torch.equal(cache2.k[l], cache.k[l]) and torch.equal(cache2.v[l], cache.v[l])


def test_llama_slot_outside_cache_is_an_error(api):
    """A token whose KV slot lies outside the cache is skipped and reported
    (E3_EINVAL at the pipeline's end), never a silent out-of-bounds write."""
    cfg = e3data.get("tiny-llama")
    N = 8
    slot_of = {i: i for i in range(N)}
    pos_of = {s: cfg.ctx for s in range(N)}
    W, kv_np, cache, model = _setup(api, cfg, N, slot_of, pos_of, N)
    cache.slot_of_id[3] = 1000
    X = e3data.make_inputs(cfg, range(N), seed=9)
    ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, DEV)
    from paper_conf_sosp_iyergdpgn24_b200._lib import E3Error
    with pytest.raises(E3Error, match="EINVAL"):
        api.Pipeline(model, api.make_plan(cfg, (0, 2, 4), cfg.tau)).run(
            bf16_tensor(X), torch.arange(N, dtype=torch.int64, device=DEV), ex)
    # no other slot was written on token 3's behalf: slot 3 is nobody's
    assert np.array_equal(to64(cache.k[0][3]), kv_np[0][0][3])
