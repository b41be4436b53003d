"""-m gpu: FP32 mode (E3_DTYPE_FP32) end to end from seeded inputs vs the
fp64 oracle at the north_star's fp32 bounds: exit layers and survivor ids
exact wherever every ramp margin exceeds 1e-3, logits and exit metrics within
1e-4 absolute (R14).  Every input of every job is
compared -- no re-seeding of the oracle with GPU rows, no sampling."""
import numpy as np
import pytest
import torch

import e3data
import oracle
from oracle.pipeline_sim import Plan, simulate_pipeline
from tests import parity_util as pu
from tests.gpu_util import DEV, requires_cuda, to64

pytestmark = [pytest.mark.gpu, requires_cuda]

LOGIT_TOL = 1e-4
MARGIN = 1e-3


@pytest.fixture(scope="module")
def api():
    from paper_conf_sosp_iyergdpgn24_b200 import api as A
    return A


def _f32(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(DEV)


def _assert_job(gpu, recs):
    st = pu.compare(gpu, recs, MARGIN)
    assert st["flips"] == 0, st
    assert st["decided"] >= 0.9 * st["n"], st
    assert st["logit_err"]["max"] < LOGIT_TOL, st["logit_err"]
    assert st["metric_err_max"] < LOGIT_TOL
    assert st["label_mismatch"] == 0
    return st


@pytest.mark.parametrize("name,n", [("tiny", 256), ("tiny-vit", 200)])
def test_fp32_pipeline_whole_job(api, name, n):
    cfg = e3data.get(name)
    W = e3data.make_weights(cfg)
    X = e3data.make_inputs(cfg, range(n))
    model = api.DeviceModel(cfg, W, DEV)
    gpu = pu.run_gpu_pipeline(api, cfg, model, X, cfg.tau, dtype="fp32")
    recs = oracle.run(cfg, W, X, mode="fp64")
    _assert_job(gpu, recs)
    # the dispatch sequence is the simulator's for these exit outcomes
    bounds = Plan.per_ramp(cfg.ramp_layers).bounds
    pipe = api.Pipeline(model, api.make_plan(cfg, bounds, cfg.tau, trace=True, dtype="fp32"))
    ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV)
    pipe.run(_f32(X), torch.arange(n, dtype=torch.int64, device=DEV), ex)
    exit_layer = {i: int(v) for i, v in enumerate(ex.exit_layer.cpu().numpy())}
    sim = simulate_pipeline(exit_layer, list(range(n)), Plan(bounds), cfg.batch, lag=1)
    assert [(r.split, r.n_valid, r.ids) for r in sim.runs] == pipe.trace()


def test_fp32_bert_base_12_split_job(api):
    """EE-BERT-base, 12 per-ramp splits, calibrated entropy thresholds,
    B = 64: 128 inputs (two full split-0 batches, then re-batched survivors)
    from seeds, every one compared with the fp64 oracle."""
    cfg = e3data.get("bb")
    tau = e3data.tau_for(cfg)
    W = e3data.make_weights(cfg)
    n = 128
    X = e3data.make_inputs(cfg, range(n))
    model = api.DeviceModel(cfg, W, DEV)
    gpu = pu.run_gpu_pipeline(api, cfg, model, X, tau, dtype="fp32")
    recs = oracle.run(cfg, W, X, tau=tau, mode="fp64")
    st = _assert_job(gpu, recs)
    assert len(set(gpu["exit_layer"].tolist())) >= 8   # exits spread over the ramps


def test_fp32_split_survivor_rows_and_padding(api):
    """One fp32 split run on a padded batch (27 of 32 valid): survivors' hidden
    states vs the fp64 oracle's, in stable order; padding never exits."""
    from oracle.model import run_split
    cfg = e3data.get("tiny")
    W = e3data.make_weights(cfg)
    model = api.DeviceModel(cfg, W, DEV)
    B, nv = cfg.batch, 27
    X = e3data.make_inputs(cfg, range(B))
    xb = X.copy()
    xb[nv:] = 0
    split = api.Split(model, api.split_desc(cfg, 0, 2, cfg.tau, dtype="fp32"))
    x_out = torch.zeros((B, cfg.seq, cfg.hidden), dtype=torch.float32, device=DEV)
    id_out = torch.full((B,), -9, dtype=torch.int64, device=DEV)
    n_surv = torch.zeros(1, dtype=torch.int32, device=DEV)
    ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, DEV)
    split.run(_f32(xb), torch.arange(B, dtype=torch.int64, device=DEV), x_out, id_out, n_surv, ex,
              n_valid=torch.tensor([nv], dtype=torch.int32, device=DEV))
    torch.cuda.synchronize()
    ns = int(n_surv.item())
    assert ns + int(ex.n_exit.item()) == nv
    recs, surv, h, margins = run_split(cfg, W, X[:nv], 0, 2, ids=list(range(nv)), mode="fp64")
    got = id_out[:ns].cpu().tolist()
    assert all(m > MARGIN for m in margins.values())
    assert got == surv
    assert torch.all(id_out[ns:] == -9)
    assert np.max(np.abs(to64(x_out[:ns]) - h)) < 1e-4
    el = ex.exit_layer.cpu().numpy()
    assert (el[nv:] == -1).all()
    for r in recs:
        assert el[r.id] == r.exit_layer
        assert np.max(np.abs(ex.logits[r.id].cpu().numpy() - r.logits)) < LOGIT_TOL


def test_fp32_plan_invariance_bitwise(api):
    """inner = EXACT in fp32: one split holding both ramps == per-ramp splits."""
    cfg = e3data.get("tiny")
    W = e3data.make_weights(cfg)
    model = api.DeviceModel(cfg, W, DEV)
    n = 100
    X = _f32(e3data.make_inputs(cfg, range(n), seed=7))
    ids = torch.arange(n, dtype=torch.int64, device=DEV)
    outs = []
    for bounds in ((0, 2, 4), (0, 4)):
        ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV)
        api.Pipeline(model, api.make_plan(cfg, bounds, cfg.tau, dtype="fp32")).run(X, ids, ex)
        outs.append((ex.exit_layer.cpu(), ex.logits.cpu()))
    assert torch.equal(outs[0][0], outs[1][0]) and torch.equal(outs[0][1], outs[1][1])


def test_fp32_tiny_llama_pipeline(api):
    """LLaMA decode in FP32 (fp32 KV cache): 90 tokens at positions
    ctx - (slot % 5) through the per-ramp plan vs the fp64 oracle."""
    cfg = e3data.get("tiny-llama")
    gpu, recs = pu.llama_job(api, cfg, 90, "fp32", ("fp64",))
    _assert_job(gpu, recs["fp64"])


@pytest.mark.parametrize("name", ["lm", "l8"])
def test_fp32_llama7b_calibrated_32_layer_chain(api, name):
    """Llama-7B shape: 16 tokens through the calibrated 4-split, 32-layer
    chain (ramps after layers 8/16/24/32, V = 32000) in FP32 vs the fp64
    oracle: decisions exact at margin > 1e-3, logits within 1e-4.  l8: the
    Llama-3.1-8B shape (GQA 32 / 8 heads, V 128256, RoPE base 5e5)."""
    cfg = e3data.get(name)
    gpu, recs = pu.llama_job(api, cfg, 16, "fp32", ("fp64",))
    st = pu.compare(gpu, recs["fp64"], MARGIN)
    assert st["flips"] == 0, st
    assert st["logit_err"]["max"] < LOGIT_TOL, st["logit_err"]
    assert st["label_mismatch"] == 0
