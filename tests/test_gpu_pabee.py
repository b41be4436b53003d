"""-m gpu: dependent exits (E3_TEST_PATIENCE; NEXT-4, PAPER.md:2241-2250,
2877-2879; DESIGN R26) vs oracle/pabee.py.  The per-input counter state
travels with the input across splits through e3_exits.state.

FP32 mode against the fp64 oracle at the north_star's fp32 bounds (decisions
exact wherever the oracle's top-2 logit gap exceeds 1e-3 at every ramp the
input reached; logits within 1e-4); bf16 against the bf16-emulating oracle
with decisions exact where that gap exceeds 0.1 (twice the measured bf16
logit error, R13)."""
import numpy as np
import pytest
import torch

import e3data
from oracle import pabee
from oracle.pipeline_sim import Plan
from tests import parity_util as pu
from tests.gpu_util import DEV, requires_cuda

pytestmark = [pytest.mark.gpu, requires_cuda]


@pytest.fixture(scope="module")
def api():
    from paper_conf_sosp_iyergdpgn24_b200 import api as A
    return A


def _job(api, cfg, model, X, dtype, bounds):
    return pu.run_gpu_pipeline(api, cfg, model, X, cfg.tau, bounds=bounds, dtype=dtype)


@pytest.mark.parametrize("t", [1, 2])
def test_pabee_tiny_fp32_every_input(api, t):
    import dataclasses
    cfg = dataclasses.replace(e3data.get("tp"), tau=(float(t),) * 4)
    W = e3data.make_weights(cfg)
    model = api.DeviceModel(cfg, W, DEV)
    X = e3data.make_inputs(cfg, range(256))
    recs = pabee.run(cfg, W, X, t, mode="fp64")
    for bounds in (Plan.per_ramp(cfg.ramp_layers).bounds, (0, 2, 4), (0, 4)):
        gpu = _job(api, cfg, model, X, "fp32", bounds)
        st = pu.compare(gpu, recs, margin=1e-3)
        assert st["flips"] == 0 and st["decided"] >= 0.9 * 256, st
        assert st["logit_err"]["max"] < 1e-4
        assert st["metric_err_max"] == 0.0          # the counter itself
        assert st["label_mismatch"] == 0
    assert len(set(gpu["exit_layer"].tolist())) >= 2


def test_pabee_tiny_bf16_plan_invariance(api):
    """bf16: decisions exact where the top-2 gap > 0.1; the per-ramp plan and
    one split holding all four ramps give bitwise-equal records."""
    cfg = e3data.get("tp")
    W = e3data.make_weights(cfg)
    model = api.DeviceModel(cfg, W, DEV)
    X = e3data.make_inputs(cfg, range(256), seed=3)
    recs = pabee.run(cfg, W, X, 1, mode="bf16")
    a = _job(api, cfg, model, X, "bf16", Plan.per_ramp(cfg.ramp_layers).bounds)
    b = _job(api, cfg, model, X, "bf16", (0, 4))
    assert np.array_equal(a["exit_layer"], b["exit_layer"]) and np.array_equal(a["logits"], b["logits"])
    st = pu.compare(a, recs, margin=0.1)
    assert st["flips"] == 0 and st["decided"] >= 0.7 * 256, st


def test_pabee_bert_base_bf16(api):
    """EE-BERT-base shape with patience 2, 12 per-ramp splits, 128 inputs."""
    cfg = e3data.get("bbp")
    W = e3data.make_weights(cfg)
    model = api.DeviceModel(cfg, W, DEV)
    X = e3data.make_inputs(cfg, range(128))
    gpu = _job(api, cfg, model, X, "bf16", Plan.per_ramp(cfg.ramp_layers).bounds)
    recs = pabee.run(cfg, W, X, 2, mode="bf16")
    st = pu.compare(gpu, recs, margin=0.1)
    assert st["flips"] == 0, st
    assert len(set(gpu["exit_layer"].tolist())) >= 4
