"""-m gpu: the exit-wrapper's ramp control (NEXT-4; PAPER.md:985-1017,
2648-2654): every ramp's metric recorded on the GPU (e3_exits.ramp_metric)
in a profiling run whose thresholds never pass, checked against the oracle's
per-ramp metrics; the planner's chosen ramp set run with inner ramps
DISABLED exits every input where the recorded metrics predict."""
import dataclasses
import os

import numpy as np
import pytest
import torch

import e3data
from oracle import model as omodel
from tests.gpu_util import DEV, bf16_tensor, requires_cuda

pytestmark = [pytest.mark.gpu, requires_cuda]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def api():
    from paper_conf_sosp_iyergdpgn24_b200 import api as A
    return A


def _profile(api, cfg, model, X, tau_never):
    n = X.shape[0]
    ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV, ramp_metrics=True)
    bounds = tuple(range(cfg.layers + 1))
    api.Pipeline(model, api.make_plan(cfg, bounds, tau_never)).run(
        bf16_tensor(X), torch.arange(n, dtype=torch.int64, device=DEV), ex)
    torch.cuda.synchronize()
    return ex.ramp_metric.cpu().numpy().astype(np.float64)


def test_ramp_metrics_and_chosen_plan(api):
    from paper_conf_sosp_iyergdpgn24_b200 import planner as pl
    cfg = e3data.get("bb")
    tau = e3data.tau_for(cfg)
    W = e3data.make_weights(cfg)
    model = api.DeviceModel(cfg, W, DEV)
    never = (0.0,) * cfg.n_ramps                          # entropy < 0 never holds
    n = 256
    X = e3data.make_inputs(cfg, range(n))
    M = _profile(api, cfg, model, X, never)
    assert not np.isnan(M).any()                          # every row evaluated at every ramp
    # against the oracle's metrics at every ramp (bf16-emulate, first 24 inputs)
    _, Z, Mo = omodel.brute_force(cfg, W, X[:24], tau=never, mode="bf16")
    assert np.max(np.abs(M[:24] - Mo)) < 0.05
    prof = pl.Profile.load(os.path.join(ROOT, "profiles", "r02_planner_profile_bb.json"))
    en, cost, _ = pl.choose_ramps(M, tau, cfg.test, cfg.ramp_layers, prof)
    assert en[-1] == cfg.n_ramps - 1
    # the chosen plan: one split per enabled ramp, the other ramps disabled inside
    bounds = (0,) + tuple(cfg.ramp_layers[r] + 1 for r in en)
    ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV)
    api.Pipeline(model, api.make_plan(cfg, bounds, tau, inner="disabled")).run(
        bf16_tensor(X), torch.arange(n, dtype=torch.int64, device=DEV), ex)
    got = ex.exit_layer.cpu().numpy()
    pred = np.asarray(cfg.ramp_layers)[pl.exits_with(M, tau, cfg.test, en, cfg.n_ramps - 1)]
    clear = np.all(np.abs(M - np.asarray(tau, dtype=np.float32)[None, :]) > 1e-3, axis=1)
    assert clear.mean() > 0.8
    assert np.array_equal(got[clear], pred[clear])
