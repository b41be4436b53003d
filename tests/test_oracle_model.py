"""Pins for oracle.model: brute force, extremes, torch-composed plain encoder,
monotonicity, exactly-once exits, batch invariance and the Fig. 1 example."""
from dataclasses import replace

import numpy as np
import pytest
import torch

import e3data
import oracle
from oracle import calibrate
from oracle.model import brute_force, run

TINY = e3data.get("tiny")


@pytest.fixture(scope="module")
def tiny():
    W = e3data.make_weights(TINY)
    X = e3data.make_inputs(TINY, range(48))
    return W, X


@pytest.mark.parametrize("mode", ["fp64", "bf16"])
def test_brute_force_equals_early_stopping(tiny, mode):
    W, X = tiny
    recs = run(TINY, W, X, mode=mode)
    el, Z, M = brute_force(TINY, W, X, mode=mode)
    assert [r.exit_layer for r in recs] == list(el)
    for i, r in enumerate(recs):
        k = TINY.ramp_layers.index(r.exit_layer)
        assert np.array_equal(r.logits, Z[i, k])
        assert r.metric == M[i, k]
        assert r.label == int(np.argmax(Z[i, k]))


def test_exactly_once_and_ids(tiny):
    W, X = tiny
    ids = [1000 + 7 * i for i in range(len(X))]
    recs = run(TINY, W, X, ids=ids)
    assert [r.id for r in recs] == ids
    assert len({r.id for r in recs}) == len(ids)
    assert all(r.exit_layer in TINY.ramp_layers for r in recs)


def test_batch_invariance(tiny):
    W, X = tiny
    full = run(TINY, W, X, mode="bf16")
    perm = np.random.default_rng(0).permutation(len(X))[:17]
    sub = run(TINY, W, X[perm], ids=list(perm), mode="bf16")
    for r in sub:
        f = full[r.id]
        assert (r.exit_layer, r.label) == (f.exit_layer, f.label)
        assert np.max(np.abs(r.logits - f.logits)) < 1e-12   # BLAS blocking only


def _torch_plain_logits(cfg, W, X):
    """Plain encoder (torch.nn.TransformerEncoderLayer chain, float64) + last ramp."""
    from tests.test_oracle_encoder import _torch_layer
    h = torch.tensor(X.astype(np.float64))
    with torch.no_grad():
        for l in range(cfg.layers):
            Wl = {k: v.astype(np.float64) for k, v in W["layers"][l].items()}
            h = _torch_layer(Wl, cfg.hidden, cfg.heads, cfg.ffn, cfg.norm_eps, False)(h)
        R = {k: torch.tensor(v.astype(np.float64)) for k, v in W["ramps"][-1].items()}
        p = torch.tanh(h[:, 0] @ R["w_p"].T + R["b_p"])
        return (p @ R["w_c"].T + R["b_c"]).numpy()


def test_no_early_exit_equals_plain_encoder(tiny):
    W, X = tiny
    recs = run(TINY, W, X[:8], tau=(1.0, 1.0))
    assert all(r.exit_layer == TINY.layers - 1 for r in recs)
    ref = _torch_plain_logits(TINY, W, X[:8])
    got = np.stack([r.logits for r in recs])
    assert np.max(np.abs(got - ref)) < 1e-10


def test_everything_exits_at_first_ramp(tiny):
    W, X = tiny
    recs = run(TINY, W, X, tau=(0.49, 0.49))          # max-prob >= 1/C = 0.5 > tau
    assert all(r.exit_layer == TINY.ramp_layers[0] for r in recs)


def test_raising_maxprob_threshold_never_exits_earlier(tiny):
    W, X = tiny
    prev = None
    for t in (0.6, 0.8, 0.9, 0.97, 0.999):
        el = np.array([r.exit_layer for r in run(TINY, W, X, tau=(t, t))])
        if prev is not None:
            assert np.all(el >= prev)
        prev = el


def test_entropy_test_extremes():
    cfg = replace(TINY, test="entropy")
    W = e3data.make_weights(cfg)
    X = e3data.make_inputs(cfg, range(8))
    assert all(r.exit_layer == 3 for r in run(cfg, W, X, tau=(0.0, 0.0)))
    assert all(r.exit_layer == 1 for r in run(cfg, W, X, tau=(0.7, 0.7)))  # ln 2 < 0.7


def test_inner_disabled_only_counts_enabled_ramps(tiny):
    W, X = tiny
    recs = run(TINY, W, X, enabled=[])      # only the model's last ramp
    assert all(r.exit_layer == 3 for r in recs)


def test_fig1_worked_example_counts():
    """Fig. 1: batch 16; 1 exits at Ramp1 -> 15 continue; 2 exit at
    Ramp2 -> 13 continue; the remaining samples exit at Ramp12."""
    cfg = e3data.configs.ModelConfig(
        name="fig1", arch="bert", layers=12, hidden=64, heads=2, ffn=128, seq=8, classes=2,
        norm_eps=1e-12, ramp_layers=tuple(range(12)), batch=16, test="maxprob")
    W = e3data.make_weights(cfg, seed=5)
    X = e3data.make_inputs(cfg, range(16), seed=6)
    _, _, M = brute_force(cfg, W, X, tau=[2.0] * 12)
    s0 = np.sort(M[:, 0])[::-1]
    t0 = 0.5 * (s0[0] + s0[1])                          # exactly one passes ramp 1
    alive = M[:, 0] <= t0
    s1 = np.sort(M[alive, 1])[::-1]
    t1 = 0.5 * (s1[1] + s1[2])                          # exactly two of the 15 pass ramp 2
    tau = [t0, t1] + [1.0] * 10
    recs = run(cfg, W, X, tau=tau)
    counts = [sum(r.exit_layer == l for r in recs) for l in range(12)]
    assert counts[0] == 1 and counts[1] == 2 and counts[11] == 13 and sum(counts) == 16


def test_bf16_storage_gap_to_fp64_is_bounded(tiny):
    """Documents why bf16 logits are judged against the bf16-emulate oracle
    (R13): bf16 storage alone moves logits by O(1e-2)."""
    W, X = tiny
    a = run(TINY, W, X, mode="fp64")
    b = run(TINY, W, X, mode="bf16")
    gaps = [np.abs(x.logits - y.logits).max() for x, y in zip(a, b) if x.exit_layer == y.exit_layer]
    assert 1e-3 < np.median(gaps) < 0.05 and max(gaps) < 0.25


def test_calibration_hits_exit_profile():
    cfg = replace(TINY, name="tiny-cal", ramp_layers=(0, 1, 2, 3), test="entropy",
                  exit_profile=(0.3, 0.2, 0.1, 0.4), tau=None)
    W = e3data.make_weights(cfg)
    Xc = e3data.make_inputs(cfg, range(400), seed=2)
    tau, _ = calibrate.calibrate(cfg, W, Xc)
    Xm = e3data.make_inputs(cfg, range(400), seed=1)
    recs = run(cfg, W, Xm, tau=tau, mode="bf16")
    frac = np.array([sum(r.ramp == k for r in recs) for k in range(4)]) / 400.0
    assert np.all(np.abs(frac - np.array(cfg.exit_profile)) < 0.08), frac


@pytest.mark.parametrize("bounds", [(0, 2, 4), (0, 4)])
def test_run_split_composes_to_run(tiny, bounds):
    """Chaining run_split over a plan (inner EXACT) reproduces run (plan invariance)."""
    from oracle.model import run_split
    W, X = tiny
    full = {r.id: r for r in run(TINY, W, X, mode="bf16")}
    ids = list(range(len(X)))
    h = X.astype(np.float64)
    got = {}
    for b, e in zip(bounds[:-1], bounds[1:]):
        recs, ids, h, _ = run_split(TINY, W, h, b, e, ids=ids, mode="bf16")
        got.update({r.id: r for r in recs})
    assert not ids and set(got) == set(full)
    for i, r in got.items():
        assert (r.exit_layer, r.label) == (full[i].exit_layer, full[i].label)
        assert np.max(np.abs(r.logits - full[i].logits)) < 1e-12
