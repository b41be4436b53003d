"""Pins of oracle/pabee.py (counter-based dependent exits, NEXT-4; DESIGN R26)."""
import dataclasses

import numpy as np
import pytest

import e3data
from oracle import model, pabee


def test_hand_sequence():
    # predictions at the evaluated ramps: 1 1 0 0 0 1
    #   counters:                       0 1 0 1 2 0
    seq = [1, 1, 0, 0, 0, 1]
    assert pabee.exit_ramp_of_labels(seq, 2) == 4
    assert pabee.exit_ramp_of_labels(seq, 1) == 1
    assert pabee.exit_ramp_of_labels(seq, 0) == 0
    assert pabee.exit_ramp_of_labels(seq, 3) == 5          # never reached: the last ramp
    assert pabee.exit_ramp_of_labels([2, 2, 2], 2) == 2


@pytest.fixture(scope="module")
def tiny4():
    # 4 layers with a ramp after every layer: room for counters to build up
    cfg = dataclasses.replace(e3data.get("tiny"), ramp_layers=(0, 1, 2, 3), tau=(0.9,) * 4)
    W = e3data.make_weights(cfg)
    X = e3data.make_inputs(cfg, range(48), seed=17)
    return cfg, W, X


@pytest.mark.parametrize("t", [0, 1, 2, 3])
def test_equals_brute_force(tiny4, t):
    cfg, W, X = tiny4
    recs = pabee.run(cfg, W, X, t)
    el, Z = pabee.brute_force(cfg, W, X, t)
    assert [r.exit_layer for r in recs] == el.tolist()
    for i, r in enumerate(recs):
        ri = cfg.ramp_layers.index(r.exit_layer)
        assert np.allclose(r.logits, Z[i, ri], atol=1e-12)
        assert r.label == int(np.argmax(Z[i, ri]))


def test_extremes_and_monotonicity(tiny4):
    cfg, W, X = tiny4
    assert all(r.exit_layer == cfg.ramp_layers[0] for r in pabee.run(cfg, W, X, 0))
    assert all(r.exit_layer == cfg.ramp_layers[-1] for r in pabee.run(cfg, W, X, cfg.n_ramps))
    prev = None
    for t in range(cfg.n_ramps + 1):
        el = np.array([r.exit_layer for r in pabee.run(cfg, W, X, t)])
        if prev is not None:
            assert (el >= prev).all()
        prev = el


def test_logits_are_the_ramp_logits_of_the_plain_model(tiny4):
    """At t >= R every input runs to the last ramp: the logits and labels are
    the plain early-exit model's with thresholds that never pass."""
    cfg, W, X = tiny4
    a = pabee.run(cfg, W, X, cfg.n_ramps)
    b = model.run(cfg, W, X, tau=(1.5,) * cfg.n_ramps)
    for ra, rb in zip(a, b):
        assert ra.exit_layer == rb.exit_layer and ra.label == rb.label
        assert np.array_equal(ra.logits, rb.logits)
