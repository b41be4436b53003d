"""Pins for oracle.pipeline_sim: the paper's worked examples and the queue
invariants of the constant-batch pipeline."""
from collections import deque

import numpy as np
import pytest

from oracle.pipeline_sim import Plan, simulate_pipeline


def _check_invariants(res, exit_layer, order, plan, B):
    seen_exit = {}
    for r in res.runs:
        assert 0 < r.n_valid <= B                      # never more than B
        assert len(r.ids) == r.n_valid
        if r.n_valid < B:
            assert r.flush                             # padding only on flush batches
        end = plan.split_end(r.split)
        begin = plan.bounds[r.split]
        for i in r.ids:
            assert exit_layer[i] >= begin              # a row only reaches splits it needs
            if exit_layer[i] <= end:
                assert i not in seen_exit              # every input exits exactly once
                seen_exit[i] = r.split
    assert set(seen_exit) == set(order)
    # conservation: rows into split s+1 == survivors out of split s
    for s in range(plan.n_splits - 1):
        assert res.per_split[s]["rows_out"] == res.per_split[s + 1]["valid"]
    assert res.per_split[plan.n_splits - 1]["rows_out"] == 0


def test_fig5_two_half_batches_make_one_full_batch():
    """Fig. 5 / §3.2: batch 16, 8 survive the cut at layer 6; split 1
    runs twice and the two outputs of 8 form one batch of 16 for split 2."""
    B = 16
    ids = list(range(32))
    exit_layer = {i: (5 if i % 2 == 0 else 11) for i in ids}   # half exit at ramp 6
    plan = Plan.cuts(12, [5])
    for lag in (0, 1):
        res = simulate_pipeline(exit_layer, ids, plan, B, lag=lag)
        assert [r.split for r in res.runs] == [0, 0, 1]
        assert all(r.n_valid == B and not r.flush for r in res.runs)
        assert res.runs[2].ids == tuple(i for i in ids if i % 2 == 1)   # FIFO, stable
        _check_invariants(res, exit_layer, ids, plan, B)


def test_sec583_prediction_error_leftovers_wait_in_queue():
    """§5.8.3: 16 -> 8 expected, 12 with a 50% error.  Correctness
    is unaffected: survivors queue up and split 2 always runs exactly 16."""
    B = 16
    n_batches = 8
    ids = list(range(B * n_batches))
    exit_layer = {i: (5 if i % 16 < 4 else 11) for i in ids}   # 12 of 16 survive
    plan = Plan.cuts(12, [5])
    res = simulate_pipeline(exit_layer, ids, plan, B, lag=0)
    s2 = [r for r in res.runs if r.split == 1]
    full = [r for r in s2 if not r.flush]
    assert len(full) == (12 * n_batches) // 16 and all(r.n_valid == 16 for r in full)
    assert sum(r.n_valid for r in s2) == 12 * n_batches
    _check_invariants(res, exit_layer, ids, plan, B)


def test_queue_is_fifo_deque():
    """Split-2 input order equals a collections.deque replay of split-1 outputs."""
    rng = np.random.default_rng(0)
    B = 8
    ids = list(range(200))
    exit_layer = {i: int(rng.choice([0, 1, 2])) for i in ids}
    plan = Plan.per_ramp((0, 1, 2))
    res = simulate_pipeline(exit_layer, ids, plan, B, lag=0)
    q = [deque(), deque()]
    for r in res.runs:
        if r.split > 0:
            expect = [q[r.split - 1].popleft() for _ in range(r.n_valid)]
            assert list(r.ids) == expect
        if r.split < 2:
            q[r.split].extend(i for i in r.ids if exit_layer[i] > r.split)


@pytest.mark.parametrize("lag", [0, 1, 2])
@pytest.mark.parametrize("seed", range(5))
def test_random_invariants(lag, seed):
    rng = np.random.default_rng(seed)
    L = 12
    ramps = tuple(range(L))
    B = int(rng.choice([4, 16, 64]))
    n = int(rng.integers(1, 700))
    ids = list(rng.permutation(10 * n)[:n])
    S = 2.0 ** (-np.arange(1, L + 1) / 6)
    p = -np.diff(np.concatenate([[1.0], S[:-1], [0.0]]))
    exit_layer = {int(i): int(rng.choice(L, p=p / p.sum())) for i in ids}
    for plan in (Plan.per_ramp(ramps), Plan.cuts(L, [5]), Plan.cuts(L, [1, 3, 6])):
        res = simulate_pipeline(exit_layer, [int(i) for i in ids], plan, B, lag=lag)
        _check_invariants(res, exit_layer, ids, plan, B)


def test_deepest_ready_split_runs_first():
    B = 4
    ids = list(range(16))
    exit_layer = {i: 2 for i in ids}                    # nobody exits early
    plan = Plan.per_ramp((0, 1, 2))
    res = simulate_pipeline(exit_layer, ids, plan, B, lag=0)
    assert [r.split for r in res.runs] == [0, 1, 2] * 4
    res1 = simulate_pipeline(exit_layer, ids, plan, B, lag=1)
    assert sorted(r.split for r in res1.runs) == sorted([0, 1, 2] * 4)
    _check_invariants(res1, exit_layer, ids, plan, B)


def test_empty_and_tiny_inputs():
    plan = Plan.per_ramp((0, 1))
    assert simulate_pipeline({}, [], plan, 8).runs == []
    res = simulate_pipeline({5: 1}, [5], plan, 8)
    assert [(r.split, r.n_valid, r.flush) for r in res.runs] == [(0, 1, True), (1, 1, True)]
