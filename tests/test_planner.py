"""NEXT-1 planner (paper §3.2): the dynamic program over
(cut, GPUs, stages) must find the same optimum as enumerating every cut set
and replica vector (the oracle), on random measured-profile instances, with
and without a per-GPU weight-memory cap."""
import math

import numpy as np
import pytest

from paper_conf_sosp_iyergdpgn24_b200.planner import Profile, brute_force_plan, plan_dp, stage_cost


def _instance(rng, L):
    n_ramps = int(rng.integers(2, L + 1))
    ramps = sorted(rng.choice(np.arange(L - 1), size=n_ramps - 1, replace=False).tolist()) + [L - 1]
    exits = rng.dirichlet(np.ones(len(ramps)))
    surv = lambda l: 1.0 - sum(e for r, e in zip(ramps, exits) if r < l)
    prof = Profile(tuple(float(v) for v in rng.uniform(50, 150, L)), float(rng.uniform(5, 20)),
                   float(rng.uniform(0, 30)), 64)
    return ramps, surv, prof


@pytest.mark.parametrize("seed", range(24))
def test_dp_equals_brute_force(seed):
    rng = np.random.default_rng(seed)
    L = int(rng.integers(3, 9))
    ramps, surv, prof = _instance(rng, L)
    G = int(rng.integers(1, 6))
    lay_dp, v_dp = plan_dp(ramps, surv, prof, G)
    lay_bf, v_bf = brute_force_plan(ramps, surv, prof, G)
    assert v_dp == pytest.approx(v_bf, rel=1e-12)
    assert lay_dp.world == G and lay_dp.bounds[0] == 0 and lay_dp.bounds[-1] == L
    # the DP's layout achieves the value it reports
    w = [stage_cost(lay_dp.bounds[s], lay_dp.bounds[s + 1], ramps, surv, prof, L) for s in range(lay_dp.n_stages)]
    assert max(w[s] / lay_dp.replicas[s] for s in range(lay_dp.n_stages)) == pytest.approx(v_dp, rel=1e-12)
    assert lay_dp.n_stages == lay_bf.n_stages          # ties -> fewest stages on both sides


@pytest.mark.parametrize("seed", range(12))
def test_dp_equals_brute_force_with_memory_cap(seed):
    rng = np.random.default_rng(100 + seed)
    L = int(rng.integers(4, 9))
    ramps, surv, prof = _instance(rng, L)
    mem = rng.uniform(1, 2, L).tolist()
    G = int(rng.integers(2, 6))
    cap = float(np.max([sum(mem[a:b]) for a, b in zip([0] + [r + 1 for r in ramps[:-1]], [r + 1 for r in ramps])]))
    cap = max(cap, sum(mem) / 2.2)                      # forces >= 2 stages on most instances
    try:
        lay_bf, v_bf = brute_force_plan(ramps, surv, prof, G, mem_layer=mem, mem_cap=cap)
    except ValueError:
        with pytest.raises(ValueError):
            plan_dp(ramps, surv, prof, G, mem_layer=mem, mem_cap=cap)
        return
    lay_dp, v_dp = plan_dp(ramps, surv, prof, G, mem_layer=mem, mem_cap=cap)
    assert v_dp == pytest.approx(v_bf, rel=1e-12)
    assert all(sum(mem[lay_dp.bounds[s]:lay_dp.bounds[s + 1]]) <= cap for s in range(lay_dp.n_stages))


def test_free_transfers_make_replication_optimal():
    """With t_tx = 0 and no memory limit, max_g W_g / r_g >= sum W_g / G = W(0, L) / G,
    which one stage on all G GPUs attains: the DP returns pure replication."""
    rng = np.random.default_rng(7)
    ramps, surv, prof = _instance(rng, 12)
    prof = Profile(prof.t_layer, prof.t_ramp, 0.0, prof.batch)
    for G in (1, 2, 4, 8):
        lay, v = plan_dp(ramps, surv, prof, G)
        assert lay.bounds == (0, 12) and lay.replicas == (G,)
        assert v == pytest.approx(stage_cost(0, 12, ramps, surv, prof, 12) / G)


def test_more_gpus_never_slower():
    rng = np.random.default_rng(3)
    ramps, surv, prof = _instance(rng, 8)
    mem = [1.0] * 8
    vals = [plan_dp(ramps, surv, prof, G, mem_layer=mem, mem_cap=4.0)[1] for G in range(2, 9)]
    assert all(b <= a + 1e-12 for a, b in zip(vals, vals[1:]))
    assert math.isfinite(vals[0])


def test_bert_base_stage_cuts_match_the_survival_balance():
    """SURVEY.md §8(e) balances EE-BERT-base's per-layer survival weights
    S(l) = 2^(-l/6) by hand: 2 GPUs in 2 stages -> cut after layer 4 (3.392 vs
    3.483); 4 GPUs in 4 stages -> {L1-2, L3-4, L5-7, L8-12}.  With equal layer
    times and free ramps / transfers the DP must find the same cuts."""
    ramps = list(range(12))
    surv = lambda l: 2.0 ** (-l / 6.0)
    prof = Profile((1.0,) * 12, 0.0, 0.0, 1)
    lay, _ = plan_dp(ramps, surv, prof, 2, n_stages=2)
    assert lay.bounds == (0, 4, 12) and lay.replicas == (1, 1)
    lay, _ = plan_dp(ramps, surv, prof, 4, n_stages=4)
    assert lay.bounds == (0, 2, 4, 7, 12) and lay.replicas == (1, 1, 1, 1)


def test_choose_ramps_extremes_and_hand_case():
    import numpy as np
    from paper_conf_sosp_iyergdpgn24_b200 import planner as pl
    # 4 ramps after layers 0..3, max-prob metrics of 4 inputs, tau 0.5
    M = np.array([[0.9, 0.1, 0.1, 0.1],      # exits at ramp 0 if enabled
                  [0.1, 0.9, 0.1, 0.1],      # ramp 1
                  [0.1, 0.1, 0.9, 0.1],      # ramp 2
                  [0.1, 0.1, 0.1, 0.1]])     # last
    tau = [0.5] * 4
    rl = (0, 1, 2, 3)
    assert pl.exits_with(M, tau, "maxprob", (0, 1, 2, 3), 3).tolist() == [0, 1, 2, 3]
    assert pl.exits_with(M, tau, "maxprob", (1, 3), 3).tolist() == [3, 1, 3, 3]
    free = pl.Profile((1.0,) * 4, 0.0, 0.0, 1)
    en, cost, _ = pl.choose_ramps(M, tau, "maxprob", rl, free)
    assert en == (0, 1, 2, 3)                              # free ramps: keep every one
    # hand cost with t_layer 1, t_ramp 10: all ramps -> layers 1 + .75 + .5 + .25 = 2.5, ramps 10 (1 + .75
    # + .5 + .25) = 25 -> 27.5; only the last -> layers 4, its ramp sees every input: 10 -> 14
    dear = pl.Profile((1.0,) * 4, 10.0, 0.0, 1)
    assert pl.ramp_plan_cost(pl.exits_with(M, tau, "maxprob", (0, 1, 2, 3), 3), rl, (0, 1, 2, 3), dear) == 27.5
    en, cost, _ = pl.choose_ramps(M, tau, "maxprob", rl, dear)
    assert en == (3,) and cost == 14.0
    # moderate ramp cost: a ramp pays when it removes enough downstream work
    mid = pl.Profile((1.0,) * 4, 0.2, 0.0, 1)
    en, cost, _ = pl.choose_ramps(M, tau, "maxprob", rl, mid)
    brute = min(pl.ramp_plan_cost(pl.exits_with(M, tau, "maxprob", e, 3), rl, e, mid)
                for e in [tuple(r for r in range(3) if m >> r & 1) + (3,) for m in range(8)])
    assert cost == pytest.approx(brute)
