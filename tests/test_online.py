"""Pins of paper_conf_sosp_iyergdpgn24_b200/online.py (NEXT-3; R28):
the ARIMA forecaster, the profile safety checks, the SLO dispatcher and the
re-plan trigger (host logic, CPU)."""
import numpy as np
import pytest

from paper_conf_sosp_iyergdpgn24_b200 import online, planner


def test_ar1_coefficient_recovered():
    rng = np.random.default_rng(0)
    phi, c, n = 0.6, 0.2, 4000
    y = np.zeros(n)
    for t in range(1, n):
        y[t] = c + phi * y[t - 1] + 0.05 * rng.standard_normal()
    coef = online.ar_fit(y, 1)
    assert abs(coef[1] - phi) < 0.03 and abs(coef[0] - c) < 0.02


def test_linear_trend_continued_exactly_with_one_difference():
    y = 0.9 - 0.01 * np.arange(12)
    assert online.arima_forecast(y, p=2, d=1) == pytest.approx(0.9 - 0.01 * 12, abs=1e-12)
    assert online.arima_forecast(np.full(10, 0.37), p=2, d=1) == pytest.approx(0.37, abs=1e-12)
    assert online.arima_forecast([0.5, 0.4], p=2, d=1) == 0.4          # too short: persistence


def test_ar2_on_differences_matches_generating_recursion():
    # differences follow z_t = 0.5 z_{t-1} - 0.25 z_{t-2} exactly: the forecast
    # of the level is last + (0.5 z_last - 0.25 z_prev)
    z = [0.1, -0.05]
    for _ in range(20):
        z.append(0.5 * z[-1] - 0.25 * z[-2])
    y = np.concatenate([[1.0], 1.0 + np.cumsum(z)])
    nxt = y[-1] + 0.5 * z[-1] - 0.25 * z[-2]
    assert online.arima_forecast(y, p=2, d=1) == pytest.approx(nxt, abs=1e-10)


def test_safe_profile_and_estimator():
    assert online.safe_profile([1.2, 0.8, 0.9, -0.1]).tolist() == [1.0, 0.8, 0.8, 0.0]
    est = online.BatchProfileEstimator(3, p=1, d=1)
    # 100 inputs, exits 10 / 20 / 70 at ramps 0 / 1 / 2 -> alive entering ramps: 1, .9, .7
    s = est.observe([10, 20, 70], 100)
    assert np.allclose(s, [1.0, 0.9, 0.7])
    for k in range(6):                                 # a steady drift towards harder inputs
        est.observe([10 - k, 20 - k, 70 + 2 * k], 100)
    f = est.forecast()
    assert (np.diff(f) <= 1e-12).all() and f[0] <= 1.0
    assert f[2] > 0.7                                  # survival at ramp 2 keeps rising


def test_slo_batcher_dispatch_rules():
    b = online.SloBatcher(target=4, slo=0.100, slack=0.2)
    for i in range(3):
        b.add(online.Request(i, arrival=0.010 * i, deadline=0.010 * i + 0.100))
    # 3 < target; oldest deadline 0.100, budget 0.080: with 0.020 of service,
    # waiting is fine until now = 0.060
    assert b.poll(0.050, 0.020) is None
    d = b.poll(0.060, 0.020)
    assert d is not None and d.rids == [0, 1, 2] and not d.dropped
    for i in range(5):
        b.add(online.Request(10 + i, arrival=0.2, deadline=0.3))
    d = b.poll(0.2, 0.02)
    assert d.rids == [10, 11, 12, 13] and len(b.queue) == 1      # a full batch goes at once
    d = b.poll(0.31, 0.02)                                       # past its deadline: dropped
    assert d.rids == [] and d.dropped == [14]
    assert online.goodput([(0, 0.05), (0, 0.2)], [0.1, 0.1], 2.0) == 0.5


def test_replanner_triggers_on_drift_only():
    ramps = tuple(range(12))
    prof = planner.Profile(tuple([120.0] * 12), 20.0, 18.0, 64)
    calls = []

    def plan_fn(surv):
        calls.append([surv(l) for l in range(12)])
        return planner.plan_dp(ramps, surv, prof, 4)[0]

    rp = online.Replanner(ramps, plan_fn, tol=0.05)
    base = online.safe_profile(2.0 ** (-np.arange(12) / 6.0))
    assert rp.update(base) and rp.replans == 1
    assert calls[-1][0] == 1.0 and calls[-1][1] == pytest.approx(base[1])
    assert not rp.update(base + 0.01)                  # within tolerance: keep the plan
    harder = online.safe_profile(base ** 0.3)
    assert rp.update(harder) and rp.replans == 2
    assert rp.plan.world == 4
