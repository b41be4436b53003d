"""Per-ramp thresholds from a target exit profile — TEST INFRASTRUCTURE ONLY.

The paper fixes a global entropy threshold (0.4 default) on
trained models; with random-init weights the exit histogram it would give is
arbitrary, so per-ramp thresholds tau_r are calibrated so that the fraction
e_r of the inputs exits at ramp r (R5 = SURVEY C5 / §8(d)).  A
single global tau is the special case tau_r = tau.

Algorithm (on a calibration set disjoint from every measured set):
    alive <- all;  S <- 1
    for r = 0 .. R-2:
        k <- round(e_r / S * |alive|)  inputs must pass at ramp r
        tau_r <- midpoint between the k-th and (k+1)-th most confident metric
                 of the alive inputs (max-prob: largest first; entropy:
                 smallest first), rounded to fp32
        alive <- alive minus the inputs that pass;  S <- S - e_r
The last ramp exits everything (R6) and needs no threshold (stored as 0).

Run ``python -m oracle.calibrate <config> [n]`` to (re)write
tests/golden/tau_<config>.json; the file records n, seeds and the oracle mode.

Parity unpinned beyond its own definition: the resulting exit histogram is
checked against e_r within sampling noise (tests/test_oracle_model.py), which
is all the calibration promises.
"""
from __future__ import annotations

import json
import os
import sys
import time

import numpy as np

from .model import brute_force


def calibrate_from_metrics(test, M, profile):
    """Thresholds from the per-ramp metrics M [n, R] of a calibration set."""
    n, R = M.shape
    alive = np.ones(n, dtype=bool)
    surv = 1.0
    tau = []
    for r in range(R - 1):
        m = M[alive, r]
        k = int(round(profile[r] / surv * m.size)) if surv > 0 else 0
        order = np.sort(m)[::-1] if test == "maxprob" else np.sort(m)
        if k <= 0:
            t = order[0] + (1e-3 if test == "maxprob" else -1e-3)
        elif k >= m.size:
            t = order[-1] - (1e-3 if test == "maxprob" else -1e-3)
        else:
            t = 0.5 * (order[k - 1] + order[k])
        t = float(np.float32(t))
        tau.append(t)
        p = (M[:, r] > t) if test == "maxprob" else (M[:, r] < t)
        alive &= ~p
        surv -= profile[r]
    tau.append(0.0)
    return tuple(tau)


def calibrate(cfg, weights, X, mode="bf16"):
    _, _, M = brute_force(cfg, weights, X, tau=[0.0] * cfg.n_ramps, mode=mode)
    return calibrate_from_metrics(cfg.test, M, cfg.exit_profile), M


def calibrate_llama(cfg, n, seed_w=0, seed_x=2, seed_kv=4, mode="bf16"):
    """llama decode: every calibration token through all layers (weights and
    its KV cache generated layer by layer, so fp64 memory stays ~ one layer),
    the shared LM-head ramp evaluated at every ramp layer; then the same
    quantile rule.  Token i sits in its own slot at position cfg.ctx."""
    import e3data
    from .llama import decode_layer, ramp_logits
    from .ramp import metric
    X = e3data.make_inputs(cfg, range(n), seed=seed_x)[:, 0, :].astype(np.float64)
    R = {k: np.asarray(v, dtype=np.float64) for k, v in e3data.make_ramp(cfg, 0, seed_w).items()}
    M = np.zeros((n, cfg.n_ramps))
    pos = np.full(n, cfg.ctx, dtype=np.int64)
    h = X
    for l in range(cfg.layers):
        W = {k: np.asarray(v, dtype=np.float64) for k, v in e3data.make_layer(cfg, l, seed_w).items()}
        kv = e3data.make_kv(cfg, l, range(n), cfg.ctx + 1, seed=seed_kv)
        K, V = kv[0].astype(np.float64), kv[1].astype(np.float64)
        del kv
        h = decode_layer(cfg, h, W, K, V, pos, mode)
        del W, K, V
        if l in cfg.ramp_layers:
            M[:, cfg.ramp_layers.index(l)] = metric(cfg.test, ramp_logits(cfg, h, R, mode))
    return calibrate_from_metrics(cfg.test, M, cfg.exit_profile), M


def golden_path(cfg_name):
    here = os.path.dirname(os.path.abspath(__file__))
    return os.path.join(os.path.dirname(here), "tests", "golden", f"tau_{cfg_name}.json")


def load_tau(cfg):
    with open(golden_path(cfg.name)) as f:
        return tuple(json.load(f)["tau"])


def main(argv):
    import e3data
    cfg = e3data.get(argv[0])
    n = int(argv[1]) if len(argv) > 1 else 256
    seed_w, seed_x = 0, 2                     # calibration inputs: seed 2 (§8(d))
    t0 = time.time()
    if cfg.arch == "llama":
        tau, M = calibrate_llama(cfg, n, seed_w, seed_x)
    else:
        W = e3data.make_weights(cfg, seed_w)
        X = e3data.make_inputs(cfg, range(n), seed=seed_x)
        tau, M = calibrate(cfg, W, X)
    rec = {"config": cfg.name, "tau": list(tau), "n_calib": n, "weight_seed": seed_w,
           "input_seed": seed_x, "mode": "bf16", "exit_profile": list(cfg.exit_profile),
           "script": "python -m oracle.calibrate " + " ".join(argv),
           "seconds": round(time.time() - t0, 1)}
    with open(golden_path(cfg.name), "w") as f:
        json.dump(rec, f, indent=1)
    print(json.dumps(rec))


if __name__ == "__main__":
    main(sys.argv[1:])
