"""Per-input early-exit forward — TEST INFRASTRUCTURE ONLY.

The plain definition of the result: E3 changes where and with
whom an input is computed, not what is computed for it.  Encoder rows are
independent (attention is within one sequence, LN per token) and the exit
test is per input, so every input's result is the EE-DNN run
on that input alone:

    for each layer l in order:  h <- layer_l(h)
        if a ramp r follows l and is enabled:
            z <- ramp_r(h);  m <- metric(z)
            if passes(m, tau_r) or r is the model's last ramp: exit (l, z)

"Remaining samples exit" at the last ramp (Fig. 1; R6).  Inputs
are processed together only as a NumPy vectorisation over a leading axis;
no arithmetic mixes inputs.

Pins (tests/test_oracle_model.py): brute force (run every layer and ramp,
then scan for the first pass) equals the early-stopping run exactly;
tau_maxprob >= 1 (entropy tau <= 0) sends every input to the last ramp with
logits equal to the plain encoder + final ramp, itself pinned to
torch.nn.TransformerEncoderLayer; tau_maxprob < 1/C exits everything at the
first ramp; raising tau_maxprob never makes an exit earlier; every input
exits exactly once.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Optional, Sequence

import numpy as np

from .encoder import encoder_layer
from .ramp import metric, passes, ramp_logits


@dataclass
class ExitRecord:
    id: int
    exit_layer: int        # 0-based layer index the exiting ramp follows
    ramp: int              # ramp index
    label: int             # argmax z, lowest index on ties (R12)
    metric: float          # max-prob or entropy at the exit ramp
    logits: np.ndarray     # float64 [C]
    margin: float          # min |metric - tau| over tau-decided ramps reached


def _as64(W):
    return {k: np.asarray(v, dtype=np.float64) for k, v in W.items()}


def run(cfg, weights, X, ids: Optional[Sequence[int]] = None, tau=None,
        mode: str = "fp64", enabled: Optional[Sequence[int]] = None) -> List[ExitRecord]:
    """Early-exit forward of every input in X ([n, S, H]); records in input order.

    tau: per-ramp thresholds (default cfg.tau).  enabled: ramp indices whose
    test is evaluated (default all = inner EXACT; the model's last ramp always
    exits).  mode: "fp64" or "bf16" (emulated storage rounding).
    """
    X = np.asarray(X, dtype=np.float64)
    n = X.shape[0]
    ids = list(range(n)) if ids is None else [int(i) for i in ids]
    tau = cfg.tau if tau is None else tau
    last = cfg.n_ramps - 1
    en = set(range(cfg.n_ramps)) if enabled is None else set(enabled) | {last}
    ramp_at = {l: r for r, l in enumerate(cfg.ramp_layers)}
    layers = [_as64(w) for w in weights["layers"]]
    ramps = [_as64(w) for w in weights["ramps"]]

    out: List[Optional[ExitRecord]] = [None] * n
    alive = np.arange(n)
    margin = np.full(n, np.inf)
    h = X
    for l in range(cfg.layers):
        if alive.size == 0:
            break
        h = encoder_layer(cfg, h, layers[l], mode)
        r = ramp_at.get(l)
        if r is None or r not in en:
            continue
        z = ramp_logits(cfg, h, ramps[r])
        m = metric(cfg.test, z)
        if r == last:
            ok = np.ones(alive.size, dtype=bool)
        else:
            ok = passes(cfg.test, m, tau[r])
            margin[alive] = np.minimum(margin[alive],
                                       np.abs(m - np.float64(np.float32(tau[r]))))
        for j in np.nonzero(ok)[0]:
            i = alive[j]
            out[i] = ExitRecord(ids[i], l, r, int(np.argmax(z[j])), float(m[j]),
                                z[j].copy(), float(margin[i]))
        keep = ~ok
        alive, h = alive[keep], h[keep]
    assert all(o is not None for o in out), "an input did not exit"
    return out  # type: ignore[return-value]


def run_split(cfg, weights, X, begin: int, end: int, ids: Optional[Sequence[int]] = None, tau=None,
              mode: str = "fp64", inner: str = "exact"):
    """One split (layers [begin, end), ending in a ramp) on the rows X.

    The same per-input definition as ``run`` restricted to the split: apply
    layers begin..end-1; at each ramp inside the split (all of them for inner
    EXACT, only the split's last for DISABLED) evaluate the exit test; the
    model's last ramp exits every row.  Returns (records of the rows that
    exit inside the split, in input order; ids of the survivors in input
    order; survivors' hidden states [k, S, H]; {id: min margin over the
    split's tau-decided ramps}).
    """
    X = np.asarray(X, dtype=np.float64)
    n = X.shape[0]
    ids = list(range(n)) if ids is None else [int(i) for i in ids]
    tau = cfg.tau if tau is None else tau
    last = cfg.n_ramps - 1
    ramps_in = [r for r, l in enumerate(cfg.ramp_layers) if begin <= l < end]
    assert ramps_in and cfg.ramp_layers[ramps_in[-1]] == end - 1, "a split must end in a ramp"
    en = set(ramps_in) if inner == "exact" else {ramps_in[-1]}
    ramp_at = {cfg.ramp_layers[r]: r for r in ramps_in}
    exited = {}
    alive = np.arange(n)
    margin = np.full(n, np.inf)
    h = X
    for l in range(begin, end):
        h = encoder_layer(cfg, h, _as64(weights["layers"][l]), mode)
        r = ramp_at.get(l)
        if r is None or r not in en or alive.size == 0:
            continue
        z = ramp_logits(cfg, h, _as64(weights["ramps"][r]))
        m = metric(cfg.test, z)
        if r == last:
            ok = np.ones(alive.size, dtype=bool)
        else:
            ok = passes(cfg.test, m, tau[r])
            margin[alive] = np.minimum(margin[alive], np.abs(m - np.float64(np.float32(tau[r]))))
        for j in np.nonzero(ok)[0]:
            i = alive[j]
            exited[i] = ExitRecord(ids[i], l, r, int(np.argmax(z[j])), float(m[j]), z[j].copy(),
                                   float(margin[i]))
        alive, h = alive[~ok], h[~ok]
    recs = [exited[i] for i in sorted(exited)]
    return recs, [ids[i] for i in alive], h, {ids[i]: float(margin[i]) for i in range(n)}


def run_input(cfg, weights, x, id: int = 0, tau=None, mode="fp64", enabled=None) -> ExitRecord:
    """The EE-DNN run on one input alone."""
    return run(cfg, weights, np.asarray(x)[None], [id], tau, mode, enabled)[0]


def brute_force(cfg, weights, X, tau=None, mode="fp64"):
    """Every layer and every ramp for every input, then the first passing ramp.

    Returns (exit_layer[n], logits_all[n, R, C], metric_all[n, R])."""
    X = np.asarray(X, dtype=np.float64)
    tau = cfg.tau if tau is None else tau
    ramp_at = {l: r for r, l in enumerate(cfg.ramp_layers)}
    layers = [_as64(w) for w in weights["layers"]]
    ramps = [_as64(w) for w in weights["ramps"]]
    n, R = X.shape[0], cfg.n_ramps
    Z = np.zeros((n, R, cfg.classes))
    M = np.zeros((n, R))
    h = X
    for l in range(cfg.layers):
        h = encoder_layer(cfg, h, layers[l], mode)
        if l in ramp_at:
            r = ramp_at[l]
            Z[:, r] = ramp_logits(cfg, h, ramps[r])
            M[:, r] = metric(cfg.test, Z[:, r])
    exit_layer = np.empty(n, dtype=np.int64)
    for i in range(n):
        first = R - 1
        for r in range(R - 1):
            if passes(cfg.test, M[i, r], tau[r]):
                first = r
                break
        exit_layer[i] = cfg.ramp_layers[first]
    return exit_layer, Z, M
