"""Profile-driven split/replica planner (PAPER.md
§3.2 "Split Placement", 750-930, and the pipelined variant 907-930).

E3's optimizer chooses where to cut the EE-DNN into splits, how many GPUs run
each split, and relies on constant-batch execution for the cost of a split.
Our reading of its dynamic program (R20; SURVEY C20 notes the
garbled base case) for one GPU type:

* A STAGE is a contiguous layer range [i, j) cut at ramps, run on r GPUs (its
  replicas).  Inside a GPU the stage still runs one split per ramp with
  re-batching (the executor's per-ramp plan), so every layer runs at the
  constant batch B.
* Measured profile (on-device, ``scripts/profile_layers.py``): t_layer[l], the
  time of layer l on a full batch of B; t_ramp, one ramp + compaction +
  re-batch per split run; t_tx, the transfer of one batch of survivors to the
  next stage (0 on the last stage).
* Expected GPU time per input of stage [i, j) (a split's
  time is the sum of its layers' times at its batch size; the fraction S(l)
  of inputs alive at layer l sets how many batches reach it):

      W(i, j) = ( sum_{l in [i, j)} S(l) t_layer[l]
                + sum_{ramps r in [i, j)} S(r) t_ramp
                + S(j) t_tx [j < L] ) / B

* Pipelined throughput is set by the slowest stage:
  minimise max_g W(stage g) / r_g subject to sum_g r_g = G.

DP over (cut position, GPUs used):
    A(0, 0) = 0,   A(j, g) = min_{i < j cut, 1 <= r <= g} max(A(i, g - r), W(i, j) / r)
with A(j, g) = inf for g = 0 < j.  The answer is A(L, G); ties prefer fewer
stages.  ``brute_force_plan`` enumerates every cut set and replica vector as
the oracle the DP is tested against (tests/test_planner.py).
"""
from __future__ import annotations

import itertools
import json
import math
from dataclasses import dataclass
from typing import Callable, Dict, Optional, Sequence, Tuple

from .parallel import StageLayout


@dataclass(frozen=True)
class Profile:
    """Per-batch times in microseconds at the constant batch B."""
    t_layer: Tuple[float, ...]      # [L]
    t_ramp: float                   # ramp + compaction + re-batch, per split run
    t_tx: float                     # one batch of survivors to the next stage
    batch: int

    @staticmethod
    def load(path: str) -> "Profile":
        d = json.load(open(path))
        return Profile(tuple(d["t_layer_us"]), float(d["t_ramp_us"]), float(d.get("t_tx_us", 0.0)), int(d["batch"]))


def stage_cost(i: int, j: int, ramp_layers: Sequence[int], survival: Callable[[int], float], prof: Profile,
               L: int) -> float:
    """W(i, j): expected GPU microseconds per input entering the model."""
    w = sum(survival(l) * prof.t_layer[l] for l in range(i, j))
    w += sum(survival(r) * prof.t_ramp for r in ramp_layers if i <= r < j)
    if j < L:
        w += survival(j) * prof.t_tx
    return w / prof.batch


def _fits(i: int, j: int, mem_layer: Optional[Sequence[float]], mem_cap: float) -> bool:
    return mem_layer is None or sum(mem_layer[i:j]) <= mem_cap


def plan_dp(ramp_layers: Sequence[int], survival: Callable[[int], float], prof: Profile, gpus: int,
            max_stages: Optional[int] = None, mem_layer: Optional[Sequence[float]] = None,
            mem_cap: float = math.inf, n_stages: Optional[int] = None) -> Tuple[StageLayout, float]:
    """Optimal (bounds, replicas) and its bottleneck (us per input); `n_stages`
    forces the number of stages (to exercise the transport).  A stage
    must hold its layers' weights: sum(mem_layer[i:j]) <= mem_cap (the reason
    the paper splits models across GPUs at all; with no such limit and free
    transfers, pure replication is optimal)."""
    L = ramp_layers[-1] + 1
    cuts = [0] + [r + 1 for r in ramp_layers]          # allowed stage boundaries, cuts[-1] == L
    n = len(cuts)
    max_stages = max_stages or gpus
    INF = math.inf
    # A[c][g][k]: (bottleneck, back-pointer) for layers [0, cuts[c]) on g GPUs in k stages
    A: Dict[Tuple[int, int, int], Tuple[float, Optional[Tuple[int, int, int, int]]]] = {(0, 0, 0): (0.0, None)}
    for c in range(1, n):
        for g in range(1, gpus + 1):
            for k in range(1, min(max_stages, g) + 1):
                best = (INF, None)
                for p in range(c):
                    if not _fits(cuts[p], cuts[c], mem_layer, mem_cap):
                        continue
                    w = stage_cost(cuts[p], cuts[c], ramp_layers, survival, prof, L)
                    for r in range(1, g - (k - 1) + 1):
                        prev = A.get((p, g - r, k - 1))
                        if prev is None or prev[0] == INF:
                            continue
                        v = max(prev[0], w / r)
                        if v < best[0] - 1e-12:
                            best = (v, (p, g - r, k - 1, r))
                A[(c, g, k)] = best
    # fewest stages among the optimum (ties within 1e-12)
    ks = [n_stages] if n_stages else range(1, min(max_stages, gpus) + 1)
    if n_stages:
        max_stages = max(max_stages, n_stages)
    cands = [(A[(n - 1, gpus, k)][0], k) for k in ks
             if (n - 1, gpus, k) in A and A[(n - 1, gpus, k)][0] < INF]
    if not cands:
        raise ValueError("no feasible plan: a ramp-to-ramp range exceeds the memory cap or too few GPUs")
    opt = min(v for v, _ in cands)
    k = min(k for v, k in cands if v <= opt + 1e-12)
    bounds, reps = [cuts[-1]], []
    key = (n - 1, gpus, k)
    while key[2] > 0:
        _, bp = A[key]
        p, g_prev, k_prev, r = bp
        bounds.append(cuts[p])
        reps.append(r)
        key = (p, g_prev, k_prev)
    return StageLayout(tuple(reversed(bounds)), tuple(reversed(reps))), opt


def brute_force_plan(ramp_layers: Sequence[int], survival: Callable[[int], float], prof: Profile, gpus: int,
                     max_stages: Optional[int] = None, mem_layer: Optional[Sequence[float]] = None,
                     mem_cap: float = math.inf) -> Tuple[StageLayout, float]:
    """Enumerate every cut set and replica vector (small cases: the DP's oracle)."""
    L = ramp_layers[-1] + 1
    inner = [r + 1 for r in ramp_layers[:-1]]
    max_stages = max_stages or gpus
    best = None
    for k in range(1, min(max_stages, gpus, len(ramp_layers)) + 1):
        for cs in itertools.combinations(inner, k - 1):
            bounds = (0,) + cs + (L,)
            if not all(_fits(bounds[s], bounds[s + 1], mem_layer, mem_cap) for s in range(k)):
                continue
            w = [stage_cost(bounds[s], bounds[s + 1], ramp_layers, survival, prof, L) for s in range(k)]
            for reps in itertools.product(range(1, gpus + 1), repeat=k):
                if sum(reps) != gpus:
                    continue
                v = max(w[s] / reps[s] for s in range(k))
                key = (v, k)
                if best is None or v < best[0][0] - 1e-12 or (abs(v - best[0][0]) <= 1e-12 and k < best[0][1]):
                    best = (key, StageLayout(bounds, tuple(reps)))
    if best is None:
        raise ValueError("no feasible plan")
    return best[1], best[0][0]


def throughput(bottleneck_us_per_input: float) -> float:
    """Inputs per second of a pipeline whose slowest stage costs `bottleneck`."""
    return 1e6 / bottleneck_us_per_input


# ---------------------------------------------------------------------------
# Exit-wrapper ramp control (§3.4 PAPER.md:985-1017 "A
# simple use-case here is to disable ramps that are not useful", §5.8.6
# disabling the exits inside a split "(except the last one
# which is required)" gains up to 16 % "by avoiding exit-checking overheads").
# Given every input's exit metric at every ramp (recorded on the GPU,
# e3_exits.ramp_metric, in a profiling run whose thresholds never pass) the
# choice of enabled ramps E changes where inputs exit; the cost per input of
# a single-GPU chain cut at the enabled ramps is
#     sum_l S_E(l) t_layer[l] + sum_{r in E} S_E(layer_r) t_ramp     (/ B)
# with S_E(l) the fraction alive entering layer l.  Exhaustive over the
# subsets of the non-final ramps (2^11 for EE-BERT-base).

def exits_with(M, tau, test: str, enabled: Sequence[int], last: int):
    """Exit ramp index of every input (rows of M [n, R]) when only the ramps
    in `enabled` (plus the last) are evaluated; strict tests (R12)."""
    import numpy as np
    M = np.asarray(M, dtype=np.float64)
    n = M.shape[0]
    out = np.full(n, last, dtype=np.int64)
    undecided = np.ones(n, dtype=bool)
    for r in sorted(set(enabled) - {last}):
        t = np.float64(np.float32(tau[r]))
        ok = (M[:, r] > t) if test == "maxprob" else (M[:, r] < t)
        hit = undecided & ok
        out[hit] = r
        undecided &= ~hit
    return out


def ramp_plan_cost(exit_ramp, ramp_layers: Sequence[int], enabled: Sequence[int], prof: Profile) -> float:
    """Expected GPU time per input (us) of the chain with `enabled` ramps."""
    import numpy as np
    L = ramp_layers[-1] + 1
    exit_layer = np.asarray(ramp_layers)[exit_ramp]
    alive = [float(np.mean(exit_layer >= l)) for l in range(L)]        # entering layer l
    work = sum(alive[l] * prof.t_layer[l] for l in range(L))
    ramps = sum(alive[ramp_layers[r]] * prof.t_ramp for r in set(enabled) | {len(ramp_layers) - 1})
    return (work + ramps) / prof.batch


def choose_ramps(M, tau, test: str, ramp_layers: Sequence[int], prof: Profile):
    """Enabled ramp set (ascending, always with the last) of least cost;
    returns (enabled, cost_us_per_input, exit ramp per profiled input)."""
    R = len(ramp_layers)
    last = R - 1
    best = None
    for mask in range(1 << (R - 1)):
        en = tuple(r for r in range(R - 1) if (mask >> r) & 1) + (last,)
        ex = exits_with(M, tau, test, en, last)
        c = ramp_plan_cost(ex, ramp_layers, en, prof)
        key = (round(c, 9), -len(en))                 # ties: keep more ramps (earlier answers)
        if best is None or key < best[0]:
            best = (key, en, c, ex)
    return best[1], best[2], best[3]
