"""Constant-batch split pipeline bookkeeping — TEST INFRASTRUCTURE ONLY.

Pure integer bookkeeping on the per-input exit layers produced by
oracle.model.run.  It replays the queue discipline of
E3's execution ("we execute the first split twice ... combine the
two outputs to obtain a batch size of 16"; "multiple batches are
fused to bring the batch to the correct size", "a queue that holds the
partial results"):

* split 0 consumes the inputs in id order, B at a time;
* after a run of split s, its survivors (exit layer beyond the split's last
  layer), in batch order, are appended to queue s+1 (FIFO, stable; R8);
* a batch of exactly B rows is popped whenever a queue holds >= B
  (never more than B: "without overshooting"; R10);
* when no queue holds B rows and nothing upstream can still deliver, the
  shallowest non-empty queue is flushed, padded to B (R9);
* among ready splits the deepest runs first (R8).

``lag`` models the executor's asynchronous host loop: the decision for run t
sees the survivor counts of runs <= t-1-lag; when no decision is possible
with that knowledge it waits for the outstanding runs.  lag=0 is the serial
policy; lag=1 is what e3_pipeline_run uses.  Both
are deterministic functions of the exit layers.

Pins (tests/test_oracle_pipeline.py): the Fig. 5 / §3.2 worked example
(16 in, 8 survive per run, two 8s -> one 16), the §5.8.3 arithmetic
(16 -> 8, or 12 with a 50% prediction error), collections.deque FIFO, and
the invariants: every split batch has exactly B rows, padding only on flush
batches, every input exits exactly once, conservation per split.
"""
from __future__ import annotations

from collections import deque
from dataclasses import dataclass, field
from typing import Dict, List, Sequence, Tuple


@dataclass(frozen=True)
class Plan:
    """Cut points of a split plan: split s covers layers [bounds[s], bounds[s+1])."""
    bounds: Tuple[int, ...]

    @property
    def n_splits(self) -> int:
        return len(self.bounds) - 1

    def split_end(self, s: int) -> int:
        """Last layer (0-based, inclusive) of split s."""
        return self.bounds[s + 1] - 1

    @staticmethod
    def per_ramp(ramp_layers: Sequence[int]) -> "Plan":
        """Every ramp ends a split (constant B at every layer; R7)."""
        return Plan((0,) + tuple(l + 1 for l in ramp_layers))

    @staticmethod
    def cuts(layers: int, cut_after: Sequence[int]) -> "Plan":
        """Cut after the given 0-based layers (each must carry a ramp)."""
        return Plan((0,) + tuple(c + 1 for c in cut_after) + (layers,))


@dataclass
class Run:
    split: int
    ids: Tuple[int, ...]       # valid rows, batch order
    n_valid: int
    flush: bool


@dataclass
class SimResult:
    runs: List[Run]
    batch: int
    per_split: Dict[int, Dict[str, int]] = field(default_factory=dict)


def simulate_pipeline(exit_layer: Dict[int, int], order: Sequence[int], plan: Plan,
                      B: int, lag: int = 1) -> SimResult:
    """Replay the constant-batch pipeline on one device.

    exit_layer: input id -> 0-based exit layer; order: input ids in arrival
    order; returns every split run in dispatch order.
    """
    k = plan.n_splits
    queues = [deque(order)] + [deque() for _ in range(k - 1)]
    pending = deque()          # launched runs whose pushes are not yet known
    runs: List[Run] = []

    def apply_oldest():
        s, surv = pending.popleft()
        if s + 1 < k:
            queues[s + 1].extend(surv)
        else:
            assert not surv, "the last split must exit every row"

    def decide():
        for s in range(k - 1, -1, -1):
            if len(queues[s]) >= B:
                return s, False
        if pending:
            return None
        for s in range(k):
            if queues[s]:
                return s, True
        return None

    while True:
        while len(pending) > lag:
            apply_oldest()
        d = decide()
        if d is None:
            if pending:
                apply_oldest()
                continue
            break
        s, flush = d
        n = min(B, len(queues[s]))
        batch = tuple(queues[s].popleft() for _ in range(n))
        end = plan.split_end(s)
        surv = [i for i in batch if exit_layer[i] > end]
        runs.append(Run(s, batch, n, flush))
        pending.append((s, surv))
    while pending:
        apply_oldest()

    per = {s: {"batches": 0, "valid": 0, "padded": 0, "rows_out": 0} for s in range(k)}
    for r in runs:
        p = per[r.split]
        p["batches"] += 1
        p["valid"] += r.n_valid
        p["padded"] += B - r.n_valid
        p["rows_out"] += sum(1 for i in r.ids if exit_layer[i] > plan.split_end(r.split))
    return SimResult(runs, B, per)
