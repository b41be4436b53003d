"""Multi-GPU plumbing of the split path: one process per GPU, torch.distributed
for rendezvous only.  The data path -- the
stage loop, survivor messages over NCCL, re-batching -- runs in libe3.so
(e3_comm_* / e3_pipeline_* with e3_plan placement); this module only

* plans the stages (``plan_stages``: the paper's pipelined balance,
  PAPER.md:907-930, restricted to one GPU type): contiguous cuts at ramps and
  replica counts minimising the bottleneck max_g W_g / r_g, W_g = expected
  survivor-layers of stage g;
* turns a stage layout into the per-split placement of e3_plan
  (``placement``) and each stage-0 replica's share of the inputs
  (``input_share``);
* creates the library's NCCL communicator from a torch process group
  (``make_comm``: the unique id travels over the group);
* merges the per-rank exit records (``reduce_exits``).

Two modes of bench.py --gpus N:
  stage    E3's model-parallel execution (Fig. 5): stages
           on different GPUs, survivors shipped by the library over NVLink;
  replica  every rank runs the whole chain on its own shard (no data-path
           collective) -- printed as the comparison.
"""
from __future__ import annotations

import itertools
from dataclasses import dataclass
from typing import Callable, List, Optional, Sequence, Tuple

import torch
import torch.distributed as dist


def shard(n: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous shard [lo, hi) of n inputs for `rank` (replica mode)."""
    base, extra = divmod(n, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


@dataclass(frozen=True)
class StageLayout:
    """bounds[g]..bounds[g+1]: the layers of stage g (cuts at ramps);
    replicas[g]: number of ranks running stage g; ranks are assigned in order."""
    bounds: Tuple[int, ...]
    replicas: Tuple[int, ...]

    @property
    def n_stages(self) -> int:
        return len(self.bounds) - 1

    @property
    def world(self) -> int:
        return sum(self.replicas)

    def ranks_of(self, g: int) -> List[int]:
        first = sum(self.replicas[:g])
        return list(range(first, first + self.replicas[g]))

    def stage_of(self, rank: int) -> Tuple[int, int]:
        """(stage, replica index) of a rank."""
        for g in range(self.n_stages):
            rs = self.ranks_of(g)
            if rank in rs:
                return g, rs.index(rank)
        raise ValueError(rank)


def plan_stages(ramp_layers: Sequence[int], survival: Callable[[int], float], world: int,
                max_stages: Optional[int] = None, n_stages: Optional[int] = None) -> StageLayout:
    """Balanced stage layout for `world` GPUs.

    Layer l (0-based) costs survival(l) = expected fraction of inputs still
    alive when entering it.  Cuts are allowed after ramp layers only.  Brute
    force over cut sets (L <= 32 ramps) and replica splits; minimises the
    bottleneck max_g W_g / r_g, ties broken by fewer stages.  On identical
    GPUs with free inter-GPU transfer pure replication is optimal (one stage);
    `n_stages` forces the number of stages (the paper's setting of models
    that do not fit one GPU, or to exercise the transport)."""
    if n_stages is not None and not 1 <= n_stages <= min(world, len(ramp_layers)):
        raise ValueError(f"n_stages={n_stages} needs 1 <= n_stages <= min(world={world}, "
                         f"ramps={len(ramp_layers)})")
    cut_points = [l + 1 for l in ramp_layers[:-1]]
    L = ramp_layers[-1] + 1
    best = None
    max_stages = min(world, max_stages or world, len(ramp_layers))
    ks = [n_stages] if n_stages else range(1, max_stages + 1)
    for k in ks:
        for cuts in itertools.combinations(cut_points, k - 1):
            bounds = (0,) + tuple(cuts) + (L,)
            w = [sum(survival(l) for l in range(bounds[g], bounds[g + 1])) for g in range(k)]
            # replicas: greedily give the next GPU to the current bottleneck
            r = [1] * k
            for _ in range(world - k):
                i = max(range(k), key=lambda g: w[g] / r[g])
                r[i] += 1
            cost = max(w[g] / r[g] for g in range(k))
            key = (round(cost, 12), k)
            if best is None or key < best[0]:
                best = (key, StageLayout(bounds, tuple(r)))
    return best[1]


def placement(layout: StageLayout, split_bounds: Sequence[int]) -> List[List[int]]:
    """Per split (split s = layers [split_bounds[s], split_bounds[s+1])) the
    ranks of its replicas: those of the stage containing it.  Every stage
    boundary must be a split boundary."""
    for b in layout.bounds:
        if b not in split_bounds:
            raise ValueError(f"stage boundary {b} is not a split boundary {tuple(split_bounds)}")
    out = []
    for s in range(len(split_bounds) - 1):
        g = max(i for i in range(layout.n_stages) if layout.bounds[i] <= split_bounds[s])
        out.append(layout.ranks_of(g))
    return out


def input_share(layout: StageLayout, rank: int, n: int) -> Tuple[int, int]:
    """Inputs [lo, hi) of a job of n that `rank` feeds into split 0 (stage-0
    replicas split the job contiguously; other ranks get an empty range)."""
    g, i = layout.stage_of(rank)
    if g != 0:
        return 0, 0
    return shard(n, layout.replicas[0], i)


def make_comm(rank: int, world: int, device: int, group=None):
    """The library's NCCL communicator for this rank: rank 0 creates the
    unique id, the torch process group carries it to every rank."""
    from . import api
    obj = [api.Comm.unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return api.Comm.nccl(obj[0], rank, world, device)


def reduce_exits(exits, group=None):
    """Combine per-rank exit records (each input exited on exactly one rank):
    exit_layer / label by MAX over the -1 initialisation, logits by SUM."""
    dist.all_reduce(exits.exit_layer, op=dist.ReduceOp.MAX, group=group)
    dist.all_reduce(exits.label, op=dist.ReduceOp.MAX, group=group)
    conf = torch.nan_to_num(exits.conf, nan=-float("inf"))
    dist.all_reduce(conf, op=dist.ReduceOp.MAX, group=group)
    exits.conf.copy_(conf)
    if exits.logits is not None:
        dist.all_reduce(exits.logits, op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(exits.n_exit, op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(exits.ramp_count, op=dist.ReduceOp.SUM, group=group)
