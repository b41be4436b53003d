"""Multi-GPU drivers of the split path: one process per GPU, torch.distributed
for the plumbing.

Two modes:

* replica  -- every rank runs the whole split chain on its own shard of the
  inputs (inputs are independent, so the path shards with no data-path
  collective).  ``shard`` gives the contiguous shard of a rank.

* stage    -- E3's model-parallel execution (Fig. 5): the
  split chain is cut into contiguous STAGES placed on different GPUs, each
  stage optionally replicated.  Inputs flow in chunks; stage g runs its
  splits on a chunk (constant batch inside, e3_pipeline_run_out) and ships
  the survivors -- a count, then the [n, S, H] rows and their ids -- to the
  replica of stage g+1 that owns the chunk ("outputs are then directed to the
  machines hosting the next split").  With the NCCL backend
  the rows go GPU-to-GPU over NVLink (ncclSend/ncclRecv); the count header
  lets the receiver post a receive of exactly the right size (NCCL needs
  matching counts).  Chunk c of stage g is handled by replica c mod r_g, so
  every rank knows, without any coordination, whom to receive from and send
  to.  Sends are asynchronous (isend): stage g computes chunk c+1 while chunk
  c travels and stage g+1 computes it -- the steady-state pipeline of §3.2.2
  (PAPER.md:907-913).

``plan_stages`` balances the stages (the paper's pipelined DP, PAPER.md:
907-930, restricted to one GPU type): minimise max_g W_g / r_g over contiguous
cuts at ramps and replica counts r_g (sum r_g = G), W_g = expected
survivor-layers of stage g.

The executor is duck-typed so the host-side logic runs under the gloo backend
on CPU with a stand-in executor (tests/test_parallel.py); on GPUs
``GpuStageExecutor`` wraps the C-ABI pipeline.
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

    def owner(self, g: int, chunk: int) -> int:
        """Rank of stage g that processes chunk `chunk`."""
        return self.ranks_of(g)[chunk % self.replicas[g]]


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


# ---------------------------------------------------------------- transport

class Transport:
    """Point-to-point rows between ranks.  device=True: tensors stay on the GPU
    (NCCL over NVLink); device=False: staged through host memory (gloo)."""

    def __init__(self, device: bool):
        self.device = device

    def isend(self, t: torch.Tensor, dst: int):
        if not self.device and t.is_cuda:
            t = t.cpu()
        return dist.isend(t.contiguous(), dst), t

    def recv(self, shape, dtype, src: int, dev) -> torch.Tensor:
        if self.device:
            t = torch.empty(shape, dtype=dtype, device=dev)
        else:
            t = torch.empty(shape, dtype=dtype)
        dist.recv(t, src)
        return t.to(dev) if (not self.device and dev is not None and torch.device(dev).type == "cuda") else t


def run_stage_pipeline(executor, layout: StageLayout, rank: int, n_chunks: int,
                       chunk_inputs: Callable[[int], Tuple[torch.Tensor, torch.Tensor]],
                       row_shape: Tuple[int, ...], row_dtype, dev, transport: Transport) -> dict:
    """Run this rank's stage over every chunk it owns (SPMD: call on all ranks).

    executor.run(x, ids) -> (x_surv, ids_surv, n_surv)   (stage not last)
    executor.run(x, ids) -> (None, None, 0)               (last stage)
    chunk_inputs(c) -> (x, ids) for the stage-0 owner of chunk c.
    Returns counters {chunks, rows_in, rows_out}."""
    g, _ = layout.stage_of(rank)
    last = g == layout.n_stages - 1
    stats = {"chunks": 0, "rows_in": 0, "rows_out": 0}
    pending = []                               # in-flight sends (keep tensors alive)
    for c in range(n_chunks):
        if layout.owner(g, c) != rank:
            continue
        if g == 0:
            x, ids = chunk_inputs(c)
        else:
            src = layout.owner(g - 1, c)
            hdr = transport.recv((1,), torch.int64, src, dev)
            n = int(hdr.item())
            if n > 0:
                x = transport.recv((n,) + tuple(row_shape), row_dtype, src, dev)
                ids = transport.recv((n,), torch.int64, src, dev)
            else:
                x = torch.empty((0,) + tuple(row_shape), dtype=row_dtype, device=dev)
                ids = torch.empty((0,), dtype=torch.int64, device=dev)
        stats["chunks"] += 1
        stats["rows_in"] += int(ids.shape[0])
        xs, ids_s, n_s = executor.run(x, ids)
        if last:
            continue
        dst = layout.owner(g + 1, c)
        hdr = torch.tensor([n_s], dtype=torch.int64, device=dev if transport.device else "cpu")
        pending.append(transport.isend(hdr, dst))
        if n_s > 0:
            # private copies: the executor reuses its output buffers for the
            # next chunk while an NCCL isend of this one may still be queued
            pending.append(transport.isend(xs[:n_s].clone(), dst))
            pending.append(transport.isend(ids_s[:n_s].clone(), dst))
        stats["rows_out"] += n_s
        while len(pending) > 12:               # bound the in-flight buffers
            pending.pop(0)[0].wait()
    for work, _ in pending:
        work.wait()
    return stats


class GpuStageExecutor:
    """One stage on this GPU: the split chain of layers [begin, end) through the
    C ABI (e3_pipeline_run / e3_pipeline_run_out), survivors into a buffer."""

    def __init__(self, model, cfg, begin: int, end: int, tau, exits, max_rows: int, lag: int = 1):
        from . import api
        bounds = [begin] + [l + 1 for l in cfg.ramp_layers if begin <= l < end]
        self.pipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau, lag=lag))
        self.final = end == cfg.layers
        self.exits = exits
        dev = model.device
        if not self.final:
            self.x_out = torch.empty((max_rows, cfg.seq, cfg.hidden), dtype=torch.bfloat16, device=dev)
            self.id_out = torch.empty((max_rows,), dtype=torch.int64, device=dev)

    def run(self, x, ids):
        if self.final:
            self.pipe.run(x, ids, self.exits)
            return None, None, 0
        n = int(ids.shape[0])
        _, n_out = self.pipe.run_out(x, ids, self.exits, self.x_out[:max(n, 1)], self.id_out[:max(n, 1)])
        return self.x_out, self.id_out, n_out


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
