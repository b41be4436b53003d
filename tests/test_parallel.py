"""Multi-process (gloo, CPU) tests of the multi-GPU drivers in parallel.py:
replica sharding, the stage-pipeline transport (count header + rows + ids,
chunk ownership), stage planning and the exit-record reduction.  The GPU
executor is replaced by a stand-in that applies a fixed exit-layer table, so
what is tested is exactly the host-side routing."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sosp_iyergdpgn24_b200 import parallel as par

L = 12
RAMPS = list(range(L))
N_IDS = 300
CHUNK = 40
ROW = (2, 3)


def _exit_table(seed=5):
    g = torch.Generator().manual_seed(seed)
    return torch.randint(0, L, (N_IDS,), generator=g)


class StandIn:
    """Stage [a, b): inputs whose exit layer < b exit here, the rest survive.
    Checks the payload arrived intact (row of input i == i)."""

    def __init__(self, a, b, table):
        self.a, self.b, self.table = a, b, table
        self.exit_at = torch.full((N_IDS,), -1, dtype=torch.int64)
        self.seen = torch.zeros((N_IDS,), dtype=torch.int64)
        self.bad = 0

    def run(self, x, ids):
        for r in range(ids.shape[0]):
            i = int(ids[r])
            self.seen[i] += 1
            if not torch.all(x[r] == float(i)):
                self.bad += 1
            if int(self.table[i]) < self.a:
                self.bad += 1              # should have exited upstream
        e = self.table[ids] < self.b
        self.exit_at[ids[e]] = self.table[ids[e]]
        keep = ~e
        if self.b == L:
            return None, None, 0
        xs, ids_s = x[keep].clone(), ids[keep].clone()
        # pad the survivor buffer the way the GPU executor does (capacity >= n)
        pad = 3
        xs = torch.cat([xs, torch.zeros((pad,) + ROW)])
        ids_s = torch.cat([ids_s, torch.full((pad,), -7, dtype=torch.int64)])
        return xs, ids_s, int(keep.sum())


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, bounds, replicas, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        layout = par.StageLayout(tuple(bounds), tuple(replicas))
        g, _ = layout.stage_of(rank)
        table = _exit_table()
        ex = StandIn(bounds[g], bounds[g + 1], table)
        n_chunks = (N_IDS + CHUNK - 1) // CHUNK

        def chunk_inputs(c):
            ids = torch.arange(c * CHUNK, min(N_IDS, (c + 1) * CHUNK), dtype=torch.int64)
            x = ids.to(torch.float32)[:, None, None].expand((ids.shape[0],) + ROW).contiguous()
            return x, ids

        st = par.run_stage_pipeline(ex, layout, rank, n_chunks, chunk_inputs, ROW, torch.float32, "cpu",
                                    par.Transport(device=False))
        exit_at = ex.exit_at.clone()
        dist.all_reduce(exit_at, op=dist.ReduceOp.MAX)
        exited_here = (ex.exit_at >= 0).to(torch.int64)
        dist.all_reduce(exited_here, op=dist.ReduceOp.SUM)
        seen = ex.seen.clone()
        dist.all_reduce(seen, op=dist.ReduceOp.SUM)
        bad = torch.tensor([ex.bad])
        dist.all_reduce(bad, op=dist.ReduceOp.SUM)
        if rank == 0:
            q.put({"exit_at": exit_at, "count": exited_here, "seen": seen, "bad": int(bad), "stats": st})
    finally:
        dist.destroy_process_group()


def _run(bounds, replicas):
    world = sum(replicas)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, bounds, replicas, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return res


@pytest.mark.parametrize("bounds,replicas", [((0, 4, 12), (1, 1)),
                                             ((0, 4, 12), (1, 2)),
                                             ((0, 3, 12), (2, 1)),
                                             ((0, 2, 6, 12), (1, 1, 1))])
def test_stage_pipeline_routes_every_input_once(bounds, replicas):
    res = _run(bounds, replicas)
    table = _exit_table()
    assert res["bad"] == 0
    assert torch.equal(res["exit_at"], table)           # every input exits at its own layer
    assert torch.equal(res["count"], torch.ones(N_IDS, dtype=torch.int64))   # exactly once
    # input i is seen by every stage whose first layer is <= its exit layer
    starts = torch.tensor(bounds[:-1])
    expect_seen = (starts[None, :] <= table[:, None]).sum(1)
    assert torch.equal(res["seen"], expect_seen)


def test_shard_covers_all():
    for n in (0, 1, 7, 100):
        for w in (1, 2, 3, 8):
            parts = [par.shard(n, w, r) for r in range(w)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(parts[i][1] == parts[i + 1][0] for i in range(w - 1))
            assert max(h - l for l, h in parts) - min(h - l for l, h in parts) <= 1


def test_layout_ownership():
    lay = par.StageLayout((0, 4, 12), (1, 3))
    assert lay.world == 4 and lay.n_stages == 2
    assert lay.ranks_of(1) == [1, 2, 3]
    assert [lay.owner(1, c) for c in range(6)] == [1, 2, 3, 1, 2, 3]
    assert lay.stage_of(2) == (1, 1)


def test_plan_stages_balances():
    # uniform cost: G GPUs -> the bottleneck is L / G (a perfect split exists)
    lay = par.plan_stages(RAMPS, lambda l: 1.0, 4)
    w = [lay.bounds[g + 1] - lay.bounds[g] for g in range(lay.n_stages)]
    assert max(w[g] / lay.replicas[g] for g in range(lay.n_stages)) == pytest.approx(3.0)
    assert lay.world == 4
    # one GPU -> one stage holding everything
    assert par.plan_stages(RAMPS, lambda l: 1.0, 1) == par.StageLayout((0, L), (1,))
    # steep survival decay: the first stage is the short one
    lay = par.plan_stages(RAMPS, lambda l: 0.5 ** l, 2)
    assert lay.n_stages in (1, 2)
    if lay.n_stages == 2:
        assert lay.bounds[1] <= 2
    # brute-force check of optimality on a small instance
    surv = [1.0, 0.9, 0.5, 0.45, 0.2, 0.1]
    lay = par.plan_stages(list(range(6)), lambda l: surv[l], 3)
    cost = max(sum(surv[lay.bounds[g]:lay.bounds[g + 1]]) / lay.replicas[g] for g in range(lay.n_stages))
    best = float("inf")
    import itertools
    for k in (1, 2, 3):
        for cuts in itertools.combinations(range(1, 6), k - 1):
            b = (0,) + cuts + (6,)
            for r in itertools.product(range(1, 4), repeat=k):
                if sum(r) != 3:
                    continue
                best = min(best, max(sum(surv[b[g]:b[g + 1]]) / r[g] for g in range(k)))
    assert cost == pytest.approx(best)
