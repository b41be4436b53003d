"""Multi-process (gloo, CPU) tests of the multi-GPU plumbing in parallel.py:
stage planning, per-split placement, input shares, the communicator-id
broadcast and the exit-record reduction.  The data path
itself (stage loop, messages, re-batching) is in libe3.so and is tested on
the GPU (tests/test_gpu_stage.py, LOOPBACK transport, and NCCL on >= 2 GPUs)."""
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


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class _FakeExits:
    """The fields of api.ExitBuffers that reduce_exits combines (CPU tensors)."""

    def __init__(self, n, c, r):
        self.exit_layer = torch.full((n,), -1, dtype=torch.int32)
        self.label = torch.full((n,), -1, dtype=torch.int32)
        self.conf = torch.full((n,), float("nan"))
        self.logits = torch.zeros((n, c))
        self.n_exit = torch.zeros((1,), dtype=torch.int32)
        self.ramp_count = torch.zeros((r,), dtype=torch.int32)


def _worker(rank, world, port, bounds, replicas, q):
    """One rank of a stage layout over gloo: every rank derives the same
    placement, the stage-0 replicas' input shares partition the job, the
    communicator id broadcast reaches every rank, and the exit records of
    inputs exiting on different ranks merge into one record per input."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        layout = par.StageLayout(tuple(bounds), tuple(replicas))
        split_bounds = tuple(range(L + 1))          # per-ramp splits
        pl = par.placement(layout, split_bounds)
        allp = [None] * world
        dist.all_gather_object(allp, pl)
        lo, hi = par.input_share(layout, rank, N_IDS)
        shares = [None] * world
        dist.all_gather_object(shares, (lo, hi))
        uid = [bytes(range(128)) if rank == 0 else None]   # stands in for e3_comm_unique_id
        dist.broadcast_object_list(uid, src=0)
        # exit records: input i exits on the rank of the stage holding layer table[i]
        table = torch.arange(N_IDS) % L
        g, _ = layout.stage_of(rank)
        ex = _FakeExits(N_IDS, 2, L)
        mine = [i for i in range(N_IDS) if layout.bounds[g] <= int(table[i]) < layout.bounds[g + 1]
                and i % layout.replicas[g] == layout.stage_of(rank)[1]]
        for i in mine:
            ex.exit_layer[i] = int(table[i])
            ex.label[i] = i % 2
            ex.conf[i] = 0.5
            ex.logits[i] = torch.tensor([float(i), -float(i)])
        ex.n_exit[0] = len(mine)
        par.reduce_exits(ex)
        if rank == 0:
            q.put({"placements": allp, "shares": shares, "uid": uid[0], "exit_layer": ex.exit_layer,
                   "logits": ex.logits, "n_exit": int(ex.n_exit[0]), "label": ex.label})
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
    res = q.get(timeout=600)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return res


@pytest.mark.parametrize("bounds,replicas", [((0, 4, 12), (1, 1)),
                                             ((0, 4, 12), (1, 2)),
                                             ((0, 3, 12), (2, 1)),
                                             ((0, 2, 6, 12), (1, 1, 1))])
def test_stage_plumbing_world_size_gt_1(bounds, replicas):
    res = _run(bounds, replicas)
    world = sum(replicas)
    assert all(p == res["placements"][0] for p in res["placements"])       # one plan on every rank
    pl = res["placements"][0]
    lay = par.StageLayout(tuple(bounds), tuple(replicas))
    for s in range(L):
        g = max(i for i in range(lay.n_stages) if bounds[i] <= s)
        assert pl[s] == lay.ranks_of(g)
    shares = [tuple(x) for x in res["shares"] if x[1] > x[0]]
    assert sorted(shares)[0][0] == 0 and sorted(shares)[-1][1] == N_IDS
    assert sum(h - l for l, h in shares) == N_IDS and len(shares) == replicas[0]
    assert res["uid"] == bytes(range(128))
    table = torch.arange(N_IDS) % L
    assert torch.equal(res["exit_layer"].to(torch.int64), table)       # merged: one record per input
    assert res["n_exit"] == N_IDS
    assert torch.equal(res["logits"][:, 0], torch.arange(N_IDS, dtype=torch.float32))


def test_placement_rejects_cuts_inside_a_split():
    lay = par.StageLayout((0, 3, 12), (1, 1))
    with pytest.raises(ValueError):
        par.placement(lay, (0, 2, 4, 12))
    assert par.placement(lay, (0, 3, 12)) == [[0], [1]]


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
    assert lay.stage_of(2) == (1, 1)
    assert par.input_share(lay, 0, 10) == (0, 10) and par.input_share(lay, 2, 10) == (0, 0)


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
