"""-m gpu: the stage pipeline with the real GPU executor (two processes sharing
cuda:0, survivors shipped through host memory over gloo -- this box has one
GPU; with NCCL on separate GPUs the same code ships them device to device).
Per input the exit record equals the single-process pipeline's bitwise."""
import os
import socket
import types

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from tests.gpu_util import requires_cuda

pytestmark = [pytest.mark.gpu, requires_cuda]

N = 150
CHUNK = 40


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import e3data
        from paper_conf_sosp_iyergdpgn24_b200 import api, parallel as par
        dev = torch.device("cuda", 0)
        torch.cuda.set_device(dev)
        cfg = e3data.get("tiny")
        model = api.DeviceModel(cfg, e3data.make_weights(cfg), dev)
        layout = par.StageLayout((0, 2, 4), (1, 1))
        g, _ = layout.stage_of(rank)
        ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, dev)
        execu = par.GpuStageExecutor(model, cfg, layout.bounds[g], layout.bounds[g + 1], cfg.tau, ex, CHUNK)

        def chunk_inputs(c):
            r = range(c * CHUNK, min(N, (c + 1) * CHUNK))
            x = torch.from_numpy(e3data.make_inputs(cfg, r, seed=11)).to(torch.bfloat16).to(dev)
            return x, torch.tensor(list(r), dtype=torch.int64, device=dev)

        n_chunks = (N + CHUNK - 1) // CHUNK
        par.run_stage_pipeline(execu, layout, rank, n_chunks, chunk_inputs, (cfg.seq, cfg.hidden),
                               torch.bfloat16, dev, par.Transport(device=False))
        torch.cuda.synchronize()
        cpu = types.SimpleNamespace(exit_layer=ex.exit_layer.cpu(), label=ex.label.cpu(), conf=ex.conf.cpu(),
                                    logits=ex.logits.cpu(), n_exit=ex.n_exit.cpu(), ramp_count=ex.ramp_count.cpu())
        par.reduce_exits(cpu)
        if rank == 0:
            q.put({k: getattr(cpu, k) for k in ("exit_layer", "label", "logits", "n_exit")})
    finally:
        dist.destroy_process_group()


def test_stage_pipeline_gpu_equals_single_pipeline():
    import e3data
    from paper_conf_sosp_iyergdpgn24_b200 import api
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    dev = torch.device("cuda", 0)
    cfg = e3data.get("tiny")
    model = api.DeviceModel(cfg, e3data.make_weights(cfg), dev)
    ref = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, dev)
    X = torch.from_numpy(e3data.make_inputs(cfg, range(N), seed=11)).to(torch.bfloat16).to(dev)
    api.Pipeline(model, api.make_plan(cfg, (0, 2, 4), cfg.tau)).run(X, torch.arange(N, device=dev), ref)
    assert int(res["n_exit"]) == N
    assert torch.equal(res["exit_layer"], ref.exit_layer.cpu())
    assert torch.equal(res["label"], ref.label.cpu())
    assert torch.equal(res["logits"], ref.logits.cpu())
