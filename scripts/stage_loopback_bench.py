"""The multi-rank stage pipeline measured on ONE B200 through the LOOPBACK
transport (every rank of the plan in this process, one thread per rank, the
NCCL transport's message / EOS protocol).

EE-BERT-base's per-ramp splits grouped into K stages (parallel.plan_stages
forced to K stages over K ranks, the survival-balanced cuts); each step
pushes the whole job (8192 inputs) through all ranks concurrently on the same
GPU, so the value is one GPU's throughput running the staged plan -- compared
with the single-rank pipeline on the same job, the difference is the cost of
the stage protocol (fixed-size survivor messages, D2D copies, append kernels,
host polling) plus the loss of the single pipeline's deepest-first order.
Writes gpurun_out/r02_stage_loopback.json.

    python scripts/stage_loopback_bench.py [--stages 2,4] [--steps 5]
"""
import argparse
import json
import os
import sys
import threading
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api, parallel as par  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--stages", default="2,4")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--inputs", type=int, default=8192)
    args = ap.parse_args()
    dev = "cuda:0"
    cfg = e3data.get("bb")
    tau = e3data.tau_for(cfg)
    model = api.DeviceModel(cfg, e3data.make_weights(cfg), dev)
    n = args.inputs
    X = api.to_bf16(e3data.make_inputs(cfg, range(n)), dev)
    ids = torch.arange(n, dtype=torch.int64, device=dev)
    bounds = tuple(range(13))
    surv = lambda l: 1.0 - sum(e for r, e in zip(cfg.ramp_layers, cfg.exit_profile) if r < l)
    out = {"what": "EE-BERT-base, one B200, all ranks of a K-stage plan in one process (LOOPBACK transport); "
                   f"{n} inputs per step, {args.steps} timed steps after 2 warm-up steps", "runs": []}

    # single-rank reference
    pipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau))
    ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, dev)
    for _ in range(2):
        pipe.run(X, ids, ex)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        pipe.run(X, ids, ex)
    torch.cuda.synchronize()
    ref = n * args.steps / (time.perf_counter() - t0)
    el_ref = ex.exit_layer.cpu().numpy()
    out["single_rank_inputs_per_s"] = round(ref, 1)
    del pipe

    for k in [int(v) for v in args.stages.split(",")]:
        layout = par.plan_stages(cfg.ramp_layers, surv, k, n_stages=k)
        comms = api.Comm.loopback(k, 0)
        plan = api.make_plan(cfg, bounds, tau, placement=par.placement(layout, bounds), transport="loopback")
        pipes = [api.Pipeline(model, plan, comms[r]) for r in range(k)]
        exs = [api.ExitBuffers(n, cfg.classes, cfg.n_ramps, dev) for _ in range(k)]
        streams = [torch.cuda.Stream(dev) for _ in range(k)]
        stats = [None] * k
        errs = []

        def step():
            def work(r):
                try:
                    g, _ = layout.stage_of(r)
                    stats[r] = pipes[r].run(X if g == 0 else None, ids if g == 0 else None, exs[r], stream=streams[r])
                except Exception as e:
                    errs.append(e)
            th = [threading.Thread(target=work, args=(r,)) for r in range(k)]
            for t in th:
                t.start()
            for t in th:
                t.join()
            assert not errs, errs

        for _ in range(2):
            step()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            step()
        torch.cuda.synchronize()
        v = n * args.steps / (time.perf_counter() - t0)
        el = np.full(n, -1)
        for e in exs:
            a = e.exit_layer.cpu().numpy()
            el[a >= 0] = a[a >= 0]
        out["runs"].append({"stages": k, "bounds": list(layout.bounds), "replicas": list(layout.replicas),
                            "inputs_per_s": round(v, 1), "vs_single_rank": round(v / ref, 4),
                            "exits_equal_single_rank": bool(np.array_equal(el, el_ref)),
                            "messages": [int(s.msgs_sent) for s in stats],
                            "flushes_per_rank": [int(sum(s.flushes[j] for j in range(12))) for s in stats]})
        print(json.dumps(out["runs"][-1]), flush=True)
        del pipes
        for c in comms:
            c.close()
    json.dump(out, open(os.path.join(ROOT, "gpurun_out", "r02_stage_loopback.json"), "w"), indent=1)
    print(json.dumps({"single_rank": out["single_rank_inputs_per_s"]}))


if __name__ == "__main__":
    main()
