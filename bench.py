"""Benchmark of the E3 early-exit split path on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--config bb] [--inputs-per-gpu 8192] [--plan per-ramp|cut6]

Metric (BASELINE.json): inputs/sec at constant batch, EE-BERT-base
(12 layers, H 768, S 128, B 64, a ramp after every layer, bf16), plus %
of roofline.  One STEP = one e3_pipeline_run over a fixed job of inputs
(default 8192 per GPU, 1.6 GB of activations, larger than L2): every input
goes through split after split (all §8(a) rows: constant-B split input,
layer stack, fused ramp + threshold, stable compaction, re-batching top-up,
stage loop) until it exits.  Inputs are resident in HBM when the timed region
starts; `e2e` repeats the measurement through the same C-ABI call with HOST
(pinned) inputs, the H2D copies and the D2H read of the exit records inside
the timed region.

N > 1 (torchrun): stage mode (default) -- the per-ramp split chain is cut
into stages on different GPUs (parallel.plan_stages, balanced on the
calibrated survival profile; --stages, default min(N, 4)) and run by the
library's multi-rank pipeline: every rank calls e3_pipeline_run on the same
plan, survivors travel GPU to GPU as NCCL messages issued by libe3.so
(e3_comm_*, e3_plan.replicas / device_of).  The replica mode (every rank runs
the whole chain on its own shard, no data-path collective) is timed right
after and printed as "replica_comparison".  --mode replica times only that.
Per-GPU load is fixed (weak scaling).  Time = max over ranks of CUDA-event
time, barrier + synchronize around it.

--impl reference: the CPU oracle (oracle/, NumPy float64) timed on the host
cores on a bounded sample of the same workload (this tier has no reference
implementation to install).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "inputs/sec at constant batch (EE-BERT-base) at 1/2/4/8 B200; % roofline"
METRIC_LM = "tokens/sec of the early-exit decode step (EE decoder LLM, Llama-7B shape) at constant batch"
# BASELINE.json's metric names the headline model; the other encoder configs
# report the same metric for their own model
MODEL_NAME = {"ee-bert-base": "EE-BERT-base", "ee-bert-large": "EE-BERT-large", "ee-vit-b16": "EE-ViT-B/16",
              "ee-bert-base-pabee": "EE-BERT-base, PABEE patience exits", "tiny": "tiny EE encoder",
              "tiny-vit": "tiny EE-ViT"}


def metric_of(cfg):
    if cfg.arch == "llama":
        if cfg.name == "ee-llama3-8b-decode":
            return METRIC_LM.replace("Llama-7B shape", "Llama-3.1-8B shape, GQA 8 KV heads, V 128256")
        return METRIC_LM
    return METRIC.replace("EE-BERT-base", MODEL_NAME.get(cfg.name, cfg.name))


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="bb")
    ap.add_argument("--inputs-per-gpu", type=int, default=None,
                    help="default 8192 (encoders: > L2 of activations), 512 (llama: 512 sequences' KV caches, "
                         "~138 GB, so that padding stays near 5 %% at every split)")
    ap.add_argument("--decode-steps", type=int, default=0,
                    help="llama: one step = e3_decode_run of this many greedy tokens per sequence (NEXT-2: "
                         "skipped layers' K/V filled from the exit state); 0 = one token (e3_pipeline_run)")
    ap.add_argument("--plan", default="per-ramp", choices=["per-ramp", "cut6"])
    ap.add_argument("--lag", type=int, default=1, help="host look-behind of the stage loop (runs in flight)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-inputs", type=int, default=32)
    ap.add_argument("--mode", default="stage", choices=["replica", "stage"],
                    help="N>1: stages on different GPUs (library NCCL transfers), or replicas of the whole chain")
    ap.add_argument("--stages", type=int, default=0, help="stage mode: number of stages (0: min(N, 4))")
    ap.add_argument("--planner", default="balance", choices=["balance", "dp"],
                    help="stage mode: survival-balanced cuts, or the profile-driven DP (planner.py)")
    return ap.parse_args()


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.rows, self.proc = index, [], None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([c.strip() for c in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4)
                          if len(r) > 3 + i and r[3 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def load_workload(cfg_name):
    import e3data
    cfg = e3data.get(cfg_name)
    return cfg, e3data.tau_for(cfg)   # calibrated thresholds: committed data file


def plan_bounds(cfg, plan):
    if plan == "per-ramp":
        return (0,) + tuple(l + 1 for l in cfg.ramp_layers), f"per-ramp ({cfg.n_ramps} splits)"
    return (0, 6, cfg.layers), "cut after layer 6 (2 splits, inner ramps exact)"


def survival(cfg, layer):
    """Expected fraction of inputs entering `layer` (0-based) under the
    workload's calibrated exit profile (e3data.configs.survival_profile)."""
    return 1.0 - sum(e for r, e in zip(cfg.ramp_layers, cfg.exit_profile) if r < layer)


def cpu_oracle_rate(cfg, tau, n_inputs, seed_offset=0):
    """The oracle as it stands (fp64 NumPy, all host cores) on a bounded sample."""
    import e3data
    import oracle
    if cfg.arch == "llama":
        return cpu_oracle_rate_llama(cfg, tau, n_inputs, seed_offset)
    W = e3data.make_weights(cfg)
    X = e3data.make_inputs(cfg, range(seed_offset, seed_offset + n_inputs))
    t0 = time.perf_counter()
    oracle.run(cfg, W, X, tau=tau, mode="fp64")
    dt = time.perf_counter() - t0
    return n_inputs / dt, dt


def cpu_oracle_rate_llama(cfg, tau, n_inputs, seed_offset=0):
    """oracle.llama on n tokens, layer by layer (weights and caches generated
    per layer outside the timed part so fp64 memory stays ~ one layer)."""
    import e3data
    from oracle import llama as olm
    from oracle.ramp import metric, passes
    X = e3data.make_inputs(cfg, range(seed_offset, seed_offset + n_inputs))[:, 0, :].astype(np.float64)
    R = {k: np.asarray(v, dtype=np.float64) for k, v in e3data.make_ramp(cfg, 0).items()}
    alive = np.arange(n_inputs)
    pos = np.full(n_inputs, cfg.ctx, dtype=np.int64)
    h, dt = X, 0.0
    for l in range(cfg.layers):
        if alive.size == 0:
            break
        W = {k: np.asarray(v, dtype=np.float64) for k, v in e3data.make_layer(cfg, l).items()}
        kv = e3data.make_kv(cfg, l, range(seed_offset, seed_offset + n_inputs), cfg.ctx + 1)
        K, V = kv[0][alive].astype(np.float64), kv[1][alive].astype(np.float64)
        t0 = time.perf_counter()
        h = olm.decode_layer(cfg, h, W, K, V, pos[alive], "fp64")
        if l in cfg.ramp_layers:
            r = cfg.ramp_layers.index(l)
            m = metric(cfg.test, olm.ramp_logits(cfg, h, R))
            ok = np.ones(alive.size, bool) if r == cfg.n_ramps - 1 else passes(cfg.test, m, tau[r])
            alive, h = alive[~ok], h[~ok]
        dt += time.perf_counter() - t0
    return n_inputs / dt, dt


def run_reference(args):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    cfg, tau = load_workload(args.config)
    cores = len(os.sched_getaffinity(0))
    n = max(1, args.cpu_inputs // 4)
    for _ in range(args.warmup):
        cpu_oracle_rate(cfg, tau, 1)
    total, t_all = 0, 0.0
    for k in range(args.steps):
        r, dt = cpu_oracle_rate(cfg, tau, n, seed_offset=k * n)
        total += n
        t_all += dt
    v = total / t_all
    unit = "tokens/s" if cfg.arch == "llama" else "inputs/s"
    print(json.dumps({
        "impl": "reference", "metric": metric_of(cfg), "value": round(v, 3),
        "unit": unit,
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1000 * t_all / args.steps, 1), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": cfg.name, "batch": cfg.batch, "seq_len": cfg.seq, "plan": "per-input (oracle)"},
        "cpu_baseline": {"value": round(v, 3), "unit": unit, "cores": cores, "kind": "oracle",
                         "sample": f"{n} inputs per step of the {cfg.name} workload, fp64 NumPy oracle"},
        "e2e": {"value": round(v, 3), "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    world, rank, local = dist_env()
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)

    import e3data
    from paper_conf_sosp_iyergdpgn24_b200 import _lib, api

    cfg, tau = load_workload(args.config)
    bounds, plan_name = plan_bounds(cfg, args.plan)
    llama = cfg.arch == "llama"
    n = args.inputs_per_gpu or (512 if llama else 8192)
    dsteps = args.decode_steps if llama else 0
    if llama:
        # weights generated layer by layer straight into HBM (13.5 GB bf16);
        # one KV cache slot per sequence (token), ctx positions pre-filled with
        # N(0, 1) on the device (same recipe as e3data.make_kv, device stream)
        layers = (e3data.make_layer(cfg, l) for l in range(cfg.layers))
        ramp = e3data.make_ramp(cfg, 0)
        kv = api.KVCache(cfg, n, cfg.ctx + max(1, dsteps), n * world, dev)
        g = torch.Generator(device=dev)
        g.manual_seed(1234 + rank)
        for t in kv.k + kv.v:
            t[:, :, :cfg.ctx].normal_(generator=g)
        kv.slot_of_id.copy_(torch.arange(n * world, device=dev, dtype=torch.int32) % n)
        model = api.DeviceModel(cfg, {"layers": layers, "ramps": [ramp] * cfg.n_ramps}, dev, kv=kv)
        if dsteps:
            embed = torch.from_numpy(e3data.make_embed(cfg)).to(torch.bfloat16).to(dev)
    else:
        W = e3data.make_weights(cfg)
        model = api.DeviceModel(cfg, W, dev)
    stream = torch.cuda.Stream(dev)
    model_bytes = sum(t.numel() * 2 for w in model.layers for t in w.values())
    kv_bytes = sum(t.numel() * 2 for t in (model.kv.k + model.kv.v)) if llama else 0
    stage_mode = args.mode == "stage" and world > 1 and not llama
    first_id = rank * n
    ids_all = None
    if stage_mode:
        # stages on different GPUs; the job is n inputs per GPU, fed into
        # split 0 by the stage-0 replicas; ids are global so every exit record
        # lands at its input's slot on the rank where the input exits
        from paper_conf_sosp_iyergdpgn24_b200 import parallel as par
        k = args.stages or min(world, 4)
        prof_path = os.path.join(ROOT, "profiles", f"r02_planner_profile_{args.config}.json")
        if not os.path.exists(prof_path):
            prof_path = os.path.join(ROOT, "profiles", f"r01_planner_profile_{args.config}.json")
        if args.planner == "dp" and os.path.exists(prof_path):
            # profile-driven DP (planner.py, NEXT-1) restricted to k stages
            from paper_conf_sosp_iyergdpgn24_b200 import planner as pln
            layout, _ = pln.plan_dp(cfg.ramp_layers, lambda l: survival(cfg, l), pln.Profile.load(prof_path),
                                    world, n_stages=min(k, world, cfg.n_ramps))
        else:
            layout = par.plan_stages(cfg.ramp_layers, lambda l: survival(cfg, l), world,
                                     n_stages=min(k, world, cfg.n_ramps))
        total = n * world
        lo, hi = par.input_share(layout, rank, total)
        comm = par.make_comm(rank, world, local)
        plan = api.make_plan(cfg, bounds, tau, lag=args.lag, placement=par.placement(layout, bounds), transport="nccl")
        pipe = api.Pipeline(model, plan, comm)
        ex = api.ExitBuffers(total, cfg.classes, cfg.n_ramps, dev)
        plan_name = f"stages {list(layout.bounds)} replicas {list(layout.replicas)} (per-ramp splits inside)"
        first_id, n_mine = lo, hi - lo
    else:
        n_mine = n
    X = e3data.make_inputs(cfg, range(first_id, first_id + n_mine))
    x_host = torch.from_numpy(X).to(torch.bfloat16).pin_memory() if n_mine else None
    del X
    x_dev = x_host.to(dev) if n_mine else None
    if stage_mode:
        ids_dev = torch.arange(first_id, first_id + n_mine, dtype=torch.int64, device=dev) if n_mine else None
        ids_host = ids_dev.cpu().pin_memory() if n_mine else None
    else:
        ids_dev = torch.arange(0, n, dtype=torch.int64, device=dev)   # local ids index the exit arrays
        ids_host = torch.arange(0, n, dtype=torch.int64).pin_memory()
        ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, dev, hidden=cfg.hidden if dsteps else 0)
        pipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau, lag=args.lag))
        if dsteps:
            x_dec = torch.empty_like(x_dev[:, 0, :])

    def barrier():
        if world > 1:
            dist.barrier()

    def step(host=False, res=None, p=None):
        p = p or pipe
        with torch.cuda.stream(stream):
            if cfg.test == "patience":   # dependent exits: per-input counters start at zero every job
                ex.state.zero_()
            if dsteps:                   # multi-step decode: every sequence restarts at position ctx
                model.kv.pos_of_slot.fill_(cfg.ctx)
                x_dec.copy_(x_dev[:, 0, :])
                return p.decode(x_dec, ids_dev, dsteps, embed, ex, stream=stream)[1]
            st = p.run(x_host if host else x_dev, ids_host if host else ids_dev, ex, stream=stream)
            if res is not None:   # D2H read of the step's result (exit records)
                res[0].copy_(ex.exit_layer, non_blocking=True)
                res[1].copy_(ex.label, non_blocking=True)
                res[2].copy_(ex.conf, non_blocking=True)
        return st

    def max_over_ranks(ms):
        if world == 1:
            return ms
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def timed(K, host=False, res=None, p=None):
        barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        stats = None
        for _ in range(K):
            stats = step(host, res, p)
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        return max_over_ranks(e0.elapsed_time(e1)), stats

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    launches0 = _lib.lib.e3_kernel_launches()
    with ClockSampler(local) as clk:
        ms, stats = timed(args.steps)
    launches = (_lib.lib.e3_kernel_launches() - launches0) // args.steps * args.steps
    clocks = clk.summary()
    total_inputs = n * world * args.steps * max(1, dsteps)    # llama: tokens
    value = total_inputs / (ms / 1000.0)
    unit = "tokens/s" if llama else "inputs/s"

    # exit histogram + invariants of the last step
    if stage_mode:
        par.reduce_exits(ex)
    el = ex.exit_layer.cpu().numpy()
    assert (el >= 0).all(), "an input did not exit"
    hist = (np.bincount(el, minlength=cfg.layers) / len(el)).round(4).tolist()
    splits = len(bounds) - 1
    valid = [int(stats.valid_rows[s]) for s in range(splits)] if stats else None
    padded = [int(stats.padded_rows[s]) for s in range(splits)] if stats else None
    batches = [int(stats.batches[s]) for s in range(splits)] if stats else None

    # e2e: host-pinned inputs through the same C-ABI call, results read back
    e2e = None
    if not args.no_e2e and not dsteps:
        cap = ex.capacity
        res = (torch.empty(cap, dtype=torch.int32).pin_memory(), torch.empty(cap, dtype=torch.int32).pin_memory(),
               torch.empty(cap, dtype=torch.float32).pin_memory())
        step(host=True, res=res)
        torch.cuda.synchronize()
        ms_e2e, _ = timed(args.steps, host=True, res=res)
        row = cfg.seq * cfg.hidden * 2
        e2e = {"value": round(total_inputs / (ms_e2e / 1000.0), 1), "unit": unit,
               "h2d_bytes_per_step": int(n * world * (row + 8)),        # the whole job's inputs + ids
               "d2h_bytes_per_step": int(cap * 12 * world)}             # every rank reads its exit records

    # stage mode: the replica mode on the same per-GPU load, as the comparison
    replica_cmp = None
    if stage_mode:
        Xr = e3data.make_inputs(cfg, range(rank * n, rank * n + n))
        xr = torch.from_numpy(Xr).to(torch.bfloat16).to(dev)
        del Xr
        idr = torch.arange(0, n, dtype=torch.int64, device=dev)
        exr = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, dev)
        rpipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau, lag=args.lag))

        def rstep():
            with torch.cuda.stream(stream):
                rpipe.run(xr, idr, exr, stream=stream)

        for _ in range(max(args.warmup, 3)):
            rstep()
        barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            rstep()
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ms_r = max_over_ranks(e0.elapsed_time(e1))
        replica_cmp = {"value": round(total_inputs / (ms_r / 1000.0), 1), "unit": "inputs/s",
                       "ms_per_step": round(ms_r / args.steps, 3), "mode": "replica (whole chain per GPU)"}
        del rpipe, xr, exr

    # per-kernel CUDA-event profile of one extra step (same stream, same launches)
    _lib.lib.e3_profile_reset()
    _lib.lib.e3_profile_enable(1)
    step()
    torch.cuda.synchronize()
    _lib.lib.e3_profile_enable(0)
    kern = {}
    import ctypes as C
    for k in range(9):
        t, f, b, c, nm = C.c_double(), C.c_double(), C.c_double(), C.c_longlong(), C.c_char_p()
        _lib.lib.e3_profile_read(k, C.byref(t), C.byref(f), C.byref(b), C.byref(c), C.byref(nm))
        kern[nm.value.decode()] = {"ms": t.value, "flops": f.value, "bytes": b.value, "launches": c.value}
    prof_ms = sum(v["ms"] for v in kern.values())
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    tf_peak = peaks.get("bf16_tflops_sustained", 1400.0)
    bw_peak = peaks.get("hbm_gbs", 6650.0)
    peak_src = "MEASURED_PEAKS.json" if peaks else "fallback (B200_PROFILING.md)"
    top = max(kern, key=lambda k: kern[k]["ms"])
    tk = kern[top]
    traffic = None
    ncu_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(ncu_path):
        nt = json.load(open(ncu_path))
        if nt.get("_workload") == cfg.name:   # the capture is of one workload's kernels
            traffic = nt.get(top)
    if tk["flops"] > 0:
        ach = tk["flops"] / (tk["ms"] / 1e3) / 1e12
        roof = {"bound": "tensor", "achieved": round(ach, 1), "peak": tf_peak, "unit": "TFLOP/s",
                "frac": round(ach / tf_peak, 4)}
    else:
        ach = tk["bytes"] / (tk["ms"] / 1e3) / 1e9
        roof = {"bound": "hbm", "achieved": round(ach, 1), "peak": bw_peak, "unit": "GB/s",
                "frac": round(ach / bw_peak, 4)}
    roof.update({"traffic": traffic, "kernel": top, "launches_per_step": tk["launches"],
                 "peak_source": peak_src + " (sustained bf16 / copy GB/s)"})
    # whole-path model: tensor work at peak + HBM work at peak vs elapsed
    f_alg = sum(v["flops"] for v in kern.values())
    b_alg = sum(v["bytes"] for v in kern.values() if v["flops"] == 0)
    ms_step = ms / args.steps
    whole = (f_alg / (tf_peak * 1e12) + b_alg / (bw_peak * 1e9)) / (ms_step / 1e3)
    per_kernel = {k: {"share": round(v["ms"] / prof_ms, 4) if prof_ms else None,
                      "achieved": (round(v["flops"] / (v["ms"] / 1e3) / 1e12, 1) if v["flops"] and v["ms"]
                                   else round(v["bytes"] / (v["ms"] / 1e3) / 1e9, 1) if v["ms"] else None),
                      "unit": "TFLOP/s" if v["flops"] else "GB/s", "launches": v["launches"]}
                  for k, v in kern.items()}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        rate, dt = cpu_oracle_rate(cfg, tau, args.cpu_inputs)
        cpu = {"value": round(rate, 3), "unit": unit, "cores": len(os.sched_getaffinity(0)),
               "kind": "oracle",
               "sample": f"{args.cpu_inputs} inputs of the {cfg.name} workload through the fp64 NumPy "
                         f"oracle ({dt:.1f} s)"}
        # the same oracle on ONE host thread (core count stated)
        from threadpoolctl import threadpool_limits
        n1 = max(1, args.cpu_inputs // 4)
        with threadpool_limits(limits=1):
            rate1, dt1 = cpu_oracle_rate(cfg, tau, n1, seed_offset=10_000)
        cpu["one_thread"] = {"value": round(rate1, 3), "unit": unit, "cores": 1,
                             "sample": f"{n1} inputs ({dt1:.1f} s)"}

    if rank == 0:
        out = {
            "metric": metric_of(cfg), "value": round(value, 1), "unit": unit, "n_gpus": world,
            "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": round(ms_step, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
            "data": "synthetic (seeded random-init weights and N(0,1) embedded inputs, e3data)",
            "config": {"workload": cfg.name, "layers": cfg.layers, "hidden": cfg.hidden, "batch": cfg.batch,
                       "seq_len": cfg.seq, "ramps": cfg.n_ramps, "test": cfg.test, "plan": plan_name,
                       "inputs_per_step_per_gpu": n,
                       "parallelism": (f"stage x{world}" if stage_mode else f"replica x{world}") if world > 1 else "1 GPU",
                       "l2": ("weights %.1f GB + KV cache %.1f GB streamed per step, >> L2" % (
                           model_bytes / 1e9, kv_bytes / 1e9) if llama else
                           "inputs larger than L2 (%.2f GB per step per GPU)" % (n * cfg.seq * cfg.hidden * 2 / 1e9))},
            "roofline": roof,
            "whole_path_roofline_frac": round(whole, 4),
            "per_kernel": per_kernel,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "replica_comparison": replica_cmp,
            "gpu_launches": int(launches),
            "clocks": clocks,
            "exit_hist": hist,
            "split_batches": batches, "split_valid_rows": valid, "split_padded_rows": padded,
            "host_waits": int(stats.host_waits) if stats else None,
            "host_launch_ms": round(stats.host_launch_ms, 2) if stats else None,
            "host_sync_ms": round(stats.host_sync_ms, 2) if stats else None,
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
