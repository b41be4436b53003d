"""Goodput of the split path under a time-varying open-loop workload, with the
online batch-profile estimator and the re-planner in the loop (SURVEY §8(f)
NEXT-3; §3.1, §3.3, §5.7; paper_conf_sosp_iyergdpgn24_b200/online.py).

Virtual-time serving simulation whose service times are MEASURED: every
dispatched batch of requests really runs through e3_pipeline_run on the GPU
(EE-BERT-base, per-ramp splits) and the clock advances by its CUDA-event time.
  * arrivals: Poisson with a time-varying rate (a daily-cycle-like sinusoid
    plus bursts), compressed windows of --window seconds (the paper's 2 min);
  * hardness drift: each request is drawn from an "easy" pool (inputs that
    exit at ramps 1-3) or a "hard" pool (ramps >= 9), the hard fraction
    drifting across the windows, so the per-ramp batch profile moves;
  * dispatch: online.SloBatcher (target = --batch requests, SLO 100 ms, 20 %
    slack, late requests dropped);
  * after each window the estimator observes the per-ramp exit counts of the
    completed requests and forecasts the next window; the re-planner re-runs
    planner.plan_dp for --plan-gpus GPUs when the forecast moved.
Writes gpurun_out/r02_online_goodput.json.

    python scripts/online_goodput.py [--windows 10] [--window 1.0] [--rate 40000]
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api, online, planner  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--windows", type=int, default=10)
    ap.add_argument("--window", type=float, default=1.0, help="virtual seconds per window")
    ap.add_argument("--rate", type=float, default=40000.0, help="mean arrivals per second")
    ap.add_argument("--batch", type=int, default=1024, help="dispatch target (requests)")
    ap.add_argument("--slo", type=float, default=0.100)
    ap.add_argument("--plan-gpus", type=int, default=8)
    ap.add_argument("--pool", type=int, default=4096)
    args = ap.parse_args()
    dev = "cuda:0"
    cfg = e3data.get("bb")
    tau = e3data.tau_for(cfg)
    model = api.DeviceModel(cfg, e3data.make_weights(cfg), dev)
    pipe = api.Pipeline(model, api.make_plan(cfg, (0,) + tuple(l + 1 for l in cfg.ramp_layers), tau))
    # pools: calibration-seed inputs classified by where they exit
    Xp = api.to_bf16(e3data.make_inputs(cfg, range(args.pool), seed=2), dev)
    exp = api.ExitBuffers(args.pool, cfg.classes, cfg.n_ramps, dev, logits=False)
    pipe.run(Xp, torch.arange(args.pool, dtype=torch.int64, device=dev), exp)
    el = exp.exit_layer.cpu().numpy()
    easy = np.nonzero(el <= 2)[0]
    hard = np.nonzero(el >= 8)[0]
    rng = np.random.default_rng(7)
    prof = planner.Profile.load(os.path.join(ROOT, "profiles", "r02_planner_profile_bb.json")) \
        if os.path.exists(os.path.join(ROOT, "profiles", "r02_planner_profile_bb.json")) else \
        planner.Profile.load(os.path.join(ROOT, "profiles", "r01_planner_profile_bb.json"))
    est = online.BatchProfileEstimator(cfg.n_ramps, p=2, d=1)
    # two stages forced (with free transfers pure replication is always optimal on identical GPUs,
    # so the cut position is what the drifting profile moves)
    rp = online.Replanner(cfg.ramp_layers, lambda s: planner.plan_dp(cfg.ramp_layers, s, prof, args.plan_gpus,
                                                                       n_stages=2)[0])
    batcher = online.SloBatcher(args.batch, args.slo, 0.2)
    xbuf = torch.empty((args.batch, cfg.seq, cfg.hidden), dtype=torch.bfloat16, device=dev)
    ex = api.ExitBuffers(args.batch, cfg.classes, cfg.n_ramps, dev, logits=False)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    per_req_us = 17.0e-6                              # service-time model for the dispatcher, refined online
    clock, gpu_free = 0.0, 0.0
    windows = []
    rid = 0
    t_wall = time.time()
    for w in range(args.windows):
        hard_frac = 0.2 + 0.6 * w / max(1, args.windows - 1)
        t0, t1 = w * args.window, (w + 1) * args.window
        # arrivals of this window (time-varying Poisson + a burst)
        times = []
        t = t0
        while True:
            lam = args.rate * (1.0 + 0.4 * np.sin(2 * np.pi * t / (3 * args.window)))
            if t0 + 0.45 * args.window < t < t0 + 0.5 * args.window:
                lam *= 2.5                              # burst
            t += rng.exponential(1.0 / lam)
            if t >= t1:
                break
            times.append(t)
        kinds = rng.random(len(times)) < hard_frac
        src = np.where(kinds, rng.choice(hard, len(times)), rng.choice(easy, len(times)))
        reqs = [online.Request(rid + i, a, a + args.slo) for i, a in enumerate(times)]
        src_of = {rid + i: int(src[i]) for i in range(len(times))}
        dl = {r.rid: r.deadline for r in reqs}
        rid += len(times)
        done_ok = done_late = dropped = 0
        counts = np.zeros(cfg.n_ramps, dtype=np.int64)
        served = 0
        i = 0
        clock = max(clock, t0)
        while i < len(reqs) or batcher.queue:
            # admit every arrival up to the current clock
            while i < len(reqs) and reqs[i].arrival <= clock:
                batcher.add(reqs[i])
                i += 1
            est_service = per_req_us * min(len(batcher.queue), args.batch) + 2e-3
            d = batcher.poll(max(clock, gpu_free), est_service) if clock >= gpu_free else None
            if d is None:
                nxt = reqs[i].arrival if i < len(reqs) else float("inf")
                # next event: an arrival, the GPU freeing up, or the oldest request's dispatch point
                cand = [nxt]
                if clock < gpu_free:
                    cand.append(gpu_free)
                if batcher.queue:
                    oldest = batcher.queue[0]
                    cand.append(max(clock + 1e-6, oldest.deadline - 0.2 * args.slo - est_service))
                clock = min(cand)
                if clock == float("inf"):
                    break
                continue
            dropped += len(d.dropped)
            if d.rids:
                n = len(d.rids)
                idx = torch.tensor([src_of[r] for r in d.rids], dtype=torch.int64, device=dev)
                torch.index_select(Xp, 0, idx, out=xbuf[:n])
                ex.reset()
                ev0.record()
                pipe.run(xbuf[:n], torch.arange(n, dtype=torch.int64, device=dev), ex)
                ev1.record()
                torch.cuda.synchronize()
                svc = ev0.elapsed_time(ev1) / 1000.0
                per_req_us = 0.8 * per_req_us + 0.2 * (svc / n)
                finish = max(clock, gpu_free) + svc
                gpu_free = finish
                e = ex.exit_layer[:n].cpu().numpy()
                counts += np.bincount(e, minlength=cfg.n_ramps)[:cfg.n_ramps]
                served += n
                ok = sum(1 for r in d.rids if finish <= dl[r])
                done_ok += ok
                done_late += n - ok
            clock = max(clock, gpu_free if d.rids else clock)
        fc_before = est.forecast() if est.windows else None
        obs = est.observe(counts, max(served, 1))
        fc = est.forecast()
        replanned = rp.update(fc)
        windows.append({
            "window": w, "hard_fraction": round(hard_frac, 3), "arrivals": len(reqs),
            "goodput_rps": round(done_ok / args.window, 1), "late": done_late, "dropped": dropped,
            "observed_profile": [round(float(v), 4) for v in obs],
            "forecast_error_max": None if fc_before is None else round(float(np.max(np.abs(fc_before - obs))), 4),
            "forecast_next": [round(float(v), 4) for v in fc], "replanned": replanned,
            "plan": {"bounds": list(rp.plan.bounds), "replicas": list(rp.plan.replicas)},
        })
        print(json.dumps({k: windows[-1][k] for k in ("window", "hard_fraction", "arrivals", "goodput_rps", "late",
                                                     "dropped", "forecast_error_max", "replanned", "plan")}),
              flush=True)
    total = sum(w["arrivals"] for w in windows)
    good = sum(w["goodput_rps"] * args.window for w in windows)
    out = {"what": "virtual-time open-loop serving of EE-BERT-base through e3_pipeline_run (per-ramp splits, B = 64) "
                   "on one B200; service times measured by CUDA events; SLO 100 ms, 20 % slack, dispatch target "
                   f"{args.batch}; estimator ARIMA(2,1,0) per ramp; re-plan for {args.plan_gpus} GPUs with planner.plan_dp",
           "windows": windows, "total_arrivals": total, "goodput_rps": round(good / (args.windows * args.window), 1),
           "drop_or_late_fraction": round(1 - good / max(total, 1), 4), "replans": rp.replans,
           "wall_s": round(time.time() - t_wall, 1)}
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "r02_online_goodput.json"), "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps({k: out[k] for k in ("total_arrivals", "goodput_rps", "drop_or_late_fraction", "replans")}))


if __name__ == "__main__":
    main()
