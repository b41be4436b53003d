"""Whole-job parity measurement: the GPU pipeline from seeded inputs vs the
oracle, every input compared (VERDICT r01 "what to do" 1(b)).

    python tests/tools/parity_stats.py [--dtype bf16|fp32] [--configs t,tv,bb,bl,vt,tl,lm] [--out FILE]

Per config: the per-ramp plan through e3_pipeline_run on N inputs (tiny 256,
tiny-vit 200, BB 128, BL 32, VT 32, tiny-llama 90, Llama-7B shape 16 tokens
through all 32 layers), the oracle in bf16-emulate mode (decisions, R13) and
fp64 (logits, C13) on the same inputs; flips at margin > 1e-3 and the
quantiles of the max-abs logit error per input.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import e3data  # noqa: E402
import oracle  # noqa: E402
from tests import parity_util as pu  # noqa: E402

N_DEFAULT = {"tiny": 256, "tiny-vit": 200, "ee-bert-base": 128, "ee-bert-large": 32, "ee-vit-b16": 32,
             "tiny-llama": 90, "ee-llama-7b-decode": 16}


def encoder_case(api, cfg, n, dtype, modes):
    import torch
    tau = e3data.tau_for(cfg)
    W = e3data.make_weights(cfg)
    X = e3data.make_inputs(cfg, range(n))
    model = api.DeviceModel(cfg, W, "cuda:0")
    t0 = time.time()
    gpu = pu.run_gpu_pipeline(api, cfg, model, X, tau, dtype=dtype)
    out = {"gpu_s": round(time.time() - t0, 1)}
    for mode in modes:
        t0 = time.time()
        recs = oracle.run(cfg, W, X, tau=tau, mode=mode)
        out[mode] = pu.compare(gpu, recs)
        out[mode]["oracle_s"] = round(time.time() - t0, 1)
    del model
    torch.cuda.empty_cache()
    return out


def llama_case(api, cfg, n, dtype, modes):
    t0 = time.time()
    gpu, recs = pu.llama_job(api, cfg, n, dtype, modes)
    out = {"job_s": round(time.time() - t0, 1), "n_tokens": n, "positions": "ctx - (slot % 5)"}
    for mode in modes:
        out[mode] = pu.compare(gpu, recs[mode])
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dtype", default="bf16")
    ap.add_argument("--configs", default="t,tv,bb,bl,vt,tl,lm")
    ap.add_argument("--modes", default="bf16,fp64")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    from paper_conf_sosp_iyergdpgn24_b200 import api
    modes = args.modes.split(",")
    res = {"dtype": args.dtype, "margin": pu.MARGIN, "cores": len(os.sched_getaffinity(0)), "configs": {}}
    for name in args.configs.split(","):
        cfg = e3data.get(name)
        n = N_DEFAULT[cfg.name]
        t0 = time.time()
        case = llama_case if cfg.arch == "llama" else encoder_case
        r = case(api, cfg, n, args.dtype, modes)
        r["wall_s"] = round(time.time() - t0, 1)
        res["configs"][cfg.name] = r
        brief = {m: {k: r[m][k] for k in ("n", "decided", "flips", "same_layer", "logit_err")} for m in modes}
        print(cfg.name, json.dumps(brief), flush=True)
    out = args.out or os.path.join(ROOT, "gpurun_out", f"parity_{args.dtype}.json")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    for r in res["configs"].values():
        for m in modes:
            r[m].pop("logit_err_all", None)
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    print("wrote", out)


if __name__ == "__main__":
    main()
