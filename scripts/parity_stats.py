"""Whole-job parity measurement: the GPU pipeline from seeded inputs vs the
oracle, every input compared (VERDICT r01 "what to do" 1(b)).

    python scripts/parity_stats.py [--dtype bf16|fp32] [--configs t,tv,bb,bl,vt,tl,lm] [--out FILE]

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

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
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
    import torch
    from oracle import llama as olm
    tau = e3data.tau_for(cfg)
    max_ctx = cfg.ctx + 1
    slot_of = {i: i for i in range(n)}
    pos_of = {s: cfg.ctx - (s % 5) for s in range(n)}
    cache = api.KVCache(cfg, n, max_ctx, n, "cuda:0")
    for l in range(cfg.layers):
        k, v = e3data.make_kv(cfg, l, range(n), max_ctx)
        cache.k[l].copy_(torch.from_numpy(k).to(torch.bfloat16))
        cache.v[l].copy_(torch.from_numpy(v).to(torch.bfloat16))
    cache.slot_of_id.copy_(torch.arange(n, dtype=torch.int32))
    cache.pos_of_slot.copy_(torch.tensor([pos_of[s] for s in range(n)], dtype=torch.int32))
    ramp = e3data.make_ramp(cfg, 0)
    lazy = cfg.layers > 8
    layers = pu.LazyLayers(cfg) if lazy else [e3data.make_layer(cfg, l) for l in range(cfg.layers)]
    W = {"layers": layers, "ramps": [ramp] * cfg.n_ramps}
    model = api.DeviceModel(cfg, {"layers": (layers[l] for l in range(cfg.layers)) if lazy else layers,
                                  "ramps": W["ramps"]}, "cuda:0", kv=cache)
    X = e3data.make_inputs(cfg, range(n), seed=5)
    t0 = time.time()
    gpu = pu.run_gpu_pipeline(api, cfg, model, X, tau, dtype=dtype)
    out = {"gpu_s": round(time.time() - t0, 1), "n_tokens": n, "positions": "ctx - (slot % 5)"}
    del model, cache
    torch.cuda.empty_cache()
    for mode in modes:
        t0 = time.time()
        kv = pu.LazyKV(cfg, range(n), max_ctx)
        recs = olm.run(cfg, W, X[:, 0, :], list(range(n)), kv, slot_of, pos_of, tau=tau, mode=mode)
        out[mode] = pu.compare(gpu, recs)
        out[mode]["oracle_s"] = round(time.time() - t0, 1)
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
