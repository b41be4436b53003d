"""Whole-job parity helpers (GPU pipeline from seeded inputs vs the oracle).

Shared by the -m gpu tests (tests/test_gpu_e2e.py) and the measurement
script tests/tools/parity_stats.py that writes profiles/r02_parity_*.json.
Nothing here computes the method: the GPU side goes through the C ABI
(paper_conf_sosp_iyergdpgn24_b200.api), the expected side through oracle/.
"""
from __future__ import annotations

import numpy as np

import e3data

MARGIN = 1e-3          # north_star: decisions exact where the margin exceeds 1e-3


def run_gpu_pipeline(api, cfg, model, X, tau, bounds=None, dtype="bf16", inner="exact", dev="cuda:0"):
    """Every input of X through e3_pipeline_run; returns the exit records as
    numpy arrays indexed by input position."""
    import torch
    from oracle.pipeline_sim import Plan
    N = X.shape[0]
    bounds = Plan.per_ramp(cfg.ramp_layers).bounds if bounds is None else bounds
    ex = api.ExitBuffers(N, cfg.classes, cfg.n_ramps, dev)
    pipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau, inner=inner, dtype=dtype))
    x = torch.from_numpy(np.ascontiguousarray(X, dtype=np.float32)).to(dev)
    x = x.to(torch.bfloat16) if dtype == "bf16" else x
    pipe.run(x, torch.arange(N, dtype=torch.int64, device=dev), ex)
    torch.cuda.synchronize()
    assert int(ex.n_exit.item()) == N, "every input exits exactly once"
    return {"exit_layer": ex.exit_layer.cpu().numpy(), "label": ex.label.cpu().numpy(),
            "conf": ex.conf.cpu().numpy().astype(np.float64),
            "logits": ex.logits.cpu().numpy().astype(np.float64)}


def compare(gpu, recs, margin=MARGIN):
    """GPU exit records vs oracle records (same inputs, same order).

    decisions: exit layer equal wherever the oracle's margin at every ramp the
    input reached exceeds `margin` (C12/C21); `flips` counts violations.
    logits / metric: absolute error where both exited at the same layer.
    labels: compared where the oracle's top-2 logit gap exceeds 2x the logit
    error of that input (otherwise both labels are correct, C21)."""
    el = gpu["exit_layer"]
    n = len(recs)
    decided = flips = same_layer = label_bad = 0
    errs, merrs, flip_ids = [], [], []
    for i, r in enumerate(recs):
        if r.margin > margin:
            decided += 1
            if el[i] != r.exit_layer:
                flips += 1
                flip_ids.append(i)
        if el[i] == r.exit_layer:
            same_layer += 1
            e = float(np.max(np.abs(gpu["logits"][i] - r.logits)))
            errs.append(e)
            merrs.append(abs(float(gpu["conf"][i]) - r.metric))
            top2 = np.sort(r.logits)[-2:]
            if top2[1] - top2[0] > 2 * e and gpu["label"][i] != r.label:
                label_bad += 1
    q = (lambda a, p: float(np.quantile(a, p)) if len(a) else None)
    return {"n": n, "decided": decided, "flips": flips, "flip_ids": flip_ids[:20],
            "same_layer": same_layer, "label_mismatch": label_bad,
            "logit_err": {"p50": q(errs, .5), "p90": q(errs, .9), "p99": q(errs, .99),
                          "max": max(errs) if errs else None},
            "logit_err_all": errs,
            "metric_err_max": max(merrs) if merrs else None}


class LazyLayers:
    """weights["layers"] for the 7B shape: generated per access, never cached
    (32 layers x 0.8 GB would not fit the oracle's memory budget)."""

    def __init__(self, cfg, seed=0):
        self.cfg, self.seed = cfg, seed

    def __getitem__(self, l):
        return e3data.make_layer(self.cfg, l, self.seed)

    def __len__(self):
        return self.cfg.layers


class LazyKV:
    """kv[l] for oracle.llama: the pre-filled cache of the tokens' slots at
    layer l, regenerated per access from e3data.make_kv."""

    def __init__(self, cfg, slots, max_ctx):
        self.cfg, self.slots, self.max_ctx = cfg, list(slots), max_ctx

    def __getitem__(self, l):
        return e3data.make_kv(self.cfg, l, self.slots, self.max_ctx).astype(np.float64)


def llama_job(api, cfg, n, dtype, modes=("bf16",), dev="cuda:0"):
    """The decode step of n tokens through the whole calibrated per-ramp chain
    (Llama-7B shape: 4 splits of 8 layers): GPU records and, per oracle mode,
    oracle records.  Token i sits in KV slot i at position ctx - (i % 5); the
    pre-filled caches come from e3data.make_kv (the same values on both sides,
    fp32 caches for FP32 mode)."""
    import torch
    from oracle import llama as olm
    tau = e3data.tau_for(cfg)
    max_ctx = cfg.ctx + 1
    slot_of = {i: i for i in range(n)}
    pos_of = {s: cfg.ctx - (s % 5) for s in range(n)}
    cache = api.KVCache(cfg, n, max_ctx, n, dev, dtype=dtype)
    for l in range(cfg.layers):
        k, v = e3data.make_kv(cfg, l, range(n), max_ctx)
        cache.k[l].copy_(torch.from_numpy(k).to(cache.k[l].dtype))
        cache.v[l].copy_(torch.from_numpy(v).to(cache.v[l].dtype))
    cache.slot_of_id.copy_(torch.arange(n, dtype=torch.int32))
    cache.pos_of_slot.copy_(torch.tensor([pos_of[s] for s in range(n)], dtype=torch.int32))
    ramp = e3data.make_ramp(cfg, 0)
    lazy = cfg.layers > 8
    layers = LazyLayers(cfg) if lazy else [e3data.make_layer(cfg, l) for l in range(cfg.layers)]
    W = {"layers": layers, "ramps": [ramp] * cfg.n_ramps}
    model = api.DeviceModel(cfg, {"layers": (layers[l] for l in range(cfg.layers)) if lazy else layers,
                                  "ramps": W["ramps"]}, dev, kv=cache)
    X = e3data.make_inputs(cfg, range(n), seed=5)
    gpu = run_gpu_pipeline(api, cfg, model, X, tau, dtype=dtype, dev=dev)
    del model, cache
    torch.cuda.empty_cache()
    recs = {}
    for mode in modes:
        kv = LazyKV(cfg, range(n), max_ctx)
        recs[mode] = olm.run(cfg, W, X[:, 0, :], list(range(n)), kv, slot_of, pos_of, tau=tau, mode=mode)
    return gpu, recs
