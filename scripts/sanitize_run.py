"""Tiny pipelines for compute-sanitizer (memcheck / racecheck / synccheck):
tiny BERT, tiny ViT and tiny LLaMA through e3_pipeline_run (bf16 and FP32),
and a 2-rank LOOPBACK stage pipeline.  Exits non-zero on any E3 error.

    compute-sanitizer --tool memcheck python scripts/sanitize_run.py
"""
import os
import sys
import threading

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402

DEV = "cuda:0"


def enc(name, dtype, n=96):
    cfg = e3data.get(name)
    model = api.DeviceModel(cfg, e3data.make_weights(cfg), DEV)
    X = torch.from_numpy(e3data.make_inputs(cfg, range(n))).to(DEV)
    X = X.to(torch.bfloat16) if dtype == "bf16" else X
    ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV)
    api.Pipeline(model, api.make_plan(cfg, (0,) + tuple(l + 1 for l in cfg.ramp_layers), cfg.tau, dtype=dtype)).run(
        X, torch.arange(n, dtype=torch.int64, device=DEV), ex)
    torch.cuda.synchronize()
    assert int(ex.n_exit.item()) == n
    print(name, dtype, "ok", np.bincount(ex.exit_layer.cpu().numpy(), minlength=cfg.layers).tolist(), flush=True)


def llama(dtype, n=40):
    from tests import parity_util as pu
    cfg = e3data.get("tiny-llama")
    gpu, _ = pu.llama_job(api, cfg, n, dtype, ())
    print("tiny-llama", dtype, "ok", np.bincount(gpu["exit_layer"], minlength=cfg.layers).tolist(), flush=True)


def loopback(n=96):
    cfg = e3data.get("tiny")
    model = api.DeviceModel(cfg, e3data.make_weights(cfg), DEV)
    X = torch.from_numpy(e3data.make_inputs(cfg, range(n))).to(torch.bfloat16).to(DEV)
    ids = torch.arange(n, dtype=torch.int64, device=DEV)
    comms = api.Comm.loopback(2, 0)
    pipes = [api.Pipeline(model, api.make_plan(cfg, (0, 2, 4), cfg.tau, placement=[[0], [1]],
                                               transport="loopback"), comms[r]) for r in range(2)]
    exs = [api.ExitBuffers(n, cfg.classes, cfg.n_ramps, DEV) for _ in range(2)]
    errs = []

    def work(r):
        try:
            pipes[r].run(X if r == 0 else None, ids if r == 0 else None, exs[r], stream=torch.cuda.Stream(DEV))
            torch.cuda.synchronize()
        except Exception as e:
            errs.append(e)

    th = [threading.Thread(target=work, args=(r,)) for r in range(2)]
    [t.start() for t in th]
    [t.join() for t in th]
    assert not errs, errs
    assert int(exs[0].n_exit.item()) + int(exs[1].n_exit.item()) == n
    print("loopback 2-stage ok", flush=True)


if __name__ == "__main__":
    which = sys.argv[1:] or ["tiny", "tiny-vit", "llama", "fp32", "loopback"]
    if "tiny" in which:
        enc("tiny", "bf16")
    if "tiny-vit" in which:
        enc("tiny-vit", "bf16")
    if "llama" in which:
        llama("bf16")
    if "fp32" in which:
        enc("tiny", "fp32")
        enc("tiny-vit", "fp32")
        llama("fp32")
    if "loopback" in which:
        loopback()
    print("SANITIZE_RUN_DONE")
