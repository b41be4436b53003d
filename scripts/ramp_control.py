"""Exit-wrapper ramp control on B200 (§3.4,
§5.8.6): record every ramp's metric for a calibration set on the GPU
(e3_exits.ramp_metric, thresholds that never pass), let planner.choose_ramps
pick the enabled ramps under the measured profile (r02_planner_profile_bb),
then time EE-BERT-base through the per-ramp plan and through the chosen plan
(splits at the enabled ramps, the others disabled) on the bench workload,
and report the label agreement between the two.
Writes gpurun_out/r02_ramp_control.json.
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import e3data  # noqa: E402
from paper_conf_sosp_iyergdpgn24_b200 import api, planner  # noqa: E402

dev = "cuda:0"
cfg = e3data.get("bb")
tau = e3data.tau_for(cfg)
model = api.DeviceModel(cfg, e3data.make_weights(cfg), dev)
nc = 2048
Xc = api.to_bf16(e3data.make_inputs(cfg, range(nc), seed=2), dev)
exc = api.ExitBuffers(nc, cfg.classes, cfg.n_ramps, dev, ramp_metrics=True, logits=False)
api.Pipeline(model, api.make_plan(cfg, tuple(range(13)), (0.0,) * 12)).run(
    Xc, torch.arange(nc, dtype=torch.int64, device=dev), exc)
M = exc.ramp_metric.cpu().numpy().astype(np.float64)
prof = planner.Profile.load(os.path.join(ROOT, "profiles", "r02_planner_profile_bb.json"))
en, cost, _ = planner.choose_ramps(M, tau, cfg.test, cfg.ramp_layers, prof)
all_en = tuple(range(12))
cost_all = planner.ramp_plan_cost(planner.exits_with(M, tau, cfg.test, all_en, 11), cfg.ramp_layers, all_en, prof)
n = 8192
X = api.to_bf16(e3data.make_inputs(cfg, range(n)), dev)
ids = torch.arange(n, dtype=torch.int64, device=dev)


def timed(bounds, inner, steps=10):
    pipe = api.Pipeline(model, api.make_plan(cfg, bounds, tau, inner=inner))
    ex = api.ExitBuffers(n, cfg.classes, cfg.n_ramps, dev)
    for _ in range(3):
        pipe.run(X, ids, ex)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        pipe.run(X, ids, ex)
    e1.record()
    torch.cuda.synchronize()
    return n * steps / (e0.elapsed_time(e1) / 1000.0), ex.exit_layer.cpu().numpy(), ex.label.cpu().numpy()


v_all, el_all, lab_all = timed(tuple(range(13)), "exact")
bounds = (0,) + tuple(cfg.ramp_layers[r] + 1 for r in en)
v_en, el_en, lab_en = timed(bounds, "disabled")
out = {"what": "EE-BERT-base, 8192 bench inputs per step; ramps chosen by planner.choose_ramps on 2048 calibration "
               "inputs' GPU-recorded metrics and the measured r02 profile",
       "enabled_ramps_1based": [r + 1 for r in en], "predicted_us_per_input": {"all": round(cost_all, 3),
                                                                             "chosen": round(cost, 3)},
       "inputs_per_s": {"per_ramp_all_enabled": round(v_all, 1), "chosen": round(v_en, 1),
                        "gain": round(v_en / v_all, 4)},
       "label_agreement_with_all_ramps": round(float(np.mean(lab_all == lab_en)), 4),
       "mean_exit_layer": {"all": round(float(el_all.mean() + 1), 3), "chosen": round(float(el_en.mean() + 1), 3)}}
os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
json.dump(out, open(os.path.join(ROOT, "gpurun_out", "r02_ramp_control.json"), "w"), indent=1)
print(json.dumps(out))
