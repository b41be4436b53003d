"""On-device profile for the split planner (paper_conf_sosp_iyergdpgn24_b200/planner.py;
SURVEY.md §8(f) NEXT-1): graph-timed split runs of EVERY layer l (split
[l, l+1), its ramp at l when the layer has one) at the constant batch B, with
and without the ramp + compaction kernels (E3_SKIP), give t_layer[l] and
t_ramp; t_tx: the inter-stage message of one batch (header | B ids | B rows,
e3.h) measured as a device-to-device copy on this GPU (what the LOOPBACK
transport does) and, for NCCL over NVLink, the same bytes at an assumed
675 GB/s (900 GB/s per direction x 0.75; one GPU here, not measured).
Writes gpurun_out/r02_planner_profile_<cfg>.json (committed under profiles/).

    python scripts/profile_layers.py [config]
"""
import json
import os
import subprocess
import sys

sys.path.insert(0, ".")


def graph_time(cfg_name, begin, end, n=20):
    import torch
    import e3data
    from paper_conf_sosp_iyergdpgn24_b200 import api
    dev = "cuda:0"
    cfg = e3data.get(cfg_name)
    tau = e3data.tau_for(cfg)
    model = api.DeviceModel(cfg, e3data.make_weights(cfg), dev)
    B = cfg.batch
    X = api.to_bf16(e3data.make_inputs(cfg, range(B)), dev)
    ids = torch.arange(B, dtype=torch.int64, device=dev)
    split = api.Split(model, api.split_desc(cfg, begin, end, tau))
    x_out, id_out = torch.empty_like(X), torch.empty_like(ids)
    n_surv = torch.zeros(1, dtype=torch.int32, device=dev)
    ex = api.ExitBuffers(B, cfg.classes, cfg.n_ramps, dev)
    for _ in range(3):
        split.run(X, ids, x_out, id_out, n_surv, ex)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            for _ in range(n):
                split.run(X, ids, x_out, id_out, n_surv, ex)
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1000.0, cfg


def copy_time_us(nbytes, n=50):
    import torch
    a = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    b = torch.empty_like(a)
    for _ in range(3):
        b.copy_(a)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        b.copy_(a)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1000.0


if __name__ == "__main__":
    name = sys.argv[1] if len(sys.argv) > 1 else "bb"
    import e3data
    cfg = e3data.get(name)
    # splits [l, l+1) need a ramp at l: per-layer timing for configs with a ramp after every layer
    bounds = [(l, l + 1) for l in range(cfg.layers)] if len(cfg.ramp_layers) == cfg.layers else \
        [(0, cfg.ramp_layers[0] + 1)]
    if os.environ.get("_E3_PROFILE_CHILD"):
        print(" ".join("%.3f" % graph_time(name, b, e)[0] for b, e in bounds))
        sys.exit(0)
    env = dict(os.environ, _E3_PROFILE_CHILD="1")
    run = lambda e: [float(v) for v in subprocess.run([sys.executable, __file__, name], env=e, capture_output=True,
                                                      text=True, check=True).stdout.split()]
    t_full = run(env)
    env["E3_SKIP"] = str(64 + 128)   # ramp and compaction kernels left out
    t_lay = run(env)
    nl = [e - b for b, e in bounds]
    t_layer = [t_lay[i] / nl[i] for i in range(len(bounds))]
    if len(t_layer) < cfg.layers:
        t_layer = t_layer * cfg.layers
    t_ramp = sum(f - l for f, l in zip(t_full, t_lay)) / len(bounds)
    B = cfg.batch
    msg = 16 + (B * 8 + 15) // 16 * 16 + B * cfg.seq * cfg.hidden * 2
    t_copy = copy_time_us(msg)
    tx_nvlink = msg / 675e9 * 1e6
    out = {"config": cfg.name, "batch": B, "t_layer_us": [round(t, 2) for t in t_layer],
           "t_ramp_us": round(t_ramp, 2), "t_tx_us": round(tx_nvlink, 2),
           "t_tx_loopback_measured_us": round(t_copy, 2), "message_bytes": msg,
           "how": "graph-timed split runs [l, l+1) at B (20 per graph): t_layer[l] = time with "
                  "E3_SKIP=ramp|compaction, t_ramp = mean(full - that); t_tx_loopback = measured D2D copy of "
                  "one message (the LOOPBACK transport); t_tx = the message at an assumed 675 GB/s NVLink "
                  "(NCCL; one GPU here, not measured)"}
    os.makedirs("gpurun_out", exist_ok=True)
    path = f"gpurun_out/r02_planner_profile_{name}.json"
    json.dump(out, open(path, "w"), indent=1)
    print(json.dumps(out))
