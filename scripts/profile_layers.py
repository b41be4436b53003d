"""On-device profile for the split planner (paper_conf_sosp_iyergdpgn24_b200/planner.py;
SURVEY.md §8(f) NEXT-1): graph-timed split runs of one layer at the constant
batch B, with and without the ramp + compaction kernels (E3_SKIP), give
t_layer and t_ramp; t_tx is the survivors' bytes of one batch over NVLink at
an assumed 675 GB/s (900 GB/s per direction x 0.75; one GPU here, so not
measured).  Writes gpurun_out/r01_planner_profile_<cfg>.json (committed under profiles/).

    python scripts/profile_layers.py [config]
"""
import json
import os
import subprocess
import sys

sys.path.insert(0, ".")


def graph_time(cfg_name, nl, n=20):
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
    split = api.Split(model, api.split_desc(cfg, 0, nl, tau))
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


if __name__ == "__main__":
    name = sys.argv[1] if len(sys.argv) > 1 else "bb"
    import e3data
    cfg = e3data.get(name)
    nl = cfg.ramp_layers[0] + 1          # one split = the layers up to the first ramp
    if os.environ.get("_E3_PROFILE_CHILD"):
        t, _ = graph_time(name, nl)
        print(t)
        sys.exit(0)
    env = dict(os.environ, _E3_PROFILE_CHILD="1")
    t_full = float(subprocess.run([sys.executable, __file__, name], env=env, capture_output=True, text=True,
                                  check=True).stdout.split()[-1])
    env["E3_SKIP"] = str(64 + 128)   # ramp and compaction kernels left out
    t_layer = float(subprocess.run([sys.executable, __file__, name], env=env, capture_output=True, text=True,
                                   check=True).stdout.split()[-1])
    tx = cfg.batch * cfg.seq * cfg.hidden * 2 / 675e9 * 1e6
    t_layer /= nl
    out = {"config": cfg.name, "batch": cfg.batch, "t_layer_us": [round(t_layer, 2)] * cfg.layers,
           "t_ramp_us": round(t_full - t_layer * nl, 2), "t_tx_us": round(tx, 2),
           "how": f"graph-timed split runs of the {nl} layer(s) up to the first ramp at B (20 per graph): "
                  "t_layer = time with E3_SKIP=ramp|compaction / layers, t_ramp = full - that; "
                  "t_tx = B*S*H*2 bytes at an assumed 675 GB/s NVLink (not measured)"}
    os.makedirs("gpurun_out", exist_ok=True)
    path = f"gpurun_out/r01_planner_profile_{name}.json"
    json.dump(out, open(path, "w"), indent=1)
    print(json.dumps(out))
