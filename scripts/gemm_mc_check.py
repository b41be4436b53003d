"""Layer-GEMM tile / multicast variants: each (E3_GEMM_BN, E3_GEMM_MC) setting
runs in its own process (the library reads them once); the outputs must be
bitwise equal to the unicast kernel's and close to a torch fp32 reference,
and the graph-timed duration is printed.
python scripts/gemm_mc_check.py M,N,K,epi[,bn] ..."""
import os
import subprocess
import sys

import torch

sys.path.insert(0, ".")

if os.environ.get("_GEMM_MC_CHILD"):
    from paper_conf_sosp_iyergdpgn24_b200 import api  # noqa: E402
    from gemm_sweep_util import timeit  # noqa: E402
    M, N, K, epi = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
    g = torch.Generator(device="cuda").manual_seed(1)
    dev = "cuda:0"
    A = torch.randn(M, K, device=dev, generator=g).to(torch.bfloat16)
    W = (torch.randn(N, K, device=dev, generator=g) * K ** -0.5).to(torch.bfloat16)
    bias = torch.randn(N, device=dev, generator=g).to(torch.bfloat16)
    R = torch.randn(M, N, device=dev, generator=g).to(torch.bfloat16)
    C = torch.full((M, N), float("nan"), device=dev, dtype=torch.bfloat16)
    run = lambda: api.ops.gemm(A, W, bias, epi, resid=R if epi == "bias_resid" else None, out=C)  # noqa: E731
    run()
    torch.cuda.synchronize()
    ref = A.float() @ W.float().t() + bias.float()
    if epi == "bias_gelu":
        ref = torch.nn.functional.gelu(ref)
    if epi == "bias_resid":
        ref = ref + R.float()
    err = (C.float() - ref).abs().max().item()
    torch.save(C.cpu(), sys.argv[5])
    t = timeit(run)
    print(f"{t:.2f} {err:.4f}")
    sys.exit(0)

os.makedirs("gpurun_out", exist_ok=True)
args = sys.argv[1:]
libs = [None]
if args and args[0].startswith("--libs="):   # A/B of library builds (scripts/build_variant.py), unicast only
    libs = args[0][len("--libs="):].split(",")
    args = args[1:]
for case in args:
    f = case.split(",")
    M, N, K, epi = int(f[0]), int(f[1]), int(f[2]), f[3]
    bns = [int(f[4])] if len(f) > 4 else [0]
    base = None
    for bn in bns:
        for mc, lib in ([(0, x) for x in libs] if libs[0] else [(m, None) for m in (0, 1, 2)]):
            env = dict(os.environ, _GEMM_MC_CHILD="1", E3_GEMM_MC=str(mc))
            if lib:
                env["E3_LIB_PATH"] = os.path.abspath(lib)
            if bn:
                env["E3_GEMM_BN"] = str(bn)
            out = f"gpurun_out/_mc_{mc}.pt"
            r = subprocess.run([sys.executable, __file__, str(M), str(N), str(K), epi, out], env=env,
                               capture_output=True, text=True, timeout=300)
            if r.returncode != 0:
                print(f"{case} mc={mc}: FAILED rc={r.returncode} {r.stderr[-600:]}")
                continue
            t, err = r.stdout.split()[-2:]
            C = torch.load(out)
            same = "base" if base is None else ("bitwise-equal" if torch.equal(C, base) else "DIFFERENT")
            if base is None:
                base = C
            fl = 2 * M * N * K
            print(f"M={M} N={N} K={K} {epi:10s} bn={bn or 'auto'} mc={mc}: {float(t):7.2f} us "
                  f"({fl / float(t) / 1e6:6.0f} TF/s) max|err| {err} {same} {lib or ''}", flush=True)
