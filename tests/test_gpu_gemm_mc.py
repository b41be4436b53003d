"""-m gpu: the layer GEMM's optional cluster multicast modes (E3_GEMM_MC=1: A
shared by two N-neighbour pair tiles, 2: W shared by two M-neighbour pair
tiles; gemm_tc.cu) give the unicast kernel's output bit for bit -- a tile's
MMAs and epilogue are the same, only who fetches the operand boxes changes --
on BB shapes and on ragged M (an odd number of 256-row blocks: the second
pair of the last cluster unit computes rows past M, which the TMA store
clips).  The library reads E3_GEMM_MC once per process, so every setting runs
in its own interpreter (scripts/gemm_mc_check.py's child mode)."""
import os
import subprocess
import sys

import pytest
import torch

from tests.gpu_util import requires_cuda

pytestmark = [pytest.mark.gpu, requires_cuda]

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(tmp_path, M, N, K, epi, bn, mc):
    out = str(tmp_path / f"c_{mc}.pt")
    env = dict(os.environ, _GEMM_MC_CHILD="1", E3_GEMM_MC=str(mc), E3_GEMM_BN=str(bn))
    r = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "gemm_mc_check.py"), str(M), str(N), str(K),
                        epi, out], env=env, capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    t_us, err = (float(v) for v in r.stdout.split()[-2:])
    return torch.load(out), err


@pytest.mark.parametrize("M,N,K,epi,bn", [(8192, 3072, 768, "bias_gelu", 192), (8192, 768, 3072, "bias_resid", 384),
                                          (700, 768, 768, "bias", 128), (1000, 2304, 768, "bias", 256)])
def test_gemm_multicast_modes_bitwise_equal_unicast(tmp_path, M, N, K, epi, bn):
    base, err0 = _run(tmp_path, M, N, K, epi, bn, 0)
    assert err0 < 0.05                      # vs the torch fp32 reference (bf16 output rounding)
    for mc in (1, 2):
        got, _ = _run(tmp_path, M, N, K, epi, bn, mc)
        assert torch.equal(got, base), mc
