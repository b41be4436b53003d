"""Helpers shared by the -m gpu parity tests."""
import numpy as np
import pytest
import torch

requires_cuda = pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")
DEV = "cuda:0"


def bf16_tensor(a, device=DEV):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(device=device, dtype=torch.bfloat16)


def to64(t):
    return t.detach().float().cpu().numpy().astype(np.float64)


def rand_bf16(rng, shape, scale=1.0):
    from e3data import bf16_round
    return bf16_round(rng.standard_normal(shape).astype(np.float32) * np.float32(scale))


def bf16_ulp(x):
    """Spacing of bf16 values at |x| (2^(e-7) for |x| in [2^e, 2^(e+1)))."""
    x = np.maximum(np.abs(x), 2.0 ** -100)
    e = np.floor(np.log2(x))
    return 2.0 ** (e - 7)
