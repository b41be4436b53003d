"""bf16 storage-point rounding for the oracle's ``bf16`` (emulate) mode.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper never states precision.  The GPU
path stores activations in bf16 at the points listed in DESIGN.md
"Rounding contract"; the oracle's ``bf16`` mode rounds an exact float64 value
to the nearest bf16 (ties to even) at exactly those points and keeps every
other operation in float64.

Pins (tests/test_oracle_numerics.py): exhaustive agreement with the bit-level
definition of bf16 on every bf16 value and every midpoint between neighbours
in a range of binades; ties go to the even mantissa.
"""
from __future__ import annotations

import numpy as np


def bf16_rne(x):
    """Nearest bf16 value of float64 ``x`` (ties to even), as float64.

    bf16 keeps 8 significant bits (7 stored); a float64 keeps 53 (52 stored),
    so RNE drops the low 45 bits of the float64 encoding: add 2^44 - 1 plus the
    lowest kept bit (ties to even), then clear the 45 bits.  A carry out of the
    significand correctly bumps the exponent.  Valid for normal finite values.
    """
    x = np.asarray(x, dtype=np.float64)
    u = np.ascontiguousarray(x).view(np.uint64)
    u = (u + np.uint64((1 << 44) - 1) + ((u >> np.uint64(45)) & np.uint64(1))) \
        & np.uint64(~((1 << 45) - 1) & 0xFFFFFFFFFFFFFFFF)
    return u.view(np.float64).reshape(x.shape)


def store(x, mode: str):
    """Round at a storage point: bf16 RNE in ``bf16`` mode, identity in ``fp64``."""
    if mode == "bf16":
        return bf16_rne(x)
    if mode == "fp64":
        return np.asarray(x, dtype=np.float64)
    raise ValueError(mode)
