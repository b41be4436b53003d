"""Pins for oracle.numerics.bf16_rne against the bit-level definition of bf16."""
import numpy as np

from oracle.numerics import bf16_rne, store


def _all_finite_bf16():
    bits = np.arange(1 << 16, dtype=np.uint32)
    f = (bits << 16).view(np.float32)
    f = f[np.isfinite(f)]
    return f.astype(np.float64)


def test_bf16_values_are_fixed_points():
    v = _all_finite_bf16()
    v = v[np.abs(v) >= np.finfo(np.float32).tiny]   # normal range
    assert np.array_equal(bf16_rne(v), v)


def test_midpoints_round_to_even_and_neighbours_round_to_nearest():
    # consecutive positive normal bf16 values in several binades
    bits = np.arange(0x3C00, 0x4400, dtype=np.uint32)   # ~[2^-7, 2^9)
    lo = (bits << 16).view(np.float32).astype(np.float64)
    hi = ((bits + 1) << 16).view(np.float32).astype(np.float64)
    mid = 0.5 * (lo + hi)
    r = bf16_rne(mid)
    even_lo = (bits & 1) == 0
    assert np.array_equal(r, np.where(even_lo, lo, hi))
    # just off the midpoint goes to the nearer neighbour
    eps = (hi - lo) * 1e-6
    assert np.array_equal(bf16_rne(mid - eps), lo)
    assert np.array_equal(bf16_rne(mid + eps), hi)
    assert np.array_equal(bf16_rne(-(mid + eps)), -hi)


def test_random_values_within_half_ulp_and_representable():
    rng = np.random.default_rng(0)
    x = rng.standard_normal(100000) * np.exp(rng.uniform(-20, 20, 100000))
    r = bf16_rne(x)
    # representable: float32 of r is exact and its low 16 bits are zero
    r32 = r.astype(np.float32)
    assert np.array_equal(r32.astype(np.float64), r)
    assert np.all((r32.view(np.uint32) & 0xFFFF) == 0)
    # nearest: |x - r| <= half a bf16 ulp of |r|
    _, e = np.frexp(r)
    ulp = np.ldexp(1.0, e - 8)
    assert np.all(np.abs(x - r) <= 0.5 * ulp * (1 + 1e-12))


def test_store_modes():
    x = np.array([1.0 + 2 ** -10, 3.14159])
    assert np.array_equal(store(x, "fp64"), x)
    assert np.array_equal(store(x, "bf16"), bf16_rne(x))
