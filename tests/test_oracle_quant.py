"""Pins for the oracle's conservative rounding (readings R5-R9; Alg. 1).

Definition under test: k(x) = clamp(floor(x * RN(1/eps)), int64) with the
product taken exactly, NaN -> 0.  The pin is exact rational arithmetic
(fractions.Fraction), i.e. the definition itself evaluated without rounding.
"""
import math
import struct
from fractions import Fraction

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
from oracle import py_ref

I64_MAX = (1 << 63) - 1
I64_MIN = -(1 << 63)


def exact_k(x, eps):
    if math.isnan(x):
        return 0
    inv = 1.0 / eps
    if math.isinf(x):
        return I64_MAX if x > 0 else I64_MIN
    return max(I64_MIN, min(I64_MAX, math.floor(Fraction(x) * Fraction(inv))))


EPS = [1e-3, 1e-4, 1e-5, 1e-6, 1e-7, 1e-8, 2.0 ** -10, 0.3, 7.0, 1e-300, 1e300]


@settings(max_examples=2000, deadline=None)
@given(st.floats(allow_nan=True, allow_infinity=True, width=64), st.sampled_from(EPS))
def test_quant_k_matches_exact_rational_f64(x, eps):
    assert oracle.quant_k(x, eps) == exact_k(x, eps)


@settings(max_examples=2000, deadline=None)
@given(st.floats(allow_nan=True, allow_infinity=True, width=32), st.sampled_from(EPS))
def test_quant_k_matches_exact_rational_f32(x, eps):
    x32 = float(np.float32(x))
    assert oracle.quant_k(x32, eps) == exact_k(x32, eps)


def test_py_ref_agrees_on_specials():
    for eps in EPS:
        for x in (0.0, -0.0, 5e-324, -5e-324, 1e-310, -1e-310, 1.0, -1.0, 0.5, -0.5,
                  1e18, -1e18, 2.0 ** 62, -(2.0 ** 62), 2.0 ** 63, -(2.0 ** 63), 1e300,
                  -1e300, float("inf"), float("-inf"), float("nan")):
            assert oracle.quant_k(x, eps) == py_ref.quant_k(x, eps) == exact_k(x, eps), (x, eps)


def test_power_of_two_closed_forms():
    e = 2.0 ** -10  # 1/e exact, products exact
    assert oracle.quant_k(3 * e, e) == 3
    assert oracle.quant_k(-(2.0 ** -11), e) == -1   # floor, not truncation (R5)
    assert oracle.quant_k(-0.0, e) == 0
    assert oracle.quant_k(0.0, e) == 0
    assert oracle.quant_k(e - 2.0 ** -60, e) == 0
    assert oracle.quant_k(-e, e) == -1
    assert oracle.quant_k(-e - 2.0 ** -60, e) == -2
    assert oracle.quant_k(float("nan"), e) == 0
    assert oracle.quant_k(float("inf"), e) == I64_MAX
    assert oracle.quant_k(float("-inf"), e) == I64_MIN


def test_underflowing_negative_product_floors_to_minus_one():
    # |x * inv| below half the smallest subnormal: RN gives -0 but floor(exact) = -1
    assert oracle.quant_k(-5e-324, 4.0) == -1
    assert oracle.quant_k(5e-324, 4.0) == 0


def test_saturation_boundary_near_2_63():
    # x*inv rounds to exactly 2^63 but the exact product is below it
    inv = 1.0 / 3.0
    x = math.ldexp(3.0, 63)      # exact product 2^63 * (3 * RN(1/3)) slightly below 2^63
    assert oracle.quant_k(x, 3.0) == exact_k(x, 3.0)
    for x in np.nextafter(np.float64(2.0 ** 63) * 3, 0) * np.array([1.0, -1.0]):
        assert oracle.quant_k(float(x), 3.0) == exact_k(float(x), 3.0)


def test_truncation_would_merge_but_floor_separates():
    # R5: a = 0.9 eps, b = -0.9 eps, |a-b| = 1.8 eps > eps; truncation puts both in bin 0
    eps = 1e-5
    assert oracle.quant_k(0.9 * eps, eps) != oracle.quant_k(-0.9 * eps, eps)


def test_rescale_reading_would_lose_changes_but_bin_index_keeps_them():
    # R7 regression: at eps=1e-6 on f32 values in [16, 32) the f32 ulp (1.9e-6) exceeds eps,
    # so every pair of adjacent f32 values differs by more than eps and must get different words.
    eps = 1e-6
    rng = np.random.default_rng(7)
    base = rng.uniform(16.0, 32.0, 5000).astype(np.float32)
    nxt = np.nextafter(base, np.float32(np.inf))
    wa = oracle.quantize(base, eps)
    wb = oracle.quantize(nxt, eps)
    assert np.all(np.abs(nxt.astype(np.float64) - base.astype(np.float64)) > eps)
    assert np.all(wa != wb)
    # the rejected "rescale to the input precision" reading merges some of these pairs
    inv = 1.0 / eps
    resc_a = (np.floor(base.astype(np.float64) * inv) / inv).astype(np.float32)
    resc_b = (np.floor(nxt.astype(np.float64) * inv) / inv).astype(np.float32)
    assert np.any(resc_a == resc_b)


@settings(max_examples=1000, deadline=None)
@given(st.floats(-1e6, 1e6), st.floats(1.5, 1e3), st.sampled_from([1e-3, 1e-5, 1e-6, 1e-8]))
def test_no_false_negative_bins(a, mult, eps):
    # |a - b| >= 1.5 eps  =>  different bins (in-domain: |x*inv| < 2^62)
    b = a + mult * eps
    if b - a < 1.5 * eps or abs(a) / eps > 2.0 ** 60:
        return
    assert oracle.quant_k(a, eps) != oracle.quant_k(b, eps)


def test_quantize_words_f32_low_bits_and_f64_full():
    eps = 1e-3
    x32 = np.array([0.0, -0.0005, 1.0, -1.0, 2.5e6], np.float32)
    w32 = oracle.quantize(x32, eps)
    for xi, wi in zip(x32, w32):
        assert int(wi) == exact_k(float(xi), eps) & 0xFFFFFFFF
    x64 = np.array([0.0, -0.0005, 1.0, -1.0, 2.5e12, -7.25], np.float64)
    w64 = oracle.quantize(x64, eps)
    for xi, wi in zip(x64, w64):
        assert int(wi) == exact_k(float(xi), eps) & ((1 << 64) - 1)
