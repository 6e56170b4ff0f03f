"""Property-based pins for the oracle (hypothesis): the C oracle against the independent pure-Python
reference (oracle/py_ref.py, itself pinned to SMHasher's 0x6384BA69 and to exact rational
rounding) on random tiny checkpoints -- any values including NaN, +-inf, -0, subnormals and
magnitudes beyond 2^63*eps, any eps (0 = raw bits), chunk sizes and hash blocks -- plus the
paper's comparison invariants on random pairs:

* leaves: Alg. 1 P:499-512, P:607-618 (readings R2-R5, R8-R10, R12, R23);
* levels / root: Alg. 1 P:513-521 (R13, R14);
* no false negatives and verify == brute force (R11).
"""
import math

import numpy as np
from hypothesis import HealthCheck, given, settings, strategies as st

import oracle
from oracle import py_ref

F32_SPECIALS = [0.0, -0.0, float("inf"), float("-inf"), float("nan"), 1e-45, -1e-45,
                3.4028234663852886e38, -3.4028234663852886e38, 1.0, -1.0]
F64_SPECIALS = F32_SPECIALS + [5e-324, 1.7976931348623157e308, 2.0 ** 63, -(2.0 ** 63)]


def _values(is_f32):
    fl = st.floats(width=32 if is_f32 else 64, allow_nan=True, allow_infinity=True)
    sp = st.sampled_from(F32_SPECIALS if is_f32 else F64_SPECIALS)
    return st.lists(st.one_of(fl, fl, sp), min_size=1, max_size=40)


EPS = st.one_of(st.just(0.0), st.floats(min_value=1e-30, max_value=1e30, allow_nan=False,
                                        allow_infinity=False))


@st.composite
def checkpoint(draw):
    is_f32 = draw(st.booleans())
    vals = draw(_values(is_f32))
    eps = draw(EPS)
    chunk = 16 * draw(st.integers(1, 6))
    block = draw(st.sampled_from([16, 16, 32, 48, 0]))
    return is_f32, vals, eps, chunk, block


@settings(max_examples=200, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(checkpoint())
def test_leaves_and_levels_match_py_ref(case):
    is_f32, vals, eps, chunk, block = case
    if eps and not math.isfinite(1.0 / eps):
        return                                                 # outside R10's domain
    a = np.array(vals, dtype=np.float32 if is_f32 else np.float64)
    # py_ref reads the stored values (an f32 array holds f32-rounded values)
    ref_vals = [float(v) for v in a]
    got = oracle.leaves(a, chunk, eps, hash_block=block)
    ref = py_ref.leaves(ref_vals, is_f32, chunk, eps, block)
    assert [bytes(r) for r in got] == ref
    lv_c = oracle.levels(got)
    lv_p = py_ref.levels(ref)
    assert bytes(lv_c[-1]) == lv_p[-1][0]                      # the root
    assert [bytes(r) for r in lv_c] == [n for level in lv_p for n in level]


@st.composite
def pair(draw):
    is_f32 = draw(st.booleans())
    dt = np.float32 if is_f32 else np.float64
    n = draw(st.integers(1, 300))
    seed = draw(st.integers(0, 2 ** 32 - 1))
    eps = draw(st.floats(min_value=1e-9, max_value=1e3, allow_nan=False))
    chunk = 16 * draw(st.integers(1, 20))
    rng = np.random.default_rng(seed)
    scale = 10.0 ** rng.uniform(-3, 3)
    a = (rng.standard_normal(n) * scale).astype(dt)
    b = a.copy()
    k = rng.integers(0, n + 1)
    pos = rng.integers(0, n, size=k)
    b[pos] = (b[pos].astype(np.float64) + eps * 10.0 ** rng.uniform(-2, 2, size=k)
              * np.where(rng.random(k) < 0.5, -1, 1)).astype(dt)
    return a, b, eps, chunk


@settings(max_examples=150, deadline=None)
@given(pair())
def test_no_false_negatives_and_verify_equals_brute(p):
    a, b, eps, chunk = p
    la, lb = oracle.leaves(a, chunk, eps), oracle.leaves(b, chunk, eps)
    na, nb = oracle.levels(la), oracle.levels(lb)
    L = la.shape[0]
    flagged = oracle.diff(na, nb, L)
    truth = oracle.brute(a, b, eps)
    per = chunk // a.itemsize
    assert set((truth // per).tolist()) <= set(flagged.tolist())     # no false negatives
    assert np.array_equal(oracle.verify(a, b, chunk, flagged, eps), truth)
    # the BFS from any start level lists exactly the chunks whose leaves differ
    plain = np.nonzero(np.any(la != lb, axis=1))[0]
    for T in (1, 3, 10 ** 9):
        assert np.array_equal(oracle.diff(na, nb, L, T), plain)
    if np.array_equal(a.view(np.uint8), b.view(np.uint8)):
        assert bytes(na[-1]) == bytes(nb[-1]) and flagged.size == 0
