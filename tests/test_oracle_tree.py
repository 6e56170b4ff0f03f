"""Pins for the oracle's leaves, levels, BFS diff and verify.

Leaves/levels: Alg. 1 P:497-526, P:607-615 (readings R2-R4, R10, R12-R14).
Diff: P:555-566, P:642-648 (R16).  Verify: P:568-578, P:713-716 (R11).
"""
import os
import re

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
from oracle import py_ref


def rand_arr(rng, n, dt):
    if dt == np.float32:
        return rng.uniform(-1, 1, n).astype(np.float32)
    return rng.normal(0, 1, n)


# ---------------------------------------------------------------- leaves ----

@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-3, 1e-6, 0.0])
@pytest.mark.parametrize("n,chunk", [(1, 16), (3, 16), (7, 32), (64, 64), (100, 48), (257, 128),
                                     (1000, 512)])
def test_leaves_match_py_ref(dt, eps, n, chunk):
    rng = np.random.default_rng(n * 31 + chunk)
    a = rand_arr(rng, n, dt)
    got = oracle.leaves(a, chunk, eps)
    ref = py_ref.leaves([float(v) for v in a], dt == np.float32, chunk, eps)
    assert [bytes(r) for r in got] == ref


def test_first_block_is_standard_murmur3f_seed0():
    # Alg. 1 P:503 "seed = 0": a one-block chunk's leaf is Murmur3F(words, 16, seed 0)
    rng = np.random.default_rng(1)
    a = rng.uniform(-1, 1, 4).astype(np.float32)
    w = oracle.quantize(a, 1e-4).tobytes()
    assert oracle.leaves(a, 16, 1e-4)[0].tobytes() == oracle.murmur3f(w, 0)


def test_two_block_chain_seeds_with_full_digest():
    # R2: block 2 is hashed from the full 128-bit digest of block 1
    rng = np.random.default_rng(2)
    a = rng.uniform(-1, 1, 8).astype(np.float32)
    w = oracle.quantize(a, 1e-4).tobytes()
    h1, h2 = oracle.murmur3f_state(w[:16], 0, 0)
    h1, h2 = oracle.murmur3f_state(w[16:], h1, h2)
    leaf = oracle.leaves(a, 32, 1e-4)[0].tobytes()
    assert leaf == h1.to_bytes(8, "little") + h2.to_bytes(8, "little")


# ------------------------------------------- hash block size (R23) ----
# "the block size is variable and can be adjusted": the chain runs
# over blocks of `hash_block` bytes; 16 is the paper's default, 0 the
# whole chunk in one call.

@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-5, 0.0])
@pytest.mark.parametrize("n,chunk,blk", [(7, 32, 32), (100, 48, 32), (257, 128, 64),
                                         (1000, 512, 128), (1000, 512, 0), (33, 64, 48),
                                         (300, 256, 1024)])
def test_hash_block_leaves_match_py_ref(dt, eps, n, chunk, blk):
    rng = np.random.default_rng(n * 7 + blk)
    a = rand_arr(rng, n, dt)
    got = oracle.leaves(a, chunk, eps, hash_block=blk)
    ref = py_ref.leaves([float(v) for v in a], dt == np.float32, chunk, eps, blk)
    assert [bytes(r) for r in got] == ref


def test_hash_block_16_is_the_default_chain():
    rng = np.random.default_rng(5)
    a = rng.uniform(-1, 1, 999).astype(np.float32)
    assert np.array_equal(oracle.leaves(a, 256, 1e-5), oracle.leaves(a, 256, 1e-5, hash_block=16))


@pytest.mark.parametrize("chunk", [16, 64, 4096])
def test_whole_chunk_block_is_one_standard_murmur3f_call(chunk):
    # block = chunk: the leaf is SMHasher MurmurHash3_x64_128(words of the chunk, seed 0),
    # computed here by the independent pure-Python implementation pinned to 0x6384BA69
    rng = np.random.default_rng(chunk)
    a = rng.uniform(-1, 1, 3 * chunk // 4 + 1).astype(np.float32)   # ragged last chunk
    got = oracle.leaves(a, chunk, 1e-4, hash_block=0)
    assert np.array_equal(got, oracle.leaves(a, chunk, 1e-4, hash_block=chunk))
    per = chunk // 4
    for c in range(got.shape[0]):
        w = py_ref.words([float(v) for v in a[c * per:(c + 1) * per]], True, 1e-4)
        assert got[c].tobytes() == py_ref.murmur3f(w, 0)


def test_hash_block_larger_than_chunk_is_whole_chunk():
    rng = np.random.default_rng(6)
    a = rng.normal(size=77)
    assert np.array_equal(oracle.leaves(a, 64, 1e-3, hash_block=1024),
                          oracle.leaves(a, 64, 1e-3, hash_block=0))


def test_hash_block_changes_digest_but_not_the_diff():
    # different block sizes give different leaves, yet flag exactly the same chunks
    rng = np.random.default_rng(8)
    a = rng.uniform(-1, 1, 4096).astype(np.float32)
    b = a.copy()
    b[[5, 700, 701, 3000]] += np.float32(1e-2)
    out = {}
    for blk in (16, 64, 0):
        la, lb = oracle.leaves(a, 512, 1e-5, hash_block=blk), oracle.leaves(b, 512, 1e-5, hash_block=blk)
        out[blk] = np.nonzero((la != lb).any(axis=1))[0].tolist()
    assert out[16] == out[64] == out[0] == [0, 5, 23]
    assert not np.array_equal(oracle.leaves(a, 512, 1e-5), oracle.leaves(a, 512, 1e-5, hash_block=0))


def test_hash_block_must_be_multiple_of_16():
    with pytest.raises(ValueError):
        oracle.leaves(np.zeros(8, np.float32), 32, 1e-3, hash_block=24)


def test_raw_mode_hashes_input_bytes():
    # R10: eps == 0 hashes the raw element bytes
    rng = np.random.default_rng(3)
    a = rng.normal(size=6)
    raw = a.tobytes()
    h1 = h2 = 0
    for off in range(0, len(raw), 16):
        h1, h2 = oracle.murmur3f_state(raw[off:off + 16], h1, h2)
    assert oracle.leaves(a, 64, 0.0)[0].tobytes() == h1.to_bytes(8, "little") + h2.to_bytes(8, "little")


def test_within_bin_changes_do_not_change_leaf_and_bin_changes_do():
    eps = 2.0 ** -10
    a = (np.arange(256, dtype=np.float32) + 0.25) * np.float32(eps)
    b = a + np.float32(0.5 * eps)           # same bins
    c = a.copy()
    c[100] += np.float32(eps)               # one element one bin up
    la, lb, lc = (oracle.leaves(x, 256, eps) for x in (a, b, c))
    assert np.array_equal(la, lb)
    diff = np.any(la != lc, axis=1)
    assert list(np.nonzero(diff)[0]) == [100 * 4 // 256]


def test_invalid_args_rejected():
    a = np.zeros(10, np.float32)
    with pytest.raises(ValueError):
        oracle.leaves(a, 24, 1e-3)       # not a multiple of 16
    with pytest.raises(ValueError):
        oracle.leaves(a, 16, -1.0)
    with pytest.raises(ValueError):
        oracle.leaves(a, 16, float("nan"))


def test_threads_do_not_change_leaves():
    rng = np.random.default_rng(4)
    a = rand_arr(rng, 100_003, np.float32)
    l1 = oracle.leaves(a, 512, 1e-5, threads=1)
    l8 = oracle.leaves(a, 512, 1e-5, threads=8)
    assert np.array_equal(l1, l8)


# ---------------------------------------------------------------- levels ----

def H(x, y):
    return py_ref.murmur3f(bytes(x) + bytes(y), 0)


@pytest.mark.parametrize("L", [1, 2, 3, 4, 5])
def test_tree_closed_forms(L):
    rng = np.random.default_rng(L)
    lv = rng.integers(0, 256, (L, 16), dtype=np.uint8)
    nodes = oracle.levels(lv)
    l = [lv[i].tobytes() for i in range(L)]
    expect = {
        1: l[0] if L == 1 else None,
        2: H(l[0], l[1]) if L >= 2 else None,
        3: H(H(l[0], l[1]), l[2]) if L >= 3 else None,
        4: H(H(l[0], l[1]), H(l[2], l[3])) if L >= 4 else None,
        5: H(H(H(l[0], l[1]), H(l[2], l[3])), l[4]) if L >= 5 else None,
    }[L]
    assert nodes[-1].tobytes() == expect
    assert nodes.shape[0] == sum(oracle.level_sizes(L))


@settings(max_examples=60, deadline=None)
@given(st.integers(1, 300))
def test_levels_match_py_ref(L):
    rng = np.random.default_rng(L)
    lv = rng.integers(0, 256, (L, 16), dtype=np.uint8)
    nodes = oracle.levels(lv)
    ref = py_ref.levels([lv[i].tobytes() for i in range(L)])
    flat = [n for level in ref for n in level]
    assert [nodes[i].tobytes() for i in range(nodes.shape[0])] == flat


def test_metadata_size_matches_paper_example():
    txt = open(os.path.join(os.path.dirname(__file__), "golden", "paper_metadata_example.txt")).read()
    N = int(re.search(r"checkpoint_bytes = (\d+)", txt).group(1))
    C = int(re.search(r"chunk_bytes = (\d+)", txt).group(1))
    D = int(re.search(r"digest_bytes = (\d+)", txt).group(1))
    approx = float(re.search(r"metadata_mb_approx = (\d+)", txt).group(1))
    L = -(-N // C)
    size = sum(oracle.level_sizes(L)) * D
    assert abs(size / 1e6 - approx) < 0.5                       # "~55MB"
    paper_formula = 2 * D * (N / C - 1)
    assert abs(size - paper_formula) / paper_formula < 1e-3


# ------------------------------------------------------------------ diff ----

def _perturbed_pair(rng, n, dt, eps, n_changes, straddle=0):
    a = rand_arr(rng, n, dt)
    b = a.copy()
    if n_changes:
        idx = rng.choice(n, size=n_changes, replace=False)
        mag = rng.uniform(0.05, 20, n_changes) * eps * rng.choice([-1, 1], n_changes)
        b[idx] = (a[idx].astype(np.float64) + mag).astype(dt)
    return a, b


@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("n,chunk,changes", [(5000, 64, 0), (5000, 64, 1), (5000, 64, 17),
                                             (33333, 256, 40), (4096, 16, 300)])
def test_bfs_equals_plain_leaf_compare_for_every_start_level(dt, n, chunk, changes):
    rng = np.random.default_rng(n + changes)
    eps = 1e-4
    a, b = _perturbed_pair(rng, n, dt, eps, changes)
    la, lb = oracle.leaves(a, chunk, eps), oracle.leaves(b, chunk, eps)
    ta, tb = oracle.levels(la), oracle.levels(lb)
    L = la.shape[0]
    plain = np.nonzero(np.any(la != lb, axis=1))[0]
    sizes = oracle.level_sizes(L)
    Ts = sorted(set([1, 2, 3, L, L + 1, 10**9] + [s for s in sizes] + [s + 1 for s in sizes]))
    for T in Ts:
        got = oracle.diff(ta, tb, L, T)
        assert np.array_equal(got, plain), T


def test_start_level_rule():
    # level closest to the root with n_l >= T, else leaves
    assert oracle.start_level(1000, 1) == oracle.level_sizes(1000).index(1)
    assert oracle.start_level(1000, 1000) == 0
    assert oracle.start_level(1000, 10**6) == 0
    assert oracle.start_level(1000, 500) == 1
    assert oracle.start_level(1000, 126) == 2   # 1000,500,250,125 -> level 2 (250) is the last >= 126


def test_identical_inputs_identical_roots_and_empty_diff():
    rng = np.random.default_rng(9)
    a = rand_arr(rng, 70000, np.float32)
    ta = oracle.levels(oracle.leaves(a, 4096, 1e-6))
    tb = oracle.levels(oracle.leaves(a.copy(), 4096, 1e-6))
    assert ta[-1].tobytes() == tb[-1].tobytes()
    assert oracle.diff(ta, tb, oracle.n_chunks(a.size, 0, 4096)).size == 0


# ---------------------------------------------------------------- verify ----

@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("chunk", [16, 64, 4096])
def test_no_false_negatives_and_verify_equals_brute(dt, chunk):
    rng = np.random.default_rng(chunk)
    eps = 1e-5
    n = 50_001
    a, b = _perturbed_pair(rng, n, dt, eps, 200)
    # bin straddlers: |a-b| = 0.2 eps across a bin edge -> flagged but not different
    k = rng.choice(n, 20, replace=False)
    m = np.round(a[k].astype(np.float64) / eps)
    a[k] = (m * eps - 0.1 * eps).astype(dt)
    b[k] = (m * eps + 0.1 * eps).astype(dt)
    la, lb = oracle.leaves(a, chunk, eps), oracle.leaves(b, chunk, eps)
    ta, tb = oracle.levels(la), oracle.levels(lb)
    chunks = oracle.diff(ta, tb, la.shape[0])
    truth = oracle.brute(a, b, eps)
    per = chunk // a.itemsize
    # invariant 1: no false negatives
    assert set(np.unique(truth // per)) <= set(chunks.tolist())
    # invariant 2: verify over flagged chunks equals brute force exactly
    assert np.array_equal(oracle.verify(a, b, chunk, chunks, eps), truth)


def test_brute_predicate_semantics():
    eps = 0.5
    a = np.array([0.0, 0.0, 1.0, np.nan, np.inf, np.inf, -0.0, 0.0], np.float64)
    b = np.array([0.5, 0.51, 0.4, 1.0, np.inf, -np.inf, 0.0, np.nan])
    # strict '>', NaN never differs, inf - inf (NaN) never differs
    assert oracle.brute(a, b, eps).tolist() == [1, 2, 5]


def test_verify_partial_last_chunk_and_empty_list():
    a = np.zeros(10, np.float32)
    b = a.copy()
    b[9] = 1.0
    assert oracle.verify(a, b, 16, np.array([2]), 0.5).tolist() == [9]
    assert oracle.verify(a, b, 16, np.array([], np.int64), 0.5).size == 0


def test_checkpoint_multi_array_bookkeeping():
    rng = np.random.default_rng(11)
    eps = 1e-4
    arrs_a = [rand_arr(rng, n, np.float32) for n in (1000, 1, 4097, 333)]
    arrs_b = [x.copy() for x in arrs_a]
    arrs_b[2][4096] += 1.0
    arrs_b[0][5] += 1.0
    A = oracle.build_checkpoint(arrs_a, 64, eps)
    B = oracle.build_checkpoint(arrs_b, 64, eps)
    assert A.root != B.root
    ch = oracle.diff_checkpoint(A, B)
    assert ch.tolist() == [0, A.chunk_base[2] + 4096 * 4 // 64]
    idx = oracle.verify_checkpoint(arrs_a, arrs_b, 64, ch, eps, A)
    assert idx.tolist() == oracle.brute_checkpoint(arrs_a, arrs_b, eps).tolist() == [5, 1001 + 4096]
    # the checkpoint root is the level construction over the array roots (R15)
    assert A.top[-1].tobytes() == oracle.levels(A.array_roots)[-1].tobytes()
