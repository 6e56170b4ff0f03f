"""GPU parity: libckpt (CUDA sm_100a, via the C ABI) vs the CPU oracle, bit-exact.

Covers leaves, every tree node, roots, chunk lists, element ids and counts on
seeded synthetic checkpoints (synth), ragged/partial sizes, special values,
every BFS start level, truncation and error paths.  Full-size (BASELINE
configs[1]) checks sample leaves and recompute levels/verify with the oracle.
"""
import os

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

ck = pytest.importorskip("paper_conf_middleware_tanaabcrtn24_b200")


def np_of(t):
    return t.detach().cpu().numpy()


def gpu_tree_nodes(tree, array=0):
    return np_of(tree.nodes(array))


def oracle_tree(a_np, chunk, eps):
    lv = oracle.leaves(a_np, chunk, eps, threads=8)
    return oracle.levels(lv), lv.shape[0]


# ------------------------------------------------------------ leaves/trees --

CASES = [
    # (n, dtype, chunk, eps)
    (1, torch.float32, 16, 1e-3),
    (3, torch.float32, 16, 1e-3),        # partial block only
    (5, torch.float32, 16, 1e-3),
    (1000, torch.float32, 48, 1e-4),     # runtime chunk size, not a multiple of 64
    (1025, torch.float32, 64, 1e-4),     # tail block of 4 bytes
    (4097, torch.float32, 512, 1e-5),
    (100_003, torch.float32, 4096, 1e-6),
    ((1 << 20), torch.float32, 4096, 1e-5),   # config 1
    (1_000_000, torch.float32, 4096, 1e-5),   # config 1 tail case
    (70_001, torch.float32, 65536, 1e-3),
    (3, torch.float64, 16, 1e-3),
    (999, torch.float64, 32, 1e-7),
    (123_457, torch.float64, 1024, 1e-8),
    (50_000, torch.float64, 8192, 1e-3),
    (10_000, torch.float32, 4096, 0.0),       # raw-bit mode (R10)
    (10_001, torch.float64, 160, 0.0),
]


def _data(n, dtype, seed):
    if dtype == torch.float32:
        return synth.uniform(seed, n, "cuda") * 2.0 - 1.0
    return synth.normal(seed, n, "cuda", dtype=torch.float64)


@pytest.mark.parametrize("n,dtype,chunk,eps", CASES)
def test_tree_bit_exact(n, dtype, chunk, eps):
    a = _data(n, dtype, n + chunk)
    t = ck.tree_build(a, chunk, eps)
    got = gpu_tree_nodes(t)
    ref, L = oracle_tree(np_of(a), chunk, eps)
    assert got.shape == ref.shape
    bad = np.nonzero(np.any(got != ref, axis=1))[0]
    assert bad.size == 0, f"{bad.size} nodes differ, first {bad[:5]}"
    assert t.root() == ref[-1].tobytes()
    assert t.n_leaves == L


# Interior levels (K2) over leaf counts around its CTA group (2048 nodes) and pass
# boundaries (4 nodes per thread, two levels per pass): every node vs the oracle's
# level construction (Alg. 1, R13 promotion of an odd last node).
@pytest.mark.parametrize("L", [1, 2, 3, 4, 5, 7, 8, 9, 31, 33, 511, 513, 2047, 2048, 2049, 2050,
                               4095, 4097, 6143, 65537, 300_001])
def test_levels_from_digests_bit_exact(L):
    g = torch.Generator().manual_seed(L)
    d = torch.randint(0, 256, (L, 16), dtype=torch.uint8, generator=g)
    t = ck.tree_from_digests(d.cuda())
    got = gpu_tree_nodes(t)
    ref = oracle.levels(d.numpy())
    assert got.shape == ref.shape
    bad = np.nonzero(np.any(got != ref, axis=1))[0]
    assert bad.size == 0, f"{bad.size} nodes differ, first {bad[:5]}"


def test_levels_from_digests_batch_equals_single():
    """ckpt_tree_from_digests_batch (one levels launch, the multi-GPU step's top trees)."""
    counts = [1, 7, 2049, 48]
    g = torch.Generator().manual_seed(5)
    d = torch.randint(0, 256, (sum(counts), 16), dtype=torch.uint8, generator=g)
    trees = ck.tree_from_digests_batch(d.cuda(), counts)
    off = 0
    for t, c in zip(trees, counts):
        ref = oracle.levels(d[off:off + c].numpy())
        assert np.array_equal(gpu_tree_nodes(t), ref)
        assert t.root() == ref[-1].tobytes()
        off += c
    with pytest.raises(ValueError):
        ck.tree_from_digests_batch(d.cuda(), [1, 2])


# Multi-array batch: arrays of different heights whose groups end mid-pass.
def test_levels_multi_array_ragged_groups():
    sizes = [4097 * 4096, 1 * 4096, 2049 * 4096 + 8, 3 * 4096]
    arrs = [synth.uniform(77 + i, nb // 4, "cuda") for i, nb in enumerate(sizes)]
    t = ck.tree_build(arrs, 4096, 1e-5)
    for i, x in enumerate(arrs):
        ref, _ = oracle_tree(np_of(x), 4096, 1e-5)
        assert np.array_equal(gpu_tree_nodes(t, i), ref), f"array {i}"


SPECIALS32 = np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 1e-45, -1e-45, 1.17549435e-38,
                       -1.17549435e-38, 3.4028235e38, -3.4028235e38, 1.0, -1.0, 0.5, -0.5,
                       2.0 ** 24, -(2.0 ** 24), 2.0 ** 31, 2.0 ** 40, -(2.0 ** 60), 1e-5, -1e-5,
                       2.0 ** 51 * 1e-6, -(2.0 ** 51) * 1e-6, 2.0 ** 63 * 1e-6], dtype=np.float32)


@pytest.mark.parametrize("eps", [1e-3, 1e-5, 1e-6, 1e-8, 2.0 ** -10, 0.3, 7.0, 1e-30, 1e30])
def test_quantizer_specials_and_random_bit_patterns_f32(eps):
    rng = np.random.default_rng(int(eps * 1e9) % 1000 + 1)
    bits = rng.integers(0, 2 ** 32, size=1 << 20, dtype=np.uint64).astype(np.uint32)
    x = bits.view(np.float32).copy()
    x[: SPECIALS32.size] = SPECIALS32
    x[SPECIALS32.size: 2 * SPECIALS32.size] = np.nextafter(SPECIALS32, np.float32(0))
    # chunk = one block: every leaf pins 4 words
    a = torch.from_numpy(x).cuda()
    t = ck.tree_build(a, 16, eps)
    got = gpu_tree_nodes(t)[: x.size // 4]
    ref = oracle.leaves(x, 16, eps, threads=8)
    bad = np.nonzero(np.any(got != ref, axis=1))[0]
    assert bad.size == 0, (bad[:5], x.reshape(-1, 4)[bad[:5]])


@pytest.mark.parametrize("eps", [1e-3, 1e-6, 1e-8, 2.0 ** -10, 1e-300, 1e300])
def test_quantizer_specials_and_random_bit_patterns_f64(eps):
    rng = np.random.default_rng(5)
    bits = rng.integers(0, 2 ** 63, size=1 << 19, dtype=np.uint64) * 2 + rng.integers(0, 2, 1 << 19, dtype=np.uint64)
    x = bits.view(np.float64).copy()
    sp = np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 5e-324, -5e-324, 2.0 ** 62, -(2.0 ** 62),
                   2.0 ** 63, -(2.0 ** 63), 1.7976931348623157e308, -1.7976931348623157e308,
                   1.0, -1.0, 1e-5, -1e-5, 2.0 ** 51 * eps, -(2.0 ** 51) * eps, 2.0 ** 63 * eps,
                   -(2.0 ** 63) * eps, np.nextafter(2.0 ** 63 * eps, 0)], dtype=np.float64)
    x[: sp.size] = sp
    # also values near the fast/slow-path boundary |x| ~ 2^50 * eps (finite: for eps = 1e300
    # the boundary lies beyond DBL_MAX, so the range is capped there and every value is finite)
    scale = 2.0 ** 52 * eps
    if not np.isfinite(scale):
        scale = np.finfo(np.float64).max
    near = rng.uniform(-1.0, 1.0, 1000) * scale
    assert np.all(np.isfinite(near))
    x[sp.size: sp.size + 1000] = near
    a = torch.from_numpy(x).cuda()
    t = ck.tree_build(a, 16, eps)
    got = gpu_tree_nodes(t)[: x.size // 2]
    ref = oracle.leaves(x, 16, eps, threads=8)
    bad = np.nonzero(np.any(got != ref, axis=1))[0]
    assert bad.size == 0, (bad[:5], x.reshape(-1, 2)[bad[:5]])


def test_near_boundary_f32_values():
    # values whose x*inv is within a few ulps of an integer (the floor decision)
    eps = 1e-5
    k = np.arange(-200000, 200000, 7, dtype=np.float64)
    base = (k * eps).astype(np.float32)
    x = np.concatenate([base, np.nextafter(base, np.float32(np.inf)),
                        np.nextafter(base, np.float32(-np.inf))])
    x = x[: (x.size // 4) * 4]
    a = torch.from_numpy(x).cuda()
    t = ck.tree_build(a, 16, eps)
    got = gpu_tree_nodes(t)[: x.size // 4]
    ref = oracle.leaves(x, 16, eps, threads=8)
    assert np.array_equal(got, ref)


# ---------------------------------------------------------- multi-array --

def test_multi_array_checkpoint_matches_oracle():
    sizes = [1000, 1, 4097, 333, 65536, 12345]
    arrs_a = [_data(n, torch.float32, 100 + i) for i, n in enumerate(sizes)]
    arrs_b = [t.clone() for t in arrs_a]
    arrs_b[2][4096] += 1.0
    arrs_b[4][7] += 1e-3
    chunk, eps = 256, 1e-4
    TA = ck.tree_build(arrs_a, chunk, eps)
    TB = ck.tree_build(arrs_b, chunk, eps)
    A = oracle.build_checkpoint([np_of(t) for t in arrs_a], chunk, eps)
    B = oracle.build_checkpoint([np_of(t) for t in arrs_b], chunk, eps)
    for k in range(len(sizes)):
        assert np.array_equal(gpu_tree_nodes(TA, k), A.trees[k])
        assert np.array_equal(gpu_tree_nodes(TB, k), B.trees[k])
    assert np.array_equal(np_of(TA.array_roots()), A.array_roots)
    assert TA.root() == A.root and TB.root() == B.root
    chunks = ck.tree_diff(TA, TB)
    assert np.array_equal(np_of(chunks), oracle.diff_checkpoint(A, B))
    idx, n = ck.verify(arrs_a, arrs_b, chunks, chunk, eps)
    ref = oracle.verify_checkpoint([np_of(t) for t in arrs_a], [np_of(t) for t in arrs_b], chunk,
                                   np_of(chunks), eps, A)
    assert n == ref.size and np.array_equal(np_of(idx), ref)


def test_batch_build_equals_separate_builds():
    sizes_a = [1000, 65536 + 17, 5]
    arrs_a = [_data(n, torch.float32, 300 + i) for i, n in enumerate(sizes_a)]
    arrs_b = [t.clone() for t in arrs_a]
    arrs_b[1][12345] += 1.0
    arrs_c = [_data(n, torch.float32, 400 + i) for i, n in enumerate([7, 4096 * 33])]
    TA, TB, TC = ck.tree_build_batch([arrs_a, arrs_b, arrs_c], 512, 1e-5)
    for T, arrs in ((TA, arrs_a), (TB, arrs_b), (TC, arrs_c)):
        R = oracle.build_checkpoint([np_of(t) for t in arrs], 512, 1e-5)
        assert T.root() == R.root
        for k in range(len(arrs)):
            assert np.array_equal(gpu_tree_nodes(T, k), R.trees[k])
    assert np.array_equal(np_of(ck.tree_diff(TA, TB)), [1000 * 4 // 512 + 1 + 12345 * 4 // 512])


# ------------------------------------------------------------ diff/verify --

@pytest.mark.parametrize("n", [1 << 20, 1_000_000])
def test_config1_pair_end_to_end(n):
    pair = synth.c1_pair(n=n, seed=1, device="cuda")
    a, b = pair.a[0], pair.b[0]
    C, eps = pair.chunk_bytes, pair.eps
    ta, tb = ck.tree_build(a, C, eps), ck.tree_build(b, C, eps)
    chunks = ck.tree_diff(ta, tb)
    idx, cnt = ck.verify(a, b, chunks, C, eps)
    an, bn = np_of(a), np_of(b)
    ra, L = oracle_tree(an, C, eps)
    rb, _ = oracle_tree(bn, C, eps)
    ref_chunks = oracle.diff(ra, rb, L)
    assert np.array_equal(np_of(chunks), ref_chunks)
    truth = oracle.brute(an, bn, eps)
    assert np.array_equal(np_of(idx), truth) and cnt == truth.size
    # paper invariants: no false negatives; straddlers were flagged and removed.  The recipe
    # is exact: the 50 "above" changes (>= 2 eps before rounding to f32, whose ulp on [-1, 1)
    # is <= 6e-8) are exactly the differing elements, the 50 "below" ones (<= 0.5 eps) never are
    per = C // 4
    assert set(np.unique(truth // per)) <= set(ref_chunks.tolist())
    above = np.sort(pair.meta["perturbed"][: pair.meta["n_above"]])
    assert truth.size == pair.meta["n_above"] == 50 and np.array_equal(truth, above)
    straddle = pair.meta["perturbed"][pair.meta["n_above"]: pair.meta["n_above"] + pair.meta["n_straddle"]]
    assert set(np.unique(straddle // per)) <= set(ref_chunks.tolist())   # flagged, then removed


@pytest.mark.parametrize("T", [1, 2, 3, 5, 17, 100, 1000, 4096, 10 ** 9])
def test_diff_independent_of_start_level(T):
    pair = synth.c1_pair(n=1 << 20, seed=3, device="cuda", n_above=300, n_below=300)
    a, b = pair.a[0], pair.b[0]
    ta, tb = ck.tree_build(a, 512, pair.eps), ck.tree_build(b, 512, pair.eps)
    L = ta.n_leaves
    out = torch.empty(L, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    ck.tree_diff_async(ta, tb, out, cnt, T=T)
    n = int(cnt.item())
    la = oracle.leaves(np_of(a), 512, pair.eps, threads=8)
    lb = oracle.leaves(np_of(b), 512, pair.eps, threads=8)
    plain = np.nonzero(np.any(la != lb, axis=1))[0]
    assert np.array_equal(np_of(out[:n]), plain)


def test_bfs_multi_array_mid_level_start():
    sizes = [5000, 300_000, 1, 77_777]
    arrs_a = [_data(n, torch.float64, 7 + i) for i, n in enumerate(sizes)]
    arrs_b = [t.clone() for t in arrs_a]
    g = torch.Generator(device="cpu").manual_seed(0)
    for t in arrs_b:
        k = torch.randint(0, t.numel(), (min(50, t.numel()),), generator=g).cuda()
        t[k] += 1.0
    TA, TB = ck.tree_build(arrs_a, 64, 1e-6), ck.tree_build(arrs_b, 64, 1e-6)
    A = oracle.build_checkpoint([np_of(t) for t in arrs_a], 64, 1e-6)
    B = oracle.build_checkpoint([np_of(t) for t in arrs_b], 64, 1e-6)
    ref = oracle.diff_checkpoint(A, B)
    for T in (1, 10, 1000, 20_000, 10 ** 12):
        out = torch.empty(TA.n_leaves, dtype=torch.int64, device="cuda")
        cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
        ck.tree_diff_async(TA, TB, out, cnt, T=T)
        assert np.array_equal(np_of(out[: int(cnt.item())]), ref), T


def test_identical_inputs_identical_roots_empty_diff():
    a = _data(1 << 18, torch.float32, 42)
    ta, tb = ck.tree_build(a, 4096, 1e-6), ck.tree_build(a.clone(), 4096, 1e-6)
    assert ta.root() == tb.root()
    assert ck.tree_diff(ta, tb).numel() == 0
    idx, n = ck.verify(a, a.clone(), torch.arange(ta.n_leaves, device="cuda"), 4096, 1e-6)
    assert n == 0


def test_verify_every_chunk_equals_brute_force_f64():
    pair = synth.c3_pair(n=1 << 20, seed=3, device="cuda", n_clusters=64, mean_len=256)
    a, b = pair.a[0], pair.b[0]
    for C, eps in ((512, 1e-3), (4096, 1e-6), (65536, 1e-8)):
        L = -(-a.numel() * 8 // C)
        idx, n = ck.verify(a, b, torch.arange(L, device="cuda"), C, eps)
        truth = oracle.brute(np_of(a), np_of(b), eps)
        assert n == truth.size and np.array_equal(np_of(idx), truth)


def test_truncation_returns_prefix_and_full_count():
    pair = synth.c1_pair(n=1 << 20, seed=9, device="cuda", n_above=500, n_below=0)
    a, b = pair.a[0], pair.b[0]
    ta, tb = ck.tree_build(a, 4096, pair.eps), ck.tree_build(b, 4096, pair.eps)
    full = ck.tree_diff(ta, tb)
    part = ck.tree_diff(ta, tb, cap=7)
    assert np.array_equal(np_of(part), np_of(full)[:7])
    idx_full, n_full = ck.verify(a, b, full, 4096, pair.eps)
    idx_part, n_part = ck.verify(a, b, full, 4096, pair.eps, cap=11)
    assert n_part == n_full and np.array_equal(np_of(idx_part), np_of(idx_full)[:11])


def test_compare_and_compare_host_agree_with_oracle():
    pair = synth.c2_pair(n_particles=1 << 16, seed=2, device="cuda", frac=0.02, n_clusters=8)
    C, eps = pair.chunk_bytes, pair.eps
    chunks, idx, nc, nd, ra, rb = ck.compare(pair.a, pair.b, C, eps)
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    A = oracle.build_checkpoint(an, C, eps)
    B = oracle.build_checkpoint(bn, C, eps)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, C, ref_chunks, eps, A)
    assert ra == A.root and rb == B.root
    assert np.array_equal(np_of(chunks), ref_chunks) and nc == ref_chunks.size
    assert np.array_equal(np_of(idx), ref_idx) and nd == ref_idx.size
    assert np.array_equal(ref_idx, oracle.brute_checkpoint(an, bn, eps))
    host_a = [t.cpu().pin_memory() for t in pair.a]
    host_b = [t.cpu().pin_memory() for t in pair.b]
    hidx, hnc, hnd, hra, hrb = ck.compare_host(host_a, host_b, C, eps)
    assert (hnc, hnd, hra, hrb) == (nc, nd, ra, rb)
    assert np.array_equal(hidx.numpy(), ref_idx)


@pytest.mark.parametrize("dt", [torch.float32, torch.float64])
@pytest.mark.parametrize("chunk", [512, 4096])
def test_fused_diff_verify_equals_separate_stages(dt, chunk):
    sizes = [70_000, 3, 131_072 + 5]
    arrs_a = [_data(n, dt, 500 + i) for i, n in enumerate(sizes)]
    arrs_b = [t.clone() for t in arrs_a]
    g = torch.Generator(device="cpu").manual_seed(1)
    for t in arrs_b:                    # clustered and scattered changes, above and below eps
        k = torch.randint(0, t.numel(), (min(300, t.numel()),), generator=g).cuda()
        t[k] += (torch.rand(k.numel(), generator=g, dtype=torch.float64).cuda() * 4e-5).to(dt)
        s0 = t.numel() // 3
        t[s0:s0 + 5000] += 1e-3
    eps = 1e-5
    TA, TB = ck.tree_build_batch([arrs_a, arrs_b], chunk, eps)
    L = TA.n_leaves
    n = sum(t.numel() for t in arrs_a)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(n, dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    ck.diff_verify_async(TA, TB, arrs_a, arrs_b, chunks, idx, counts)
    nc, nd = counts.tolist()
    A = oracle.build_checkpoint([np_of(t) for t in arrs_a], chunk, eps)
    B = oracle.build_checkpoint([np_of(t) for t in arrs_b], chunk, eps)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint([np_of(t) for t in arrs_a], [np_of(t) for t in arrs_b],
                                       chunk, ref_chunks, eps, A)
    assert nc == ref_chunks.size and np.array_equal(np_of(chunks[:nc]), ref_chunks)
    assert nd == ref_idx.size and np.array_equal(np_of(idx[:nd]), ref_idx)
    assert np.array_equal(ref_idx, oracle.brute_checkpoint([np_of(t) for t in arrs_a],
                                                           [np_of(t) for t in arrs_b], eps))


# ------------------------------------------------------------ error paths --

def test_error_paths():
    a = _data(1000, torch.float32, 1)
    with pytest.raises(ck.CkptError) as e:
        ck.tree_build(a, 24, 1e-3)
    assert e.value.status == ck.EINVAL
    with pytest.raises(ck.CkptError):
        ck.tree_build(a, 16, -1.0)
    with pytest.raises(ck.CkptError):
        ck.tree_build(a, 16, float("nan"))
    with pytest.raises(ck.CkptError):
        ck.tree_build(a[1:], 16, 1e-3)      # misaligned (4-byte offset)
    t1 = ck.tree_build(a, 64, 1e-3)
    t2 = ck.tree_build(a[:999], 64, 1e-3)
    t3 = ck.tree_build(a, 64, 1e-4)
    with pytest.raises(ck.CkptError) as e:
        ck.tree_diff(t1, t2)
    assert e.value.status == ck.EMISMATCH
    with pytest.raises(ck.CkptError) as e:
        ck.tree_diff(t1, t3)
    assert e.value.status == ck.EMISMATCH


# ------------------------------------------------- full size (configs[1]) --

def full_checkpoint_parity(pair, TA, TB, chunks, idx, counts, brute=True):
    """Every node of every array tree of both runs, both checkpoint roots, the chunk list and
    the element ids of a fused compare vs the oracle, one array at a time (host memory stays
    at one array pair).  Returns (n_chunks, n_diff)."""
    C, eps = pair.chunk_bytes, pair.eps
    th = os.cpu_count() or 8
    nc, nd = counts.tolist()
    got_c, got_i = np_of(chunks[:nc]), np_of(idx[:nd])
    ref_c_all, ref_i_all, roots_a, roots_b = [], [], [], []
    cbase = ebase = 0
    for k, (x, y) in enumerate(zip(pair.a, pair.b)):
        an, bn = np_of(x), np_of(y)
        la = oracle.leaves(an, C, eps, threads=th)
        lb = oracle.leaves(bn, C, eps, threads=th)
        na, nb = oracle.levels(la), oracle.levels(lb)
        assert np.array_equal(gpu_tree_nodes(TA, k), na), ("tree A", k)
        assert np.array_equal(gpu_tree_nodes(TB, k), nb), ("tree B", k)
        rc = oracle.diff(na, nb, la.shape[0])
        ri = oracle.verify(an, bn, C, rc, eps)
        if brute:
            assert np.array_equal(ri, oracle.brute(an, bn, eps)), k
        ref_c_all.append(rc + cbase)
        ref_i_all.append(ri + ebase)
        roots_a.append(na[-1])
        roots_b.append(nb[-1])
        cbase += la.shape[0]
        ebase += an.size
        del an, bn, la, lb, na, nb
    ref_c, ref_i = np.concatenate(ref_c_all), np.concatenate(ref_i_all)
    assert nc == ref_c.size and np.array_equal(got_c, ref_c)
    assert nd == ref_i.size and np.array_equal(got_i, ref_i)
    assert TA.root() == oracle.levels(np.stack(roots_a))[-1].tobytes()
    assert TB.root() == oracle.levels(np.stack(roots_b))[-1].tobytes()
    return nc, nd


def fused_compare(pair):
    """The bench step's call (ckpt_compare_pair_async, default 16-byte hash blocks)."""
    C, eps = pair.chunk_bytes, pair.eps
    L = sum(-(-t.numel() * t.element_size() // C) for t in pair.a)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(pair.a, pair.b, C, eps, chunks, idx, counts)
    TA.wait(); TB.wait()
    torch.cuda.synchronize()
    return TA, TB, chunks, idx, counts


@pytest.mark.slow
def test_config2_full_size_bench_path_parity():
    """BASELINE configs[1] at full size (2^26 particles x 6 f32 per run) through the exact call
    and launch configuration bench.py times (ckpt_compare_pair_async: the fused pair leaf kernel
    leaf_kernel<F32, 4096-byte chunks, PAIR>, K1 tile compaction read by verify_mark): every leaf
    and interior node of all 6 arrays of both trees, both checkpoint roots, the chunk list and
    the element ids equal the oracle's; the ids also equal brute force."""
    pair = synth.c2_pair(device="cuda")
    TA, TB, chunks, idx, counts = fused_compare(pair)
    nc, nd = full_checkpoint_parity(pair, TA, TB, chunks, idx, counts, brute=True)
    assert nc > 0 and nd > 0


# ------------------------------------------------ exhaustive f32 quantizer --

@pytest.mark.slow
@pytest.mark.parametrize("eps", [1e-3, 1e-6, 1e-8, 2.0 ** -10, 0.3])
def test_quantizer_exhaustive_f32(eps):
    """Every one of the 2^32 float32 bit patterns (NaNs, infinities, subnormals,
    both zeros) rounded by the GPU fast/slow paths vs the oracle, per eps: with
    16-byte chunks each leaf is Murmur3F(4 words, seed 0), so equal leaves mean
    equal words (barring a 2^-128 collision)."""
    slice_bits = 28
    per = 1 << slice_bits
    for s in range(1 << (32 - slice_bits)):
        bits = torch.arange(s * per, (s + 1) * per, dtype=torch.int64, device="cuda")
        x = bits.to(torch.int32).view(torch.float32)
        t = ck.tree_build(x, 16, eps)
        got = np_of(t.nodes()[: per // 4])
        ref = oracle.leaves(np_of(x), 16, eps, threads=os.cpu_count() or 8)
        bad = np.nonzero(np.any(got != ref, axis=1))[0]
        assert bad.size == 0, (s, bad[:4], np_of(x).reshape(-1, 4)[bad[:4]])
        del t, x, bits


def test_config5_shape_verify_heavy_bfs_path():
    """configs[4] shape at reduced size: many arrays, 10% of chunks with true differences and
    planted false positives; T small enough that the BFS starts above the leaves."""
    pair = synth.c5_pair(n_ranks=2, n_particles=1 << 16, seed=7, device="cuda")
    C, eps = pair.chunk_bytes, pair.eps
    TA, TB = ck.tree_build_batch([pair.a, pair.b], C, eps)
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    A = oracle.build_checkpoint(an, C, eps)
    B = oracle.build_checkpoint(bn, C, eps)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, C, ref_chunks, eps, A)
    assert np.array_equal(ref_idx, oracle.brute_checkpoint(an, bn, eps))
    for T in (0, 7, 1000):                  # default (leaf start) and mid-level starts
        chunks = torch.empty(TA.n_leaves, dtype=torch.int64, device="cuda")
        cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
        ck.tree_diff_async(TA, TB, chunks, cnt[0:1], T=T)
        idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
        ck.verify_async(pair.a, pair.b, chunks, cnt[0:1], C, eps, idx, cnt[1:2])
        nc, nd = cnt.tolist()
        assert np.array_equal(np_of(chunks[:nc]), ref_chunks), T
        assert np.array_equal(np_of(idx[:nd]), ref_idx), T
    # false positives exist (flagged chunks without a verified difference)
    per = C // 4
    assert np.setdiff1d(ref_chunks, np.unique(ref_idx // per)).size > 0


# ------------------------------------------------- fused pair compare path --

def _pair_cases():
    return [
        ("c1", lambda: synth.c1_pair(n=1 << 20, seed=21, device="cuda")),
        ("c1_tail", lambda: synth.c1_pair(n=1_000_003, seed=22, device="cuda")),
        ("c2_small", lambda: synth.c2_pair(n_particles=(1 << 18) + 77, seed=23, device="cuda")),
        ("c5_small", lambda: synth.c5_pair(n_ranks=2, n_particles=1 << 16, seed=24, device="cuda")),
        ("c3_small", lambda: synth.c3_pair(n=(1 << 20) + 5, seed=25, device="cuda", n_clusters=16,
                                           mean_len=512, n_isolated=500)),
        ("many_ragged", _many_ragged),
    ]


def _many_ragged():
    """20 arrays (device-resident array tables) of ragged sizes: 1 and 3 elements, one chunk,
    33 chunks, 4097 chunks (levels past one 7-level group), a partial 16-byte block."""
    sizes = [1, 3, 1024, 33 * 1024 + 1, 4097 * 1024, 5, 77_777, 1 << 16, 2, 129 * 1024 + 3,
             6, 1025, 99, 4 * 1024, 128 * 1024, 128 * 1024 + 1, 7, 16_383, 300_001, 11]
    a = [synth.uniform(700 + i, n, "cuda") * 2.0 - 1.0 for i, n in enumerate(sizes)]
    b = [t.clone() for t in a]
    for i, t in enumerate(b):
        t[(3 * i) % t.numel()::max(1, 997 + 31 * i)] += 1e-3 * (1 + (i % 3))
    return synth.Pair("many_ragged", a, b, 4096, 1e-5)


@pytest.mark.parametrize("name,make", _pair_cases(), ids=[c[0] for c in _pair_cases()])
@pytest.mark.parametrize("chunk", [4096, 512, 48])
def test_compare_pair_matches_oracle(name, make, chunk):
    pair = make()
    eps = pair.eps
    if name.startswith("c3") and chunk == 48:
        chunk = 64                                # f64: keep C a multiple of 16 and of 8
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    L = sum(-(-t.numel() * t.element_size() // chunk) for t in pair.a)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(pair.a, pair.b, chunk, eps, chunks, idx, counts)
    TA.wait(); TB.wait()
    torch.cuda.synchronize()
    A = oracle.build_checkpoint(an, chunk, eps, threads=8)
    B = oracle.build_checkpoint(bn, chunk, eps, threads=8)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, chunk, ref_chunks, eps, A)
    nc, nd = counts.tolist()
    assert np.array_equal(np_of(chunks[:nc]), ref_chunks)
    assert np.array_equal(np_of(idx[:nd]), ref_idx)
    # both trees are complete and equal the oracle's, array by array
    for k in range(len(an)):
        assert np.array_equal(gpu_tree_nodes(TA, k), A.trees[k]), k
        assert np.array_equal(gpu_tree_nodes(TB, k), B.trees[k]), k
    assert TA.root() == A.root and TB.root() == B.root


def test_compare_pair_equals_unfused_path_and_raw_mode():
    pair = synth.c2_pair(n_particles=(1 << 17) + 3, seed=31, device="cuda")
    for eps in (pair.eps, 0.0):
        L = sum(-(-t.numel() * 4 // 4096) for t in pair.a)
        n = sum(t.numel() for t in pair.a)
        outs = []
        for fused in (True, False):
            chunks = torch.empty(L, dtype=torch.int64, device="cuda")
            idx = torch.empty(n, dtype=torch.int64, device="cuda")
            counts = torch.zeros(2, dtype=torch.int64, device="cuda")
            if fused:
                TA, TB = ck.compare_pair_async(pair.a, pair.b, 4096, eps, chunks, idx, counts)
            else:
                TA, TB = ck.tree_build_batch([pair.a, pair.b], 4096, eps)
                ck.diff_verify_async(TA, TB, pair.a, pair.b, chunks, idx, counts)
            TA.wait(); TB.wait()
            nc, nd = counts.tolist()
            outs.append((np_of(chunks[:nc]), np_of(idx[:nd]), TA.root(), TB.root()))
        for x, y in zip(outs[0], outs[1]):
            assert np.array_equal(np.asarray(x), np.asarray(y)) if not isinstance(x, bytes) else x == y


def test_compare_pair_identical_and_truncated():
    a = [synth.uniform(41, 100_000, "cuda"), synth.uniform(42, 5_000, "cuda")]
    b = [t.clone() for t in a]
    chunks = torch.empty(200, dtype=torch.int64, device="cuda")
    idx = torch.empty(64, dtype=torch.int64, device="cuda")
    counts = torch.full((2,), 7, dtype=torch.int64, device="cuda")
    ck.compare_pair_async(a, b, 4096, 1e-6, chunks, idx, counts)
    assert counts.tolist() == [0, 0]
    b[0][::1000] += 1.0                                        # 100 elements
    ck.compare_pair_async(a, b, 4096, 1e-6, chunks, idx, counts)
    nc, nd = counts.tolist()
    ref = np.nonzero(np.abs(np_of(a[0]).astype(np.float64) - np_of(b[0]).astype(np.float64)) > 1e-6)[0]
    assert nc == np.unique(ref // 1024).size and nd == ref.size == 100   # full count past the cap
    assert np.array_equal(np_of(chunks[:nc]), np.unique(ref // 1024))
    assert np.array_equal(np_of(idx), ref[:64])
    with pytest.raises(ValueError):
        ck.compare_pair_async(a, [b[0]], 4096, 1e-6, chunks, idx, counts)


# K1 tile compaction (128 pair-tasks = 4096 chunks per tile) read by verify_mark
# (and, past 4096 tiles, placed by tile_gather_kernel): ragged arrays (pair-tasks
# of < 32 chunks), several tiles with a ragged last one, every chunk flagged, no
# chunk flagged, and a chunk-list cap that cuts through a tile -- all against the
# plain leaf comparison and brute force.
@pytest.mark.parametrize("mode", ["all", "none", "sparse", "cap"])
def test_compare_pair_tile_compaction(mode):
    sizes = [300 * 1024 + 5, 7 * 1024, 4096 * 1024 + 3, 1]       # f32 elements; C = 4 KiB
    a = [synth.uniform(90 + i, n, "cuda") for i, n in enumerate(sizes)]
    b = [t.clone() for t in a]
    if mode in ("all", "cap"):
        for t in b:
            t += 1.0                                              # every element differs
    elif mode == "sparse":
        for i, t in enumerate(b):
            t[(7 + 13 * i)::(5000 + 97 * i)] -= 0.5
    L = sum(-(-n * 4 // 4096) for n in sizes)
    n_el = sum(sizes)
    cap = 1500 if mode == "cap" else L
    chunks = torch.empty(cap, dtype=torch.int64, device="cuda")
    idx = torch.empty(n_el, dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(a, b, 4096, 1e-6, chunks, idx, counts)
    TA.wait(); TB.wait()
    nc, nd = counts.tolist()
    an = np.concatenate([np_of(t).astype(np.float64) for t in a])
    bn = np.concatenate([np_of(t).astype(np.float64) for t in b])
    hit = np.abs(an - bn) > 1e-6
    # chunk ids are global over the arrays in order (each array starts a new chunk)
    ids = []
    base_c = 0
    off = 0
    for n in sizes:
        h = np.nonzero(hit[off:off + n])[0]
        ids.append(base_c + np.unique(h // 1024))
        base_c += -(-n // 1024)
        off += n
    ref_chunks = np.concatenate(ids).astype(np.int64)
    assert nc == ref_chunks.size
    assert np.array_equal(np_of(chunks[:min(nc, cap)]), ref_chunks[:cap])
    if mode == "cap":
        # verify covers the first `cap` listed chunks only
        ref_idx = np.nonzero(hit)[0]
        lim = np.isin(np.concatenate([base + (np.arange(n) // 1024) for base, n in
                                      zip(np.cumsum([0] + [-(-n // 1024) for n in sizes])[:-1], sizes)]),
                      ref_chunks[:cap])
        ref_idx = np.nonzero(hit & lim)[0]
    else:
        ref_idx = np.nonzero(hit)[0]
    assert nd == ref_idx.size
    assert np.array_equal(np_of(idx[:nd]), ref_idx)


def test_compare_pair_tile_gather_path():
    """The gather kernel (used past 4096 tiles) in a fresh process with CKPT_TILE_GATHER=1."""
    import subprocess
    import sys
    code = (
        "import sys; sys.path.insert(0, %r); import test_gpu_parity as t; "
        "[t.test_compare_pair_tile_compaction(m) for m in ('all', 'none', 'sparse', 'cap')]; print('ok')"
        % os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, CKPT_TILE_GATHER="1")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                       cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=600)
    assert r.returncode == 0 and r.stdout.strip().endswith("ok"), r.stdout[-2000:] + r.stderr[-2000:]


@pytest.mark.parametrize("chunk", [1024, 2048, 8192, 16384, 32768, 65536])
@pytest.mark.parametrize("dt", [torch.float32, torch.float64])
def test_compare_pair_specialised_chunk_sizes(dt, chunk):
    """The fused pair kernels compiled for the configs[2] sweep's chunk sizes (every size of
    512 B..64 KiB has its own instantiation): ragged arrays (partial last chunk and partial last
    16-byte block), changes above and below eps, a flagged last chunk -- every node, the chunk
    list and the element ids equal the oracle's."""
    per = chunk // (4 if dt == torch.float32 else 8)
    sizes = [37 * per + 3, 5 * per, 1, 2 * per + per // 2 + 1]
    a = [_data(n, dt, 400 + i) for i, n in enumerate(sizes)]
    b = [t.clone() for t in a]
    b[0][per // 3::7 * per + 11] += 3e-6        # above eps = 1e-6
    b[0][5::3 * per + 1] += 2e-7                # below eps: straddles only
    b[1][-1] -= 1e-3
    b[3][-1] += 1.0                             # the flagged ragged last chunk
    pair = synth.Pair("specialised", a, b, chunk, 1e-6)
    TA, TB, chunks, idx, counts = fused_compare(pair)
    nc, nd = full_checkpoint_parity(pair, TA, TB, chunks, idx, counts, brute=True)
    assert nc > 2 and nd > 2


@pytest.mark.parametrize("dt,chunk", [(torch.float32, 2 << 20), (torch.float64, 4 << 20)])
def test_compare_pair_large_chunks(dt, chunk):
    """Multi-MiB chunks (several mask groups per chunk, few long chains) through the fused call:
    every node, the chunk list and the element ids equal the oracle's."""
    sizes = [3 * chunk // 8 + 5, chunk // 16, 2 * chunk // 4 + 1]
    a = [_data(n, dt, 300 + i) for i, n in enumerate(sizes)]
    b = [t.clone() for t in a]
    b[0][::100_003] += 1e-3
    b[2][-1] += 1.0
    pair = synth.Pair("fallback", a, b, chunk, 1e-6)
    TA, TB, chunks, idx, counts = fused_compare(pair)
    full_checkpoint_parity(pair, TA, TB, chunks, idx, counts, brute=True)


def test_compare_pair_repeated_and_alternating_shapes():
    """The self-resetting pair-task and tile counters and the epoch-tagged look-back states stay
    consistent over many compares on one stream, alternating between shapes: all exact."""
    p1 = synth.c1_pair(n=(1 << 19) + 3, seed=61, device="cuda")
    p2 = synth.c5_pair(n_ranks=1, n_particles=(1 << 15), seed=62, device="cuda")
    ref = {}
    for name, p in (("p1", p1), ("p2", p2)):
        an = [np_of(t) for t in p.a]
        bn = [np_of(t) for t in p.b]
        A = oracle.build_checkpoint(an, p.chunk_bytes, p.eps, threads=8)
        B = oracle.build_checkpoint(bn, p.chunk_bytes, p.eps, threads=8)
        rc = oracle.diff_checkpoint(A, B)
        ref[name] = (rc, oracle.verify_checkpoint(an, bn, p.chunk_bytes, rc, p.eps, A), A.root, B.root)
    for it in range(6):
        name, p = (("p1", p1), ("p2", p2))[it % 2]
        TA, TB, chunks, idx, counts = fused_compare(p)
        nc, nd = counts.tolist()
        rc, ri, ra, rb = ref[name]
        assert np.array_equal(np_of(chunks[:nc]), rc), (it, name)
        assert np.array_equal(np_of(idx[:nd]), ri), (it, name)
        assert TA.root() == ra and TB.root() == rb, (it, name)


# ------------------------------------------- hash block size variant (R23) --
# "the block size is variable and can be adjusted": every leaf,
# tree node, chunk list and element list equals the oracle at that block size.

HB_CASES = [
    # (n, dtype, chunk, eps, hash_block)
    (100_003, torch.float32, 4096, 1e-6, 0),      # whole chunk, ragged last chunk + tail
    ((1 << 18) + 3, torch.float32, 4096, 1e-5, 64),
    (70_001, torch.float32, 4096, 1e-5, 1024),
    (50_001, torch.float32, 4096, 1e-5, 48),      # does not divide C: exact path, short last block
    (4097, torch.float32, 512, 1e-5, 0),          # runtime chunk size, whole chunk
    (9_999, torch.float32, 48, 1e-4, 32),
    (123_457, torch.float64, 1024, 1e-8, 0),
    (123_457, torch.float64, 4096, 1e-8, 256),
    (10_001, torch.float32, 4096, 0.0, 0),        # raw-bit mode, whole chunk
    (10_001, torch.float64, 160, 0.0, 32),
]


@pytest.mark.parametrize("n,dtype,chunk,eps,hb", HB_CASES)
def test_hash_block_tree_bit_exact(n, dtype, chunk, eps, hb):
    a = _data(n, dtype, n + chunk + hb)
    t = ck.tree_build(a, chunk, eps, hash_block=hb)
    got = gpu_tree_nodes(t)
    lv = oracle.leaves(np_of(a), chunk, eps, threads=8, hash_block=hb)
    ref = oracle.levels(lv)
    bad = np.nonzero(np.any(got != ref, axis=1))[0]
    assert bad.size == 0, f"{bad.size} nodes differ, first {bad[:5]}"
    assert t.params()[3] == (chunk if hb == 0 or hb > chunk else hb)


def test_hash_block_special_values_take_the_exact_retry():
    a = synth.uniform(77, 1 << 16, "cuda") * 2.0 - 1.0
    a[5000] = float("nan"); a[20000] = float("inf"); a[40000] = 1e30
    for hb in (0, 64):
        got = gpu_tree_nodes(ck.tree_build(a, 4096, 1e-6, hash_block=hb))
        ref = oracle.levels(oracle.leaves(np_of(a), 4096, 1e-6, hash_block=hb))
        assert np.array_equal(got, ref), hb


@pytest.mark.parametrize("hb", [0, 64, 1024])
@pytest.mark.parametrize("name,make", _pair_cases()[:4], ids=[c[0] for c in _pair_cases()[:4]])
def test_compare_pair_hash_block_matches_oracle(name, make, hb):
    pair = make()
    eps, chunk = pair.eps, 4096
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    L = sum(-(-t.numel() * t.element_size() // chunk) for t in pair.a)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(pair.a, pair.b, chunk, eps, chunks, idx, counts, hash_block=hb)
    TA.wait(); TB.wait()
    torch.cuda.synchronize()
    A = oracle.build_checkpoint(an, chunk, eps, threads=8, hash_block=hb)
    B = oracle.build_checkpoint(bn, chunk, eps, threads=8, hash_block=hb)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, chunk, ref_chunks, eps, A)
    nc, nd = counts.tolist()
    assert np.array_equal(np_of(chunks[:nc]), ref_chunks)
    assert np.array_equal(np_of(idx[:nd]), ref_idx)
    for k in range(len(an)):
        assert np.array_equal(gpu_tree_nodes(TA, k), A.trees[k]), k
    assert TA.root() == A.root and TB.root() == B.root
    # same flagged chunks as the paper's default 16-byte blocks (barring collisions)
    A16 = oracle.build_checkpoint(an, chunk, eps, threads=8)
    B16 = oracle.build_checkpoint(bn, chunk, eps, threads=8)
    assert np.array_equal(ref_chunks, oracle.diff_checkpoint(A16, B16))


def test_hash_block_mismatch_and_invalid():
    a = synth.uniform(5, 10_000, "cuda")
    t16 = ck.tree_build(a, 4096, 1e-5)
    t0 = ck.tree_build(a, 4096, 1e-5, hash_block=0)
    t4k = ck.tree_build(a, 4096, 1e-5, hash_block=8192)       # >= C: the whole chunk too
    assert t0.root() == t4k.root() != t16.root()
    assert ck.tree_diff(t0, t4k).numel() == 0
    with pytest.raises(ck.CkptError) as e:
        ck.tree_diff(t16, t0)
    assert e.value.status == ck.EMISMATCH
    with pytest.raises(ck.CkptError) as e:
        ck.tree_build(a, 4096, 1e-5, hash_block=24)
    assert e.value.status == ck.EINVAL


# --------------------------------------------------- tree persistence ------

def test_serialize_matches_documented_format_and_roundtrips():
    from tests.treefmt import oracle_tree_bytes
    pair = synth.c2_pair(n_particles=(1 << 15) + 9, seed=61, device="cuda")
    an = [np_of(t) for t in pair.a]
    for hb in (16, 0):
        t = ck.tree_build(pair.a, 4096, pair.eps, hash_block=hb)
        blob = t.serialize()
        A = oracle.build_checkpoint(an, 4096, pair.eps, hash_block=hb)
        ref = oracle_tree_bytes(A, [x.size for x in an], 0, 4096, pair.eps, 4096 if hb == 0 else hb)
        assert blob == ref                                  # byte-exact against the oracle's tree
        t2 = ck.tree_deserialize(blob)
        assert t2.root() == t.root() == A.root
        assert t2.params() == t.params()
        for k in range(len(an)):
            assert np.array_equal(gpu_tree_nodes(t2, k), A.trees[k])
        assert t2.serialize() == blob
        assert ck.tree_diff(t, t2).numel() == 0


def test_oracle_written_tree_diffs_against_live_tree():
    # a tree written by the oracle (documented format) loads and diffs like a GPU-built one
    from tests.treefmt import oracle_tree_bytes
    pair = synth.c5_pair(n_ranks=1, n_particles=1 << 16, seed=62, device="cuda")
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    A = oracle.build_checkpoint(an, 4096, pair.eps)
    B = oracle.build_checkpoint(bn, 4096, pair.eps)
    ta = ck.tree_deserialize(oracle_tree_bytes(A, [x.size for x in an], 0, 4096, pair.eps))
    tb = ck.tree_build(pair.b, 4096, pair.eps)
    ref = oracle.diff_checkpoint(A, B)
    assert np.array_equal(np_of(ck.tree_diff(ta, tb)), ref)
    for T in (1, 100):                                      # mid-level BFS over a loaded tree
        chunks = torch.empty(ta.n_leaves, dtype=torch.int64, device="cuda")
        cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
        ck.tree_diff_async(ta, tb, chunks, cnt, T=T)
        assert np.array_equal(np_of(chunks[: int(cnt.item())]), ref), T


@pytest.mark.parametrize("host_a", [False, True])
def test_compare_saved_matches_oracle(host_a, tmp_path):
    pair = synth.c2_pair(n_particles=(1 << 17) + 5, seed=63, device="cuda")
    eps, C = pair.eps, 4096
    path = str(tmp_path / "runA.ckpttree")
    ck.tree_build(pair.a, C, eps).save(path)
    saved = open(path, "rb").read()
    a_data = [t.cpu().pin_memory() for t in pair.a] if host_a else pair.a
    L = sum(-(-t.numel() * 4 // C) for t in pair.a)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_saved(saved, a_data, pair.b, chunks, idx, counts)
    torch.cuda.synchronize()
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    A = oracle.build_checkpoint(an, C, eps, threads=8)
    B = oracle.build_checkpoint(bn, C, eps, threads=8)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, C, ref_chunks, eps, A)
    nc, nd = counts.tolist()
    assert nc > 0 and nd > 0
    assert np.array_equal(np_of(chunks[:nc]), ref_chunks)
    assert np.array_equal(np_of(idx[:nd]), ref_idx)
    assert TA.root() == A.root and TB.root() == B.root
    # shape mismatch with the stored tree
    with pytest.raises(ck.CkptError) as e:
        ck.compare_saved(saved, [t[:-4] for t in pair.a], [t[:-4] for t in pair.b], chunks, idx, counts)
    assert e.value.status == ck.EMISMATCH


# ------------------------------------------- config 4 snapshot shard shape --

@pytest.mark.parametrize("snapshot", range(10))
def test_c4_snapshot_shard_matches_oracle(snapshot):
    # BASELINE configs[3]: a GPU's shard of HACC ranks of one snapshot (reduced particle count)
    pair = synth.c4_snapshot(snapshot, range(3, 6), n_particles=(1 << 16) + 5, device="cuda")
    eps, C = pair.eps, 4096
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    L = sum(-(-t.numel() * 4 // C) for t in pair.a)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(pair.a, pair.b, C, eps, chunks, idx, counts)
    TA.wait(); TB.wait()
    A = oracle.build_checkpoint(an, C, eps, threads=8)
    B = oracle.build_checkpoint(bn, C, eps, threads=8)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, C, ref_chunks, eps, A)
    assert np.array_equal(ref_idx, oracle.brute_checkpoint(an, bn, eps))
    nc, nd = counts.tolist()
    assert np.array_equal(np_of(chunks[:nc]), ref_chunks)
    assert np.array_equal(np_of(idx[:nd]), ref_idx)
    assert TA.root() == A.root and TB.root() == B.root
    # at this reduced size the planted fraction rounds to zero particles up to snapshot 4
    planted = any(cl for cl in pair.meta["clusters"].values())
    if not planted:
        assert nc == 0 and nd == 0
    if snapshot == 9:
        assert planted and nc > 0 and nd > 0


@pytest.mark.slow
def test_c4_every_snapshot_full_size_rank_bench_path():
    """BASELINE configs[3] as bench.py --config c4 --snapshots all runs it: every one of the 10
    snapshots (divergence 0 for s <= 2, then 1e-6 * 4^(s-3) of the particles) on one full-size
    HACC rank (2^24 particles x 6 f32 per run), through the fused call; every node of both trees,
    the roots, the chunk list and the element ids equal the oracle's.  The ranks differ per
    snapshot so the sample covers 10 of the 64."""
    for s in range(10):
        pair = synth.c4_snapshot(s, [(7 * s + 3) % 64], n_particles=1 << 24, device="cuda")
        TA, TB, chunks, idx, counts = fused_compare(pair)
        nc, nd = full_checkpoint_parity(pair, TA, TB, chunks, idx, counts, brute=False)
        if s <= 2:
            assert nc == 0 and nd == 0
        del TA, TB, pair


# --------------------------------- one array sharded over GPUs (8e, opt) ----

@pytest.mark.parametrize("world", [2, 3, 8])
def test_array_shards_reassemble_single_gpu_results(world):
    # every rank's work done in turn on one GPU: shard subtrees + top tree over the shard roots
    from paper_conf_middleware_tanaabcrtn24_b200 import dist as ckd
    pair = synth.c3_pair(n=(1 << 20) + 77, seed=71, device="cuda", n_clusters=24, mean_len=300)
    a, b = pair.a[0], pair.b[0]
    C, eps = 2048, pair.eps
    whole = ck.compare(a, b, C, eps)
    roots_a, roots_b, chunks, idx = [], [], [], []
    for r in range(world):
        lo, hi, c_lo, _ = ckd.array_shard(a.numel(), 8, C, world, r)
        if hi == lo:
            continue
        L = -(-(hi - lo) * 8 // C)
        ch = torch.empty(L, dtype=torch.int64, device="cuda")
        ix = torch.empty(hi - lo, dtype=torch.int64, device="cuda")
        cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
        TA, TB = ck.compare_pair_async([a[lo:hi]], [b[lo:hi]], C, eps, ch, ix, cnt)
        roots_a.append(TA.array_roots()); roots_b.append(TB.array_roots())
        nc, nd = cnt.tolist()
        chunks.append(ch[:nc] + c_lo); idx.append(ix[:nd] + lo)
    assert ck.tree_from_digests(torch.cat(roots_a)).root() == whole[4]
    assert ck.tree_from_digests(torch.cat(roots_b)).root() == whole[5]
    assert torch.equal(torch.cat(chunks), whole[0])
    assert torch.equal(torch.cat(idx), whole[1])


# -------------------------------------------- out-of-core streaming (f3) ----

@pytest.mark.parametrize("seg", [4096, 1 << 16, 3 * 4096 + 100, 1 << 30])
@pytest.mark.parametrize("pinned", [True, False])
def test_compare_stream_matches_oracle(seg, pinned):
    pair = synth.c5_pair(n_ranks=1, n_particles=(1 << 15) + 300, seed=81, device="cpu")
    C, eps = 4096, pair.eps
    ha = [t.pin_memory() if pinned else t for t in pair.a]
    hb = [t.pin_memory() if pinned else t for t in pair.b]
    chunks, idx, nc, nd, ra, rb = ck.compare_stream(ha, hb, C, eps, segment_bytes=seg)
    an = [t.numpy() for t in pair.a]
    bn = [t.numpy() for t in pair.b]
    A = oracle.build_checkpoint(an, C, eps, threads=8)
    B = oracle.build_checkpoint(bn, C, eps, threads=8)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, C, ref_chunks, eps, A)
    assert nc == ref_chunks.size and nd == ref_idx.size and nd > 0
    assert np.array_equal(chunks.numpy(), ref_chunks)
    assert np.array_equal(idx.numpy(), ref_idx)
    assert ra == A.root and rb == B.root


def test_compare_stream_f64_hash_block_and_truncation():
    pair = synth.c3_pair(n=(1 << 18) + 3, seed=82, device="cpu", n_clusters=12, mean_len=200)
    C, eps = 1024, pair.eps
    an, bn = [pair.a[0].numpy()], [pair.b[0].numpy()]
    A = oracle.build_checkpoint(an, C, eps, hash_block=0)
    B = oracle.build_checkpoint(bn, C, eps, hash_block=0)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, C, ref_chunks, eps, A)
    chunks, idx, nc, nd, ra, rb = ck.compare_stream(pair.a, pair.b, C, eps, segment_bytes=50_000,
                                                    hash_block=0)
    assert np.array_equal(chunks.numpy(), ref_chunks) and np.array_equal(idx.numpy(), ref_idx)
    assert ra == A.root and rb == B.root
    # truncated outputs keep the ascending prefix and the full counts
    chunks, idx, nc, nd, _, _ = ck.compare_stream(pair.a, pair.b, C, eps, segment_bytes=50_000,
                                                  hash_block=0, chunks_cap=5, idx_cap=7)
    assert nc == ref_chunks.size and nd == ref_idx.size
    assert np.array_equal(chunks.numpy(), ref_chunks[:5]) and np.array_equal(idx.numpy(), ref_idx[:7])


# ------------------------------------------- maximum sizes (64-bit ids) ----

@pytest.mark.slow
def test_array_beyond_2pow32_elements_fused_path():
    """One f32 array of 2^32 + 4099 elements (17.2 GB per run; element ids and byte offsets
    beyond 32 bits, ragged last chunk) on the fused pair path: chunk list and element ids equal
    the oracle's on every perturbed chunk, leaves of sampled chunks (incl. both sides of the
    2^32-element boundary and the last chunk) equal the oracle's, every interior level equals
    the oracle's levels over the GPU leaves, and b == a outside the perturbed elements."""
    n = (1 << 32) + 4099
    C, eps = 4096, 1e-6
    per = C // 4
    a = torch.empty(n, dtype=torch.float32, device="cuda")
    step = 1 << 28
    for o in range(0, n, step):
        m = min(step, n - o)
        a[o:o + m] = synth.uniform(91, m, "cuda", offset=o) * 2.0 - 1.0
    b = a.clone()
    rng = np.random.default_rng(91)
    pos = np.unique(np.concatenate([rng.integers(0, n, 40), rng.integers(1 << 32, n, 16),
                                    [n - 1, (1 << 32) - 1, 1 << 32, 0]]))
    mag = rng.uniform(0.05, 20.0, pos.size) * eps * np.where(rng.random(pos.size) < 0.5, -1, 1)
    ip = torch.as_tensor(pos, dtype=torch.int64, device="cuda")
    b[ip] = (a[ip].double() + torch.as_tensor(mag, device="cuda")).float()
    changed = np_of(torch.nonzero(a != b).view(-1))
    assert np.isin(changed, pos).all() and changed.size > 40
    L = -(-n * 4 // C)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(1 << 16, dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async([a], [b], C, eps, chunks, idx, counts)
    TA.wait(); TB.wait()
    nc, nd = counts.tolist()
    # expected: only perturbed chunks can differ; the oracle decides each of them
    cand = np.unique(pos // per)
    ref_chunks, ref_idx = [], []
    for c in cand:
        lo, hi = c * per, min(n, (c + 1) * per)
        ca, cb = np_of(a[lo:hi]), np_of(b[lo:hi])
        if not np.array_equal(oracle.leaves(ca, C, eps), oracle.leaves(cb, C, eps)):
            ref_chunks.append(c)
            ref_idx.extend((oracle.brute(ca, cb, eps) + lo).tolist())
    assert nc == len(ref_chunks) and np.array_equal(np_of(chunks[:nc]), np.array(ref_chunks))
    assert nd == len(ref_idx) and np.array_equal(np_of(idx[:nd]), np.array(ref_idx))
    assert max(ref_idx) >= (1 << 32)
    # leaves of sampled chunks + every interior level of tree A
    na = gpu_tree_nodes(TA, 0)
    sample = np.unique(np.concatenate([rng.integers(0, L, 64), [0, L - 1, (1 << 32) // per - 1,
                                                                (1 << 32) // per]]))
    for c in sample:
        lo, hi = c * per, min(n, (c + 1) * per)
        assert np.array_equal(oracle.leaves(np_of(a[lo:hi]), C, eps)[0], na[c]), c
    assert np.array_equal(oracle.levels(na[:L]), na)
    del a, b


@pytest.mark.slow
def test_config5_full_size_parity():
    """BASELINE configs[4] per-GPU shard at full size (8 ranks x 50*2^20 particles x 6 f32,
    10 GB per run, verify-heavy: 10% of chunks with true differences, 1% planted false
    positives) through the bench's fused call: every node of all 48 arrays of both trees, both
    roots, the chunk list and the element ids equal the oracle's, and the element count equals a
    device brute-force count of |a-b| > eps over all 2.6e9 element pairs."""
    pair = synth.c5_pair(device="cuda")
    TA, TB, chunks, idx, counts = fused_compare(pair)
    brute = 0
    for x, y in zip(pair.a, pair.b):
        brute += int((x.double() - y.double()).abs().gt(pair.eps).sum().item())
    nc, nd = full_checkpoint_parity(pair, TA, TB, chunks, idx, counts, brute=False)
    assert nd == brute
    # false positives by construction: flagged chunks with no verified difference
    per = pair.chunk_bytes // 4
    got_c = np_of(chunks[:nc])
    got_i = np_of(idx[:nd])
    elem_base = np.cumsum([0] + [t.numel() for t in pair.a])
    chunk_base = np.cumsum([0] + [-(-t.numel() * 4 // pair.chunk_bytes) for t in pair.a])
    arr = np.searchsorted(elem_base, got_i, side="right") - 1
    hit_chunks = np.unique(chunk_base[arr] + (got_i - elem_base[arr]) // per)
    assert np.setdiff1d(got_c, hit_chunks).size > 0


@pytest.mark.slow
@pytest.mark.parametrize("C", [512, 4096, 65536])
def test_config3_full_size_parity(C):
    """BASELINE configs[2] at full size (2^29 f64 ~ N(0,1), 4 GiB per run, 1024 clustered
    divergences) on the fused pair path the bench times, at the smallest, default and largest
    chunk of the sweep: EVERY leaf of both trees equals the oracle's (full-array oracle leaves),
    every interior level equals the oracle's levels over them, and the chunk list and element
    ids equal the oracle's diff + verify; the element count also equals a device brute-force
    count of |a-b| > eps."""
    pair = synth.c3_pair(device="cuda")
    eps, n = pair.eps, pair.a[0].numel()
    a, b = pair.a[0], pair.b[0]
    L = -(-n * 8 // C)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(1 << 24, dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async([a], [b], C, eps, chunks, idx, counts)
    TA.wait(); TB.wait()
    nc, nd = counts.tolist()
    assert nd == int((a - b).abs().gt(eps).sum().item()) and 0 < nd <= idx.numel()
    an, bn = np_of(a), np_of(b)
    th = os.cpu_count() or 8
    la, lb = oracle.leaves(an, C, eps, threads=th), oracle.leaves(bn, C, eps, threads=th)
    na, nb = gpu_tree_nodes(TA), gpu_tree_nodes(TB)
    assert np.array_equal(na[:L], la) and np.array_equal(nb[:L], lb)
    assert np.array_equal(oracle.levels(la), na) and np.array_equal(oracle.levels(lb), nb)
    ref_c = np.nonzero(np.any(la != lb, axis=1))[0]
    ref_i = oracle.verify(an, bn, C, ref_c, eps)
    assert nc == ref_c.size and np.array_equal(np_of(chunks[:nc]), ref_c)
    assert nd == ref_i.size and np.array_equal(np_of(idx[:nd]), ref_i)
    del a, b, pair


# -------------------------- latency variant of the leaf kernel (few chains) --

@pytest.mark.parametrize("dt,chunk,n,eps", [(torch.float32, 16384, (1 << 22) + 5, 1e-6),
                                            (torch.float64, 65536, (1 << 21) + 3, 1e-8),
                                            (torch.float32, 32768, 300_001, 0.0)])
def test_large_chunk_latency_variant_matches_oracle(dt, chunk, n, eps):
    # few long chains -> one-warp CTAs of the LAT instantiation (pair and single-tree paths)
    a = _data(n, dt, 5 + chunk)
    b = a.clone()
    b[:: 40_000] += 1e-3
    L = -(-n * a.element_size() // chunk)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(n, dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async([a], [b], chunk, eps, chunks, idx, counts)
    TA.wait(); TB.wait()
    an, bn = np_of(a), np_of(b)
    la, lb = oracle.leaves(an, chunk, eps, threads=8), oracle.leaves(bn, chunk, eps, threads=8)
    na, nb = oracle.levels(la), oracle.levels(lb)
    assert np.array_equal(gpu_tree_nodes(TA), na) and np.array_equal(gpu_tree_nodes(TB), nb)
    ref_c = oracle.diff(na, nb, L)
    ref_i = oracle.verify(an, bn, chunk, ref_c, eps)
    nc, nd = counts.tolist()
    assert np.array_equal(np_of(chunks[:nc]), ref_c) and np.array_equal(np_of(idx[:nd]), ref_i)
    assert np.array_equal(gpu_tree_nodes(ck.tree_build(a, chunk, eps)), na)


# ------------------------------------------ verify work-buffer reuse (emit) --

@pytest.mark.parametrize("dt,chunk", [(torch.float32, 65536), (torch.float64, 16384)])
def test_flagged_ragged_last_chunk_after_dense_verify(dt, chunk):
    """A flagged short last chunk (fewer than chunk/elem_size elements, chunk > 1024 elements)
    must emit only its own ids although the verify work buffer still holds the all-ones masks
    of a previous, fully differing compare on the same stream."""
    n = 70_001
    a = _data(n, dt, 17)
    L = -(-n * a.element_size() // chunk)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(n, dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async([a], [a + 1.0], chunk, 1e-6, chunks, idx, counts)
    TA.wait(); TB.wait()
    assert counts.tolist() == [L, n]
    b = a.clone()
    b[-1] += 1.0
    TA, TB = ck.compare_pair_async([a], [b], chunk, 1e-6, chunks, idx, counts)
    TA.wait(); TB.wait()
    assert counts.tolist() == [1, 1]
    assert chunks[0].item() == L - 1 and idx[0].item() == n - 1


def test_async_wrappers_validate_output_buffers():
    a = _data(1 << 12, torch.float32, 3)
    good = torch.empty(64, dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    with pytest.raises(TypeError):
        ck.compare_pair_async([a], [a], 4096, 1e-6, good.int(), good, counts)
    with pytest.raises(ValueError):
        ck.compare_pair_async([a], [a], 4096, 1e-6, good, good, counts[:1])
    with pytest.raises(ValueError):
        ck.compare_pair_async([a], [a], 4096, 1e-6, good[::2], good, counts)
    with pytest.raises(ValueError):
        ck.compare_pair_async([a], [a], 4096, 1e-6, good.cpu(), good, counts)
    with pytest.raises(ValueError):
        ck.verify_async([a], [a], good, counts[:0], 4096, 1e-6, good, counts[1:])
