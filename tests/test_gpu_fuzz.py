"""Randomised GPU parity (deterministic seeds): many small checkpoint pairs drawn across the input
space -- dtype, number and lengths of arrays (ragged tails, single elements), chunk size (every
specialised size and arbitrary multiples of 16), eps (0 = raw bits, tiny, huge), hash block,
special values (NaN, +-inf, -0, subnormals, values beyond the fast rounding range) and changes
above, below and straddling eps -- through the fused pair call and the unfused build/diff/verify
calls, compared with the oracle: every tree node, both roots, the chunk list and the element ids.
"""
import numpy as np
import pytest
import torch

import oracle

pytestmark = pytest.mark.gpu

ck = pytest.importorskip("paper_conf_middleware_tanaabcrtn24_b200")

SPECIALISED = [512, 1024, 2048, 4096, 8192, 16384, 32768, 65536]


def _case(seed, arrays=(1, 5)):
    rng = np.random.default_rng(1000 + seed)
    dt = np.float32 if rng.random() < 0.6 else np.float64
    esz = np.dtype(dt).itemsize
    if rng.random() < 0.5:
        chunk = int(rng.choice(SPECIALISED))
    else:
        chunk = 16 * int(rng.integers(1, 300))
    r = rng.random()
    eps = 0.0 if r < 0.1 else float(10.0 ** rng.uniform(-12, 2))
    hb = 16 if rng.random() < 0.7 else int(rng.choice([0, 32, 48, 64, 256]))
    if hb and hb > chunk:
        hb = 0
    m = int(rng.integers(*arrays))
    per = chunk // esz
    a_list, b_list = [], []
    for k in range(m):
        shape = rng.random()
        if shape < 0.15:
            n = int(rng.integers(1, 8))                       # a few elements: partial 16-byte block
        elif shape < 0.4:
            n = int(per * rng.integers(1, 40) + rng.integers(0, per))   # ragged last chunk
        else:
            n = int(10 ** rng.uniform(2, 5.3))
        scale = float(10.0 ** rng.uniform(-3, 6))
        a = (rng.standard_normal(n) * scale).astype(dt)
        if rng.random() < 0.3:                                # special values
            sp = np.array([np.nan, np.inf, -np.inf, -0.0, 0.0, np.finfo(dt).tiny / 4,
                           np.finfo(dt).max, -np.finfo(dt).max], dtype=dt)
            pos = rng.integers(0, n, size=min(n, 6))
            a[pos] = rng.choice(sp, size=pos.size)
        b = a.copy()
        n_ch = int(rng.integers(0, max(1, n // 50) + 1))
        if n_ch:
            pos = rng.integers(0, n, size=n_ch)
            unit = eps if eps > 0 else 1e-3
            mag = unit * (10.0 ** rng.uniform(-2, 2, size=n_ch))
            sign = np.where(rng.random(n_ch) < 0.5, -1.0, 1.0)
            b[pos] = (b[pos].astype(np.float64) + sign * mag).astype(dt)
        a_list.append(a)
        b_list.append(b)
    return dt, chunk, eps, hb, a_list, b_list


def _oracle(a_list, b_list, chunk, eps, hb):
    A = oracle.build_checkpoint(a_list, chunk, eps, threads=8, hash_block=hb)
    B = oracle.build_checkpoint(b_list, chunk, eps, threads=8, hash_block=hb)
    rc = oracle.diff_checkpoint(A, B)
    ri = oracle.verify_checkpoint(a_list, b_list, chunk, rc, eps, A)
    return A, B, rc, ri


def _check_trees(TA, TB, A, B):
    for k in range(len(A.trees)):
        assert np.array_equal(TA.nodes(k).cpu().numpy(), A.trees[k]), ("A", k)
        assert np.array_equal(TB.nodes(k).cpu().numpy(), B.trees[k]), ("B", k)
    assert TA.root() == A.root and TB.root() == B.root


@pytest.mark.parametrize("seed", range(200))
def test_fuzz_fused_pair_matches_oracle(seed):
    dt, chunk, eps, hb, a_list, b_list = _case(seed)
    A, B, rc, ri = _oracle(a_list, b_list, chunk, eps, hb)
    ta = [torch.from_numpy(x).cuda() for x in a_list]
    tb = [torch.from_numpy(x).cuda() for x in b_list]
    L = sum(A.n_leaves)
    chunks = torch.empty(max(L, 1), dtype=torch.int64, device="cuda")
    idx = torch.empty(max(sum(x.size for x in a_list), 1), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(ta, tb, chunk, eps, chunks, idx, counts, hash_block=hb)
    TA.wait(); TB.wait()
    torch.cuda.synchronize()
    nc, nd = counts.tolist()
    assert nc == rc.size and np.array_equal(chunks[:nc].cpu().numpy(), rc), (dt, chunk, eps, hb)
    assert nd == ri.size and np.array_equal(idx[:nd].cpu().numpy(), ri), (dt, chunk, eps, hb)
    _check_trees(TA, TB, A, B)


@pytest.mark.parametrize("seed", range(200, 260))
def test_fuzz_unfused_calls_match_oracle(seed):
    dt, chunk, eps, hb, a_list, b_list = _case(seed)
    A, B, rc, ri = _oracle(a_list, b_list, chunk, eps, hb)
    ta = [torch.from_numpy(x).cuda() for x in a_list]
    tb = [torch.from_numpy(x).cuda() for x in b_list]
    TA, TB = ck.tree_build_batch([ta, tb], chunk, eps, hash_block=hb)
    chunks = torch.empty(max(sum(A.n_leaves), 1), dtype=torch.int64, device="cuda")
    idx = torch.empty(max(sum(x.size for x in a_list), 1), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    ck.diff_verify_async(TA, TB, ta, tb, chunks, idx, counts)
    torch.cuda.synchronize()
    nc, nd = counts.tolist()
    assert nc == rc.size and np.array_equal(chunks[:nc].cpu().numpy(), rc), (dt, chunk, eps, hb)
    assert nd == ri.size and np.array_equal(idx[:nd].cpu().numpy(), ri), (dt, chunk, eps, hb)
    _check_trees(TA, TB, A, B)


@pytest.mark.parametrize("seed", range(300, 340))
def test_fuzz_stream_host_and_saved_paths_match_oracle(seed):
    """The same random pairs through the host-data paths: streamed through the device ring with
    a random (chunk-aligned) segment size, staged, and compared against a stored tree of run A."""
    dt, chunk, eps, hb, a_list, b_list = _case(seed)
    A, B, rc, ri = _oracle(a_list, b_list, chunk, eps, hb)
    rng = np.random.default_rng(seed)
    ha = [torch.from_numpy(x).pin_memory() for x in a_list]
    hb_ = [torch.from_numpy(x).pin_memory() for x in b_list]
    seg = int(chunk * rng.integers(1, 9))
    c_s, i_s, nc, nd, root_a, root_b = ck.compare_stream(ha, hb_, chunk, eps, segment_bytes=seg,
                                                          hash_block=hb)
    assert nc == rc.size and np.array_equal(c_s[:nc].numpy(), rc), (dt, chunk, eps, hb, seg)
    assert nd == ri.size and np.array_equal(i_s[:nd].numpy(), ri), (dt, chunk, eps, hb, seg)
    assert root_a == A.root and root_b == B.root
    if hb == 16:                       # compare_host and compare_saved use the default blocks
        i_h, nc_h, nd_h, ra, rb = ck.compare_host(ha, hb_, chunk, eps)
        assert (nc_h, nd_h) == (rc.size, ri.size) and np.array_equal(i_h[:nd_h].numpy(), ri)
        assert ra == A.root and rb == B.root
        ta0 = ck.tree_build([torch.from_numpy(x).cuda() for x in a_list], chunk, eps)
        blob = ta0.serialize()
        tb = [torch.from_numpy(x).cuda() for x in b_list]
        chunks = torch.empty(max(sum(A.n_leaves), 1), dtype=torch.int64, device="cuda")
        idx = torch.empty(max(sum(x.size for x in a_list), 1), dtype=torch.int64, device="cuda")
        counts = torch.zeros(2, dtype=torch.int64, device="cuda")
        TA, TB = ck.compare_saved(blob, ha, tb, chunks, idx, counts)
        torch.cuda.synchronize()
        n1, n2 = counts.tolist()
        assert n1 == rc.size and np.array_equal(chunks[:n1].cpu().numpy(), rc)
        assert n2 == ri.size and np.array_equal(idx[:n2].cpu().numpy(), ri)
        assert TA.root() == A.root and TB.root() == B.root


@pytest.mark.parametrize("seed", range(400, 430))
def test_fuzz_mid_level_bfs_matches_oracle(seed):
    """The BFS diff from a random start level (threshold T) equals the oracle's chunk list."""
    dt, chunk, eps, hb, a_list, b_list = _case(seed)
    A, B, rc, _ = _oracle(a_list, b_list, chunk, eps, hb)
    rng = np.random.default_rng(seed)
    ta = [torch.from_numpy(x).cuda() for x in a_list]
    tb = [torch.from_numpy(x).cuda() for x in b_list]
    TA, TB = ck.tree_build_batch([ta, tb], chunk, eps, hash_block=hb)
    chunks = torch.empty(max(sum(A.n_leaves), 1), dtype=torch.int64, device="cuda")
    count = torch.zeros(1, dtype=torch.int64, device="cuda")
    for T in (1, int(rng.integers(2, 64)), int(rng.integers(64, 1 << 16))):
        ck.tree_diff_async(TA, TB, chunks, count, T=T)
        torch.cuda.synchronize()
        n = int(count.item())
        assert n == rc.size and np.array_equal(chunks[:n].cpu().numpy(), rc), (T, dt, chunk)


@pytest.mark.parametrize("seed", range(500, 516))
def test_fuzz_many_arrays_device_tables(seed):
    """17-80 arrays per checkpoint: the leaf, levels and verify kernels read their array tables
    from device memory instead of the kernel parameters."""
    dt, chunk, eps, hb, a_list, b_list = _case(seed, arrays=(17, 81))
    A, B, rc, ri = _oracle(a_list, b_list, chunk, eps, hb)
    ta = [torch.from_numpy(x).cuda() for x in a_list]
    tb = [torch.from_numpy(x).cuda() for x in b_list]
    chunks = torch.empty(max(sum(A.n_leaves), 1), dtype=torch.int64, device="cuda")
    idx = torch.empty(max(sum(x.size for x in a_list), 1), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(ta, tb, chunk, eps, chunks, idx, counts, hash_block=hb)
    TA.wait(); TB.wait()
    torch.cuda.synchronize()
    nc, nd = counts.tolist()
    assert nc == rc.size and np.array_equal(chunks[:nc].cpu().numpy(), rc), (len(a_list), chunk)
    assert nd == ri.size and np.array_equal(idx[:nd].cpu().numpy(), ri), (len(a_list), chunk)
    _check_trees(TA, TB, A, B)
