"""GPU parity of the pipelined pair-sequence call (ckpt_compare_pairs_async) vs the oracle.

A sequence of checkpoint pairs (the snapshots of two runs' histories, PAPER.md:212-217,
:738-741) is compared pair by pair; pair p's verify runs on the library's verify stream while
pair p+1's leaf kernel runs, and the K1 tile buffers rotate over 3 slots.  Every pair's chunk
list, element ids, counts and both trees must equal the oracle's, whatever the sequence length
(more pairs than slots), the shapes of neighbouring pairs, output aliasing, and interleaving with
the non-pipelined call on the same stream.
"""
import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

ck = pytest.importorskip("paper_conf_middleware_tanaabcrtn24_b200")


def np_of(t):
    return t.detach().cpu().numpy()


def _outputs(pair, chunk):
    L = sum(-(-t.numel() * t.element_size() // chunk) for t in pair.a)
    return (torch.empty(L, dtype=torch.int64, device="cuda"),
            torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda"),
            torch.zeros(2, dtype=torch.int64, device="cuda"))


def _check_pair(pair, chunk, TA, TB, chunks, idx, counts):
    an = [np_of(t) for t in pair.a]
    bn = [np_of(t) for t in pair.b]
    A = oracle.build_checkpoint(an, chunk, pair.eps, threads=8)
    B = oracle.build_checkpoint(bn, chunk, pair.eps, threads=8)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(an, bn, chunk, ref_chunks, pair.eps, A)
    nc, nd = counts.tolist()
    assert nc == ref_chunks.size and np.array_equal(np_of(chunks[:nc]), ref_chunks)
    assert nd == ref_idx.size and np.array_equal(np_of(idx[:nd]), ref_idx)
    for k in range(len(an)):
        assert np.array_equal(np_of(TA.nodes(k)), A.trees[k]), ("A", k)
        assert np.array_equal(np_of(TB.nodes(k)), B.trees[k]), ("B", k)
    assert TA.root() == A.root and TB.root() == B.root
    return nc, nd


def _sequence():
    """Seven 2-array f32 pairs (more than the 3 tile slots) of different lengths and
    divergence: c2-shaped particle fields, an identical pair, a one-chunk pair, a ragged one."""
    out = []
    for p, n in enumerate([(1 << 17) + 3, 1 << 16, 5000, 1, (1 << 18) + 77, 4096 * 9 + 1, 70_001]):
        a = [synth.uniform(900 + 2 * p, n, "cuda") * 256.0,
             synth.normal(901 + 2 * p, n, "cuda") * 300.0]
        b = [t.clone() for t in a]
        if p != 1:   # pair 1 identical
            for i, t in enumerate(b):
                step = max(1, 997 + 101 * p + 31 * i)
                t[(5 * p + i) % n::step] += (1e-3 if (p + i) % 2 else 3e-7) * (1 + p % 3)
        out.append(synth.Pair(f"seq{p}", a, b, 4096, 1e-6))
    return out


@pytest.mark.parametrize("chunk", [4096, 512])
def test_pairs_sequence_matches_oracle(chunk):
    seq = _sequence()
    outs = [_outputs(p, chunk) for p in seq]
    trees = ck.compare_pairs_async([p.a for p in seq], [p.b for p in seq], chunk, seq[0].eps,
                                   [o[0] for o in outs], [o[1] for o in outs], [o[2] for o in outs])
    for TA, TB in trees:
        TA.wait(); TB.wait()
    torch.cuda.synchronize()
    tot = 0
    for pair, (TA, TB), (c, i, n) in zip(seq, trees, outs):
        nc, nd = _check_pair(pair, chunk, TA, TB, c, i, n)
        tot += nc
        if pair.name == "seq1":
            assert nc == 0 and nd == 0 and TA.root() == TB.root()
    assert tot > 0


def test_pairs_shared_outputs_hold_the_last_pair():
    """Outputs shared by every pair (the bench's form): the verify stream runs the pairs in
    order, so the buffers end with the last pair's results; every tree is still complete."""
    seq = _sequence()[:5]
    big = max(seq, key=lambda p: sum(t.numel() for t in p.a))
    chunks, idx, counts = _outputs(big, 4096)
    trees = ck.compare_pairs_async([p.a for p in seq], [p.b for p in seq], 4096, 1e-6,
                                   chunks, idx, counts)
    torch.cuda.synchronize()
    _check_pair(seq[-1], 4096, *trees[-1], chunks, idx, counts)
    for pair, (TA, TB) in zip(seq, trees):
        TA.wait(); TB.wait()
        ra = oracle.build_checkpoint([np_of(t) for t in pair.a], 4096, 1e-6, threads=8).root
        assert TA.root() == ra


def test_pairs_equal_single_calls_and_interleave_on_one_stream():
    """c2-shaped pairs (6 particle fields): the sequence call equals one compare_pair_async per
    pair, and alternating both calls on one stream (tile slot 0 shared) keeps every result."""
    seq = [synth.c2_pair(n_particles=(1 << 18) + 11 * p, seed=40 + p, device="cuda")
           for p in range(4)]
    C, eps = seq[0].chunk_bytes, seq[0].eps
    ref = []
    for pair in seq:
        c, i, n = _outputs(pair, C)
        TA, TB = ck.compare_pair_async(pair.a, pair.b, C, eps, c, i, n)
        TA.wait(); TB.wait()
        torch.cuda.synchronize()
        ref.append((np_of(c[:int(n[0])]), np_of(i[:int(n[1])]), TA.root(), TB.root()))
    assert sum(r[0].size for r in ref) > 0
    for rep in range(3):
        outs = [_outputs(p, C) for p in seq]
        trees = ck.compare_pairs_async([p.a for p in seq], [p.b for p in seq], C, eps,
                                       [o[0] for o in outs], [o[1] for o in outs],
                                       [o[2] for o in outs])
        # a single call enqueued right behind the sequence on the same stream
        c1, i1, n1 = _outputs(seq[rep], C)
        SA, SB = ck.compare_pair_async(seq[rep].a, seq[rep].b, C, eps, c1, i1, n1)
        for TA, TB in trees:
            TA.wait(); TB.wait()
        SA.wait(); SB.wait()
        torch.cuda.synchronize()
        for r, (TA, TB), (c, i, n) in zip(ref, trees, outs):
            assert np.array_equal(np_of(c[:int(n[0])]), r[0])
            assert np.array_equal(np_of(i[:int(n[1])]), r[1])
            assert TA.root() == r[2] and TB.root() == r[3]
        r = ref[rep]
        assert np.array_equal(np_of(c1[:int(n1[0])]), r[0]) and np.array_equal(np_of(i1[:int(n1[1])]), r[1])
    _check_pair(seq[0], C, *trees[0], *outs[0])


def test_pairs_f64_and_truncation():
    """f64 pairs (c3-shaped) with a chunk list capacity below the flagged count on one pair:
    that pair returns the listed prefix and the full count, the others are unaffected."""
    seq = [synth.c3_pair(n=(1 << 18) + p, seed=60 + p, device="cuda", n_clusters=8, mean_len=256,
                         n_isolated=200) for p in range(4)]
    C, eps = 4096, seq[0].eps
    outs = [_outputs(p, C) for p in seq]
    cut = (outs[2][0][:3], outs[2][1], outs[2][2])
    outs[2] = cut
    trees = ck.compare_pairs_async([p.a for p in seq], [p.b for p in seq], C, eps,
                                   [o[0] for o in outs], [o[1] for o in outs], [o[2] for o in outs])
    torch.cuda.synchronize()
    for k, (pair, (TA, TB), (c, i, n)) in enumerate(zip(seq, trees, outs)):
        TA.wait(); TB.wait()
        if k != 2:
            _check_pair(pair, C, TA, TB, c, i, n)
            continue
        an, bn = [np_of(t) for t in pair.a], [np_of(t) for t in pair.b]
        A = oracle.build_checkpoint(an, C, eps, threads=8)
        B = oracle.build_checkpoint(bn, C, eps, threads=8)
        rc = oracle.diff_checkpoint(A, B)
        assert rc.size > 3
        nc, nd = n.tolist()
        assert nc == rc.size and np.array_equal(np_of(c), rc[:3])
        ri = oracle.verify_checkpoint(an, bn, C, rc[:3], eps, A)
        assert nd == ri.size and np.array_equal(np_of(i[:nd]), ri)


def test_pairs_argument_errors():
    pair = synth.c1_pair(n=1 << 12, seed=3, device="cuda")
    c, i, n = _outputs(pair, 4096)
    with pytest.raises(ValueError):
        ck.compare_pairs_async([], [], 4096, 1e-5, c, i, n)
    with pytest.raises(ValueError):
        ck.compare_pairs_async([pair.a], [pair.b, pair.b], 4096, 1e-5, c, i, n)
    short = [pair.a[0][:100]]
    with pytest.raises(ValueError):
        ck.compare_pairs_async([pair.a], [short], 4096, 1e-5, c, i, n)
    with pytest.raises(ValueError):
        ck.compare_pairs_async([pair.a, pair.a], [pair.b, pair.b], 4096, 1e-5, [c], i, n)
    with pytest.raises(ck.CkptError):
        ck.compare_pairs_async([pair.a], [pair.b], 24, 1e-5, c, i, n)   # C not a multiple of 16
