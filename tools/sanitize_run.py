#!/usr/bin/env python
"""Small workloads through every libckpt entry point, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck).  Checks results against the oracle too."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

torch.cuda.set_device(0)
pair = synth.c1_pair(n=(1 << 16) + 77, seed=5, device="cuda")          # ragged tail
a, b = pair.a[0], pair.b[0]
C, eps = 4096, pair.eps
an, bn = a.cpu().numpy(), b.cpu().numpy()
ref_c = oracle.diff(oracle.levels(oracle.leaves(an, C, eps)), oracle.levels(oracle.leaves(bn, C, eps)),
                    oracle.n_chunks(an.size, 0, C))
ref_i = oracle.verify(an, bn, C, ref_c, eps)
L = oracle.n_chunks(an.size, 0, C)
# unfused: build, BFS diff from the leaves and from a mid level, verify
ta, tb = ck.tree_build(a, C, eps), ck.tree_build(b, C, eps)
assert np.array_equal(ck.tree_diff(ta, tb).cpu().numpy(), ref_c)
for T in (1, 7):
    ch = torch.empty(L, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    ck.tree_diff_async(ta, tb, ch, cnt, T=T)
    assert np.array_equal(ch[: int(cnt.item())].cpu().numpy(), ref_c)
idx, n = ck.verify(a, b, torch.as_tensor(ref_c, device="cuda"), C, eps)
assert np.array_equal(idx.cpu().numpy(), ref_i)
# fused pair path, 16-byte and whole-chunk hash blocks
for hb in (16, 0):
    ch = torch.empty(L, dtype=torch.int64, device="cuda")
    ix = torch.empty(a.numel(), dtype=torch.int64, device="cuda")
    cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async([a], [b], C, eps, ch, ix, cnt, hash_block=hb)
    TA.wait(); TB.wait()
    nc, nd = cnt.tolist()
    assert np.array_equal(ch[:nc].cpu().numpy(), ref_c) and np.array_equal(ix[:nd].cpu().numpy(), ref_i)
# host paths, persistence, streaming
out = ck.compare_host([a.cpu()], [b.cpu()], C, eps)
assert np.array_equal(out[0].numpy(), ref_i)
out = ck.compare_stream([a.cpu().pin_memory()], [b.cpu().pin_memory()], C, eps, segment_bytes=3 * C)
assert np.array_equal(out[1].numpy(), ref_i)
blob = ta.serialize()
t2 = ck.tree_deserialize(blob)
assert t2.root() == ta.root()
ch = torch.empty(L, dtype=torch.int64, device="cuda")
ix = torch.empty(a.numel(), dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
ck.compare_saved(blob, [a.cpu().pin_memory()], [b], ch, ix, cnt)
torch.cuda.synchronize()
nc, nd = cnt.tolist()
assert np.array_equal(ix[:nd].cpu().numpy(), ref_i)
# multi-array checkpoint (c5 shape, small) through the fused path
p5 = synth.c5_pair(n_ranks=1, n_particles=1 << 13, seed=3, device="cuda")
L5 = sum(-(-t.numel() * 4 // C) for t in p5.a)
ch = torch.empty(L5, dtype=torch.int64, device="cuda")
ix = torch.empty(sum(t.numel() for t in p5.a), dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
TA, TB = ck.compare_pair_async(p5.a, p5.b, C, p5.eps, ch, ix, cnt)
TA.wait(); TB.wait()
torch.cuda.synchronize()
# a flagged short last chunk of 64 KiB chunks after a fully differing compare on the same stream
# (the verify work buffer holds all-ones masks; emit must read only the groups the chunk has)
n7 = 70_001
a7 = synth.uniform(17, n7, "cuda") * 2.0 - 1.0
L7 = -(-n7 * 4 // 65536)
ch = torch.empty(L7, dtype=torch.int64, device="cuda")
ix = torch.empty(n7, dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
TA, TB = ck.compare_pair_async([a7], [a7 + 1.0], 65536, 1e-6, ch, ix, cnt)
TA.wait(); TB.wait()
b7 = a7.clone()
b7[-1] += 1.0
TA, TB = ck.compare_pair_async([a7], [b7], 65536, 1e-6, ch, ix, cnt)
TA.wait(); TB.wait()
torch.cuda.synchronize()
assert cnt.tolist() == [1, 1] and ix[0].item() == n7 - 1
# the fused pair kernels specialised per chunk size (f64, 1 KiB and 16 KiB, ragged arrays)
for C8 in (1024, 16384):
    a8 = [synth.normal(30 + k, n, "cuda", dtype=torch.float64) for k, n in enumerate((3 * C8 // 8 + 3, 777))]
    b8 = [t.clone() for t in a8]
    b8[0][::97] += 1e-3
    b8[1][-1] += 1.0
    L8 = sum(-(-t.numel() * 8 // C8) for t in a8)
    ch = torch.empty(L8, dtype=torch.int64, device="cuda")
    ix = torch.empty(sum(t.numel() for t in a8), dtype=torch.int64, device="cuda")
    cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
    TA, TB = ck.compare_pair_async(a8, b8, C8, 1e-6, ch, ix, cnt)
    TA.wait(); TB.wait()
    torch.cuda.synchronize()
    an8 = [t.cpu().numpy() for t in a8]
    bn8 = [t.cpu().numpy() for t in b8]
    A8 = oracle.build_checkpoint(an8, C8, 1e-6)
    B8 = oracle.build_checkpoint(bn8, C8, 1e-6)
    rc8 = oracle.diff_checkpoint(A8, B8)
    ri8 = oracle.verify_checkpoint(an8, bn8, C8, rc8, 1e-6, A8)
    nc, nd = cnt.tolist()
    assert np.array_equal(ch[:nc].cpu().numpy(), rc8) and np.array_equal(ix[:nd].cpu().numpy(), ri8)
print("sanitize workload ok", ck.launch_count(), "launches")
