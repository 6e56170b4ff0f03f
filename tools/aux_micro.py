#!/usr/bin/env python
"""Time K3 (diff) and K4 (verify) alone, device counts, no host sync in the loop."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402


def timed(fn, kind, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ck.profile_reset()
    ck.profile_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    ck.profile_enable(False)
    ms, n = ck.profile_read(kind)
    return ms / n * 1e3, e0.elapsed_time(e1) / reps * 1e3


for n_part in (1 << 16, 1 << 20, 1 << 24, 1 << 26):
    pair = synth.c2_pair(n_particles=n_part, seed=5, device="cuda")
    TA, TB = ck.tree_build_batch([pair.a, pair.b], 4096, 1e-6)
    L = TA.n_leaves
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
    idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
    k_us, w_us = timed(lambda: ck.tree_diff_async(TA, TB, chunks, cnt[0:1]), "diff")
    nflag = int(cnt[0].item())
    v_us, vw_us = timed(lambda: ck.verify_async(pair.a, pair.b, chunks, cnt[0:1], 4096, 1e-6, idx,
                                                cnt[1:2]), "verify")
    print(f"L={L:8d} flagged={nflag:6d} diff kernel {k_us:7.1f} us (call {w_us:7.1f})  "
          f"verify kernel {v_us:7.1f} us (call {vw_us:7.1f}) n_diff={int(cnt[1].item())}", flush=True)
