#!/usr/bin/env python
"""Fused diff+verify vs separate diff / verify kernels, standalone (trees prebuilt)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402


def timed(fn, kinds, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ck.profile_reset()
    ck.profile_enable(True)
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    ck.profile_enable(False)
    out = []
    for k in kinds:
        ms, n = ck.profile_read(k)
        out.append(ms / max(n, 1) * 1e3)
    return out


for n_part in (1 << 20, 1 << 24, 1 << 26):
    pair = synth.c2_pair(n_particles=n_part, seed=5, device="cuda")
    TA, TB = ck.tree_build_batch([pair.a, pair.b], 4096, 1e-6)
    TA.wait()
    TB.wait()
    L = TA.n_leaves
    n = sum(t.numel() for t in pair.a)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    idx = torch.empty(n, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
    f = timed(lambda: ck.diff_verify_async(TA, TB, pair.a, pair.b, chunks, idx, cnt), ["verify"])
    s = timed(lambda: (ck.tree_diff_async(TA, TB, chunks, cnt[0:1]),
                       ck.verify_async(pair.a, pair.b, chunks, cnt[0:1], 4096, 1e-6, idx, cnt[1:2])),
              ["diff", "verify"])
    print(f"L={L:8d} flagged={int(cnt[0].item()):6d}  fused {f[0]:7.1f} us   separate diff {s[0]:6.1f} + verify {s[1]:6.1f} us",
          flush=True)
