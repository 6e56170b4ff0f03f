#!/usr/bin/env python
"""Per-pair period of the pipelined pair sequence vs one call per pair (c2 or c5): device time
of K pairs for several K; the slope of a least-squares line is the steady-state period.

usage: pipe_slope.py [c2|c5]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
pair = synth.c5_pair(device="cuda") if cfg == "c5" else synth.c2_pair(device="cuda")
A, B = pair.a, pair.b
L = sum(-(-t.numel() * t.element_size() // 4096) for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A) // (4 if cfg == "c5" else 1), dtype=torch.int64, device="cuda")
KS = [2, 4, 8, 16, 32] if cfg == "c2" else [1, 2, 4, 8]
cnt = torch.zeros((max(KS), 2), dtype=torch.int64, device="cuda")


def seq(K):
    trees = ck.compare_pairs_async([A] * K, [B] * K, 4096, 1e-6, chunks, idx, [cnt[p] for p in range(K)])
    for TA, TB in trees:
        TA.wait(); TB.wait()


def calls(K):
    for _ in range(K):
        TA, TB = ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt[0])
        TA.wait(); TB.wait()


def timed(fn, K, reps=3):
    fn(K)
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn(K)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


for name, fn in (("pipelined", seq), ("per-call", calls), ("pipelined", seq), ("per-call", calls)):
    t = [timed(fn, K) for K in KS]
    b, a = np.polyfit(KS, t, 1)
    print(f"{cfg} {name:9s} " + " ".join(f"K={K}:{x / K:.4f}" for K, x in zip(KS, t))
          + f"  | period {b:.4f} ms + {a:.4f} ms per call", flush=True)
