#!/usr/bin/env python
"""Pipelined pair sequence (ckpt_compare_pairs_async) on c2: device time of repeated K-pair
calls, then one profiled call's per-kernel timeline (events around every launch).

usage: pipe_timeline.py [K] [REPS]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 8
REPS = int(sys.argv[2]) if len(sys.argv) > 2 else 6
pair = synth.c2_pair(device="cuda")
A, B = pair.a, pair.b
L = sum(-(-t.numel() * t.element_size() // 4096) for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A), dtype=torch.int64, device="cuda")
cnt = torch.zeros((K, 2), dtype=torch.int64, device="cuda")


def seq():
    trees = ck.compare_pairs_async([A] * K, [B] * K, 4096, 1e-6, chunks, idx, [cnt[p] for p in range(K)])
    for TA, TB in trees:
        TA.wait()
        TB.wait()
    return trees


keep = seq()
torch.cuda.synchronize()
for r in range(REPS):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    keep = seq()
    e1.record()
    torch.cuda.synchronize()
    print(f"rep {r}: {e0.elapsed_time(e1) / K:.4f} ms per pair", flush=True)
ck.profile_reset()
ck.profile_enable(True)
keep = seq()
torch.cuda.synchronize()
ck.profile_enable(False)
for name, t0, t1 in sorted(ck.profile_timeline(), key=lambda x: x[1]):
    print(f"{name:8s} {t0:9.3f} {t1:9.3f} {t1 - t0:8.3f}")
print("counts", cnt[0].tolist(), bool((cnt == cnt[0]).all()))
