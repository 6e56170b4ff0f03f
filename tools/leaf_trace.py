#!/usr/bin/env python
"""K1 tail analysis: per-warp start/end times and task counts of one fused c2 pair launch.

usage: CKPT_LIB=variants/lib_trace.so python tools/leaf_trace.py   (lib built with -DCKPT_LEAF_TRACE)
Prints when warps finish relative to the launch, i.e. how much of the launch runs with fewer
than all warps busy (the dynamic-ticket tail)."""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

pair = synth.c2_pair(device="cuda")
L = sum(t.numel() * 4 // 4096 for t in pair.a)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in pair.a), dtype=torch.int64, device="cuda")
counts = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(4):
    TA, TB = ck.compare_pair_async(pair.a, pair.b, 4096, 1e-6, chunks, idx, counts)
    TA.wait(); TB.wait()
torch.cuda.synchronize()
lib = ck.lib()
f = lib.ckpt_debug_leaf_trace
f.restype = ctypes.c_int
n = 148 * 24
buf = (ctypes.c_uint64 * (3 * n))()
assert f(buf, n) == n
a = np.frombuffer(buf, dtype=np.uint64).reshape(n, 3).astype(np.int64)
t0 = a[:, 0].min()
start = (a[:, 0] - t0) / 1e3
end = (a[:, 1] - t0) / 1e3
tasks = a[:, 2] & 0xffffffff
sm = a[:, 2] >> 32
T = end.max()
print(f"launch span {T:.1f} us; warp start spread {start.max() - start.min():.1f} us")
print(f"tasks per warp: min {tasks.min()} max {tasks.max()} mean {tasks.mean():.2f}")
for q in (0, 1, 5, 10, 25, 50, 75, 90, 99, 100):
    print(f"  warp end p{q:3d}: {np.percentile(end, q):8.1f} us")
# busy-warp profile over time
grid = np.linspace(0, T, 41)
busy = [(np.sum((start <= t) & (end > t))) / n for t in grid]
print("fraction of warps busy: " + " ".join(f"{b:.2f}" for b in busy[-12:]) + "  (last 12 of 40 slices)")
lost = np.sum((T - end)) / n
print(f"mean idle time per warp before the launch ends: {lost:.1f} us ({100 * lost / T:.1f}% of warp-time)")
