#!/usr/bin/env python
"""Per-CTA timeline of the levels kernel (variant 'lvtrace'): phase-1 duration of every group CTA
and the last CTA's phase 2, for the c2 pair path, with and without the verify kernels alongside."""
import ctypes
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

lib = ctypes.CDLL(os.path.join(ROOT, sys.argv[1] if len(sys.argv) > 1 else "variants/lvtrace/libckpt.so"))
ck._lib = ck._declare(lib)
pair = synth.c2_pair(device="cuda")
A, B = pair.a, pair.b
L = sum(t.numel() * 4 // 4096 for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A), dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(3):
    ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
torch.cuda.synchronize()
buf = (ctypes.c_uint64 * (4 * 8192))()
ctypes.memset(buf, 0, ctypes.sizeof(buf))
lib.ckpt_debug_lv(buf)   # clear view
TA, TB = ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
TA.wait(); TB.wait()
torch.cuda.synchronize()
lib.ckpt_debug_lv(buf)
tr = np.frombuffer(buf, dtype=np.uint64).reshape(-1, 4).astype(np.int64)
used = tr[:, 3] == 1
n = int(used.sum())
t0 = tr[used, 0].min()
start = (tr[used, 0] - t0) / 1e3
p1 = (tr[used, 1] - tr[used, 0]) / 1e3
end1 = (tr[used, 1] - t0) / 1e3
last = tr[used, 2]
print(f"{n} CTAs; start p0/p50/p100 {np.percentile(start, [0, 50, 100]).round(1)} us")
print(f"phase1 duration p0/p50/p90/p100 {np.percentile(p1, [0, 50, 90, 100]).round(1)} us; phase-1 ends by {end1.max():.1f} us")
for i in np.nonzero(last > 0)[0]:
    print(f"  last CTA {i}: phase 2 {(last[i] - tr[used][i, 1]) / 1e3:.1f} us, ends at {(last[i] - t0) / 1e3:.1f} us")
