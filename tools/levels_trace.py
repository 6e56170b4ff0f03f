#!/usr/bin/env python
"""K2 timeline inside one bench step (debug build -DCKPT_LEVELS_TRACE):
per CTA entry / after griddepcontrol.wait / phase-1 end / ticket, and the last CTA's
phase-2 end and top-tree end.  usage: CKPT_LIB=variants/lib_lvtr.so python tools/levels_trace.py"""
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
K = 4096
buf = (ctypes.c_uint64 * (K * 4 + 16))()
assert ck.lib().ckpt_debug_levels_trace(buf) == 0
a = np.frombuffer(buf, dtype=np.uint64).astype(np.int64)
cta = a[:K * 4].reshape(K, 4)
n = int(np.sum(cta[:, 0] > 0))
cta = cta[:n]
t0 = cta[:, 0].min()
rel = (cta - t0) / 1e3
print(f"{n} CTAs; entry spread {rel[:, 0].max():.1f} us")
for j, name in enumerate(["entry", "after wait", "phase-1 end", "ticket"]):
    print(f"  {name:12s} min {rel[:, j].min():7.1f}  p50 {np.median(rel[:, j]):7.1f}  max {rel[:, j].max():7.1f} us")
print(f"  phase-1 duration per CTA: p50 {np.median(rel[:, 2] - rel[:, 1]):.1f} max {(rel[:, 2] - rel[:, 1]).max():.1f} us")
last = (a[K * 4:K * 4 + 8].reshape(4, 2) - t0) / 1e3
for k in range(2):
    print(f"  tree {k}: phase-2 levels end {last[k, 0]:7.1f} us, top end {last[k, 1]:7.1f} us")
