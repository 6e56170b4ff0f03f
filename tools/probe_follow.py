#!/usr/bin/env python
"""Co-residency probe (variant 'probe', tools/variant.py): a 1-warp kernel launched with
programmatic dependent launch right after the fused pair leaf kernel records when its CTAs
start, relative to the leaf kernel's first and last CTA activity (globaltimer, ns)."""
import ctypes
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

path = sys.argv[1] if len(sys.argv) > 1 else "variants/probe/libckpt.so"
L = ctypes.CDLL(path)
ck._lib = ck._declare(L)
L.ckpt_dbg.argtypes = [ctypes.POINTER(ctypes.c_ulonglong), ctypes.c_int]
FTRACE = "--ftrace" in sys.argv      # variant 'ftrace' (tools/ftrace_variant.sh)
pair = synth.c5_pair(device="cuda") if "--c5" in sys.argv else synth.c2_pair(device="cuda")
A, B = pair.a, pair.b
n_ch = sum(t.numel() * 4 // 4096 for t in A)
chunks = torch.empty(n_ch, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A) // 8, dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(3):
    ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
torch.cuda.synchronize()
for rep in range(3):
    L.ckpt_dbg(None, 1)
    ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
    torch.cuda.synchronize()
    h = (ctypes.c_ulonglong * 16)()
    L.ckpt_dbg(h, 0)
    if FTRACE:
        k0, f0, k1, f1 = h[0], h[1], h[2], h[3]
        nw = 148 * 4
        print(f"rep {rep}: K1 {(k1 - k0) / 1e3:8.1f} us; follower start {(f0 - k0) / 1e3:+7.1f}, last warp done "
              f"{(f1 - k0) / 1e3:+8.1f} us; per warp: wait {h[4] / nw / 1e3:7.1f} us, levels {h[5] / nw / 1e3:7.1f} us "
              f"({h[7]} groups, {h[5] / max(h[7], 1) / 1e3:.1f} us each), mark {h[6] / nw / 1e3:7.1f} us "
              f"({h[8]} chunks, {h[6] / max(h[8], 1) / 1e3:.2f} us each)")
        continue
    k0, f0, k1, f1 = h[0], h[1], h[2], h[3]
    print(f"rep {rep}: leaf {(k1 - k0) / 1e3:8.1f} us; follower CTAs start {(f0 - k0) / 1e3:+8.1f} .. "
          f"{(f1 - k0) / 1e3:+8.1f} us after the leaf kernel's start; CTAs per smid&3 {list(h[4:8])}")
