#!/usr/bin/env python
"""Ticket timeline of the finish kernel (variant 'fintrace', tools/variant.py): for one fused
compare of the c2 shape, when each ticket was drawn and by which CTA; item duration = the same
CTA's next draw."""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

lib = ctypes.CDLL(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "variants/fintrace/libckpt.so"))
ck._lib = ck._declare(lib)
ident = "--identical" in sys.argv
pair = synth.c2_pair(device="cuda")
A = pair.a
B = [t.clone() for t in A] if ident else pair.b
L = sum(t.numel() * 4 // 4096 for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A), dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
for sep in (False, True):
    for _ in range(3):
        ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
    torch.cuda.synchronize()
    ck.profile_enable(["leaf"] if sep else False)
    ck.profile_reset()
    ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
    torch.cuda.synchronize()
    buf = (ctypes.c_uint64 * (2 * 16384))()
    lib.ckpt_debug_fin_trace(buf)
    tr = np.frombuffer(buf, dtype=np.uint64).reshape(-1, 2)
    n_tiles = (L // 32 + 127) // 128
    n_level = 2 * sum(-(-(t.numel() * 4 // 4096) // 512) for t in A)
    used = tr[:, 0] > 0
    t0 = tr[used, 0].min()
    tt = (tr[:, 0].astype(np.int64) - int(t0)) / 1e3
    n = int(used.sum())
    print(f"== {'events after K1 (no overlap)' if sep else 'overlapped'}: {n} tickets drawn, span {tt[used].max():.1f} us, counts {cnt.tolist()}")
    # per CTA: consecutive draws
    cta = tr[:, 1].astype(np.int64)
    order = np.argsort(tt)
    ends = {}
    durs = []
    last = {}
    for i in order:
        if not used[i]:
            continue
        c = cta[i]
        if c in last:
            durs.append((last[c][0], tt[i] - last[c][1]))
        last[c] = (i, tt[i])
    d = np.array(durs)
    lev = d[d[:, 0] < n_level]
    ver = d[d[:, 0] >= n_level]
    for name, x in (("verify", ver), ("level", lev)):
        if len(x):
            print(f"  {name:6s} items {len(x):4d}: duration us mean {x[:, 1].mean():6.1f} p50 {np.median(x[:, 1]):6.1f} max {x[:, 1].max():6.1f}")
    b2 = (ctypes.c_uint64 * (4 * 4096))()
    if hasattr(lib, "ckpt_debug_fin_t2"):
        lib.ckpt_debug_fin_t2(b2)
        t2 = np.frombuffer(b2, dtype=np.uint64).reshape(-1, 4)[:n_tiles].astype(np.int64)
        ok = t2[:, 0] > 0
        if ok.any():
            mark = (t2[ok, 1] - t2[ok, 0]) / 1e3
            lb = (t2[ok, 2] - t2[ok, 1]) / 1e3
            st = (t2[ok, 0] - int(t0)) / 1e3
            print(f"  verify: start p50 {np.median(st):.1f}, mark p50 {np.median(mark):.1f} max {mark.max():.1f}, "
                  f"prefix+lookback p50 {np.median(lb):.1f} max {lb.max():.1f} us")
    qs = np.percentile(tt[used], [0, 10, 50, 90, 100])
    print("  draw times (us) p0/p10/p50/p90/p100:", np.round(qs, 1))
    ck.profile_enable(False)
