#!/usr/bin/env python
"""Leaf-kernel time of the fused pair call (ckpt_compare_pair_async) vs the number of flagged
chunks: identical runs, the c2 recipe, and k uniformly spread flagged chunks (one element
changed by 1.0 in each), on the c2 shape (2^26 x 6 f32, 4 KiB chunks)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

import argparse  # noqa: E402
import ctypes  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=1 << 26)
ap.add_argument("--lib", default="", help="an A/B variant library (tools/variant.py)")
ap.add_argument("--quick", action="store_true", help="identical + c2 recipe only")
args = ap.parse_args()
if args.lib:
    ck._lib = ck._declare(ctypes.CDLL(args.lib))
    print("library:", args.lib, flush=True)
n_part = args.n
pair = synth.c2_pair(n_particles=n_part, seed=5, device="cuda")
A = pair.a
L = sum(t.numel() * 4 // 4096 for t in A)
n = sum(t.numel() for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(n, dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")


def run(B, label, reps=10):
    for _ in range(3):
        ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
    torch.cuda.synchronize()
    ck.profile_reset()
    ck.profile_enable(True)
    for _ in range(reps):
        ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
    torch.cuda.synchronize()
    ck.profile_enable(False)
    lm, ln = ck.profile_read("leaf")
    vm, vn = ck.profile_read("verify")
    print(f"{label:>28s}: flagged {int(cnt[0].item()):7d} diffs {int(cnt[1].item()):8d}  "
          f"leaf {lm / max(ln, 1) * 1e3:8.1f} us  emit {vm / max(vn, 1) * 1e3:6.1f} us", flush=True)


run([t.clone() for t in A], "identical")
run(pair.b, "c2 recipe")
if args.quick:
    sys.exit(0)
per = 1024
for k in (64, 1024, 16384):
    B = [t.clone() for t in A]
    Lk = A[0].numel() // per
    for f, t in enumerate(B):
        ch = torch.arange(f, Lk, max(1, Lk * 6 // k), device="cuda")[: k // 6 + 1]
        t[ch * per + 7] += 1.0
    run(B, f"{k} spread chunks")
