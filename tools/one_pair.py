#!/usr/bin/env python
"""A few fused pair compares of the c2 shape (for ncu captures): --identical or the c2 recipe."""
import argparse
import ctypes
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--lib", default="")
ap.add_argument("--identical", action="store_true")
ap.add_argument("--config", default="c2")
ap.add_argument("--reps", type=int, default=4)
args = ap.parse_args()
if args.lib:
    ck._lib = ck._declare(ctypes.CDLL(args.lib))
pair = synth.c2_pair(device="cuda") if args.config == "c2" else synth.c5_pair(device="cuda")
A = pair.a
B = [t.clone() for t in A] if args.identical else pair.b
L = sum(t.numel() * 4 // 4096 for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A), dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(args.reps):
    ck.compare_pair_async(A, B, 4096, 1e-6, chunks, idx, cnt)
torch.cuda.synchronize()
print("counts", cnt.tolist())
