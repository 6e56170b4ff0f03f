#!/usr/bin/env python
"""Device time per fused pair compare (ckpt_compare_pair_async + both trees complete, the bench
step without collectives) for one library: CUDA events around K back-to-back steps, best of R.

usage: ab_step.py [--lib PATH] [--config c2|c5|c3] [--steps K] [--reps R]"""
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
ap.add_argument("--config", default="c2")
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--join", default="step", choices=["step", "end"],
                help="step: every step waits for both trees' levels (bench.py); end: only the last")
args = ap.parse_args()
if args.lib:
    ck._lib = ck._declare(ctypes.CDLL(args.lib))
pair = {"c2": lambda: synth.c2_pair(device="cuda"), "c5": lambda: synth.c5_pair(device="cuda"),
        "c3": lambda: synth.c3_pair(device="cuda")}[args.config]()
A, B = pair.a, pair.b
C, eps = pair.chunk_bytes, pair.eps
L = sum(-(-t.numel() * t.element_size() // C) for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A), dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")


def step(last=True):
    TA, TB = ck.compare_pair_async(A, B, C, eps, chunks, idx, cnt)
    if last or args.join == "step":
        TA.wait()
        TB.wait()
    return TA, TB


for _ in range(5):
    keep = step()
torch.cuda.synchronize()
best = 1e9
for _ in range(args.reps):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    kept = []
    for k in range(args.steps):
        kept.append(step(k == args.steps - 1))
    for TA, TB in kept:
        TA.wait()
        TB.wait()
    e1.record()
    torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1) / args.steps)
print(f"{args.config} {os.path.basename(os.path.dirname(args.lib)) if args.lib else 'product'}: "
      f"join={args.join} {best:.4f} ms/step, counts {cnt.tolist()}", flush=True)
