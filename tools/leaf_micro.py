#!/usr/bin/env python
"""Leaf-kernel throughput by mode (raw hash / f32 rounding / f64 rounding) and chunk size.

usage: python tools/leaf_micro.py [--gb 1.6] [--chunks 4096,...]
Times only the leaf kernel (ckpt_profile events), 6 arrays per checkpoint."""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--gb", type=float, default=1.6)
ap.add_argument("--chunks", default="4096")
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--modes", default="f32,raw32,f64,raw64")
ap.add_argument("--arrays", type=int, default=6)
args = ap.parse_args()
peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    "MEASURED_PEAKS.json") else 6437.9
res = {}
for mode in args.modes.split(","):
    f64 = mode.endswith("64")
    dt = torch.float64 if f64 else torch.float32
    n_total = int(args.gb * 1e9 / (8 if f64 else 4))
    per = (n_total // args.arrays) // 1024 * 1024
    arrs = [synth.uniform(10 + i, per, "cuda", dtype=dt) * 256.0 for i in range(args.arrays)]
    eps = 0.0 if mode.startswith("raw") else 1e-6
    for C in [int(c) for c in args.chunks.split(",")]:
        for _ in range(3):
            ck.tree_build(arrs, C, eps)
        torch.cuda.synchronize()
        ck.profile_reset()
        ck.profile_enable(True)
        for _ in range(args.reps):
            ck.tree_build(arrs, C, eps)
        torch.cuda.synchronize()
        ck.profile_enable(False)
        ms, n = ck.profile_read("leaf")
        nbytes = sum(t.numel() * t.element_size() for t in arrs)
        gbs = nbytes / (ms / n / 1e3) / 1e9
        res[f"{mode}/C{C}"] = round(gbs, 1)
        print(f"{mode:6s} C={C:6d}  {ms / n * 1e3:8.1f} us  {gbs:8.1f} GB/s  {gbs / peak:.3f} of HBM",
              flush=True)
    del arrs
print(json.dumps(res))
