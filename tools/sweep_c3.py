#!/usr/bin/env python
"""BASELINE configs[2]: chunk-size x error-bound sweep on a 4 GiB float64 checkpoint pair with
clustered divergence (synth.c3_pair: N(0,1), 1024 geometric clusters of mean 4096 elements,
|d| = 10^U(-9,-2)).  The synthetic analogue of the paper's Fig. 5 / Fig. 7.

Per point (C in 512 B..64 KB, eps in 1e-3..1e-8): the fused pair compare (ckpt_compare_pair_ex:
build A + build B + diff + verify) timed with CUDA events over `--steps` steps after 3 warm-ups,
reported as pair GB/s, % of the measured HBM copy peak, % of chunks flagged, and the false-positive
rate (flagged chunks without a verified difference / flagged).  Each point also checks, at full
size, that every chunk holding a verified difference is in the flagged list.  Bit-exact parity
with the oracle lives in tests/test_gpu_parity.py (c3_small cases).

    python tools/sweep_c3.py [--n 536870912] [--steps 10] [--hash-block 16] > out.jsonl
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CHUNKS = [512, 1024, 2048, 4096, 8192, 16384, 32768, 65536]
EPSS = [1e-3, 1e-4, 1e-5, 1e-6, 1e-7, 1e-8]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 29)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--hash-block", type=int, default=16)
    ap.add_argument("--chunks", default="", help="comma-separated subset of the chunk sizes")
    ap.add_argument("--eps", default="", help="comma-separated subset of the bounds")
    ap.add_argument("--lib", default="", help="an A/B variant libckpt.so (tools/variant.py)")
    args = ap.parse_args()
    import torch
    import paper_conf_middleware_tanaabcrtn24_b200 as ck
    import synth
    global CHUNKS, EPSS
    if args.chunks:
        CHUNKS = [int(x) for x in args.chunks.split(",")]
    if args.eps:
        EPSS = [float(x) for x in args.eps.split(",")]
    if args.lib:
        import ctypes
        ck._lib = ck._declare(ctypes.CDLL(args.lib))

    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    torch.cuda.set_device(0)
    pair = synth.c3_pair(n=args.n, seed=3, device="cuda")
    A, B = pair.a, pair.b
    nbytes = 2 * A[0].numel() * 8
    idx = torch.empty(A[0].numel(), dtype=torch.int64, device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    rows = []
    for C in CHUNKS:
        L = -(-A[0].numel() * 8 // C)
        chunks = torch.empty(L, dtype=torch.int64, device="cuda")
        for eps in EPSS:
            def step():
                TA, TB = ck.compare_pair_async(A, B, C, eps, chunks, idx, counts,
                                               hash_block=args.hash_block)
                TA.wait()
                TB.wait()
                return TA, TB
            for _ in range(3):
                keep = step()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(args.steps):
                keep = step()
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / args.steps
            nc, nd = counts.tolist()
            per = C // 8
            with_diff = int(torch.unique(idx[:nd] // per).numel()) if nd else 0
            # invariant: every chunk holding a verified difference is in the flagged list
            flagged = chunks[:nc]
            assert with_diff <= nc
            if nd:
                assert bool(torch.isin(torch.unique(idx[:nd] // per), flagged).all())
            row = {"chunk_bytes": C, "eps": eps, "ms": round(ms, 4),
                   "GBps": round(nbytes / ms / 1e6, 1), "pct_hbm": round(nbytes / ms / 1e6 / peak, 4),
                   "flagged": nc, "pct_flagged": round(100.0 * nc / L, 3), "diff_elems": nd,
                   "fp_rate": round((nc - with_diff) / nc, 4) if nc else 0.0}
            rows.append(row)
            print(json.dumps(row), flush=True)
            del keep
    print("| C \\ eps | " + " | ".join(f"{e:g}" for e in EPSS) + " |", file=sys.stderr)
    for C in CHUNKS:
        cells = [r for r in rows if r["chunk_bytes"] == C]
        print(f"| {C} | " + " | ".join(f"{r['GBps']:.0f} GB/s, {r['pct_flagged']:.2f}% fl, "
                                       f"FP {r['fp_rate']:.2f}" for r in cells) + " |",
              file=sys.stderr)


if __name__ == "__main__":
    main()
