#!/usr/bin/env python
"""Per-kernel timeline of bench steps (events around every library launch).

usage: step_timeline.py [N_STEPS] [--unfused] [--c5 | --c3 [--chunk=BYTES]] [--lib=PATH]   (default: the fused pair path bench.py times,
on c2; --c5: the configs[4] per-GPU shard)"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
import synth  # noqa: E402

for a in sys.argv[1:]:
    if a.startswith("--lib="):        # an A/B variant library (tools/variant.py)
        import ctypes
        ck._lib = ck._declare(ctypes.CDLL(a[6:]))
        print("library:", a[6:], flush=True)

CHUNK = 4096
for a in sys.argv[1:]:
    if a.startswith("--chunk="):
        CHUNK = int(a[8:])
if "--c5" in sys.argv:
    pair = synth.c5_pair(device="cuda")
elif "--c3" in sys.argv:                  # configs[2]: 2^29 f64, the chunk size from --chunk=
    pair = synth.c3_pair(device="cuda", chunk_bytes=CHUNK)
else:
    pair = synth.c2_pair(device="cuda")
A, B = pair.a, pair.b
L = sum(-(-t.numel() * t.element_size() // CHUNK) for t in A)
chunks = torch.empty(L, dtype=torch.int64, device="cuda")
idx = torch.empty(sum(t.numel() for t in A) // (8 if "--c5" in sys.argv else 1), dtype=torch.int64,
                  device="cuda")
counts = torch.zeros(2, dtype=torch.int64, device="cuda")


FUSED = "--unfused" not in sys.argv     # the bench path: ckpt_compare_pair_async


def step():
    if FUSED:
        TA, TB = ck.compare_pair_async(A, B, CHUNK, 1e-6, chunks, idx, counts)
    else:
        TA, TB = ck.tree_build_batch([A, B], CHUNK, 1e-6)
        ck.diff_verify_async(TA, TB, A, B, chunks, idx, counts)
    TA.wait()
    TB.wait()
    return TA, TB


for _ in range(5):
    keep = step()
torch.cuda.synchronize()
ck.profile_reset()
ck.profile_enable(True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
args = [a for a in sys.argv[1:] if not a.startswith("--")]
n_steps = int(args[0]) if args else 3
e0.record()
for _ in range(n_steps):
    keep = step()
e1.record()
torch.cuda.synchronize()
ck.profile_enable(False)
print(f"{n_steps} steps: {e0.elapsed_time(e1) / n_steps:.4f} ms/step")
tl = ck.profile_timeline()
for kind in ("leaf", "levels", "diff", "verify"):
    d = [(b - a) * 1e3 for k, a, b in tl if k == kind]
    if d:
        print(f"  {kind:7s} mean {sum(d) / len(d):8.1f} us  min {min(d):8.1f}  max {max(d):8.1f}")
prev_end = 0.0
for k, s0, s1 in sorted(tl, key=lambda r: r[1])[:8]:
    print(f"{k:7s} start {s0 * 1e3:9.1f} us  end {s1 * 1e3:9.1f} us  dur {(s1 - s0) * 1e3:7.1f} us  gap {(s0 - prev_end) * 1e3:7.1f}")
    prev_end = max(prev_end, s1)
