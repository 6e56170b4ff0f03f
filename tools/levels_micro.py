#!/usr/bin/env python
"""Time K2 (levels kernel) alone via ckpt_tree_from_digests over N random digests."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402

for n in (1, 2, 64, 512, 4096, 65536, 393216, 1 << 22):
    d = torch.randint(0, 256, (n, 16), dtype=torch.uint8, device="cuda")
    for _ in range(3):
        ck.tree_from_digests(d)
    torch.cuda.synchronize()
    ck.profile_reset()
    ck.profile_enable(True)
    for _ in range(20):
        ck.tree_from_digests(d)
    torch.cuda.synchronize()
    ck.profile_enable(False)
    ms, k = ck.profile_read("levels")
    print(f"n={n:8d}  levels kernel {ms / k * 1e3:8.1f} us")
