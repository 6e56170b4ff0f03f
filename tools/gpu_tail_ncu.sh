#!/bin/bash
# ncu --set full of the post-K1 kernels of one c2 bench-shaped pair compare (levels, verify
# mark/scan/emit).  Output: gpurun_out/t/.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
O=gpurun_out/t; mkdir -p $O
timeout 900 ncu --set full --import-source on --clock-control none -k "regex:levels|verify" -s 8 -c 4 -o $O/tail_full python tools/one_pair.py --reps 4 > $O/tail_full.log 2>&1; echo "tail rc=$?"
