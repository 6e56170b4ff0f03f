#!/bin/bash
# K1 pair kernel at 72 registers (product) vs 80 (pair80), c2 and c5, alternating order.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for rep in 1 2 3 4; do
if [ $((rep % 2)) = 1 ]; then order="product pair80"; else order="pair80 product"; fi
for v in $order; do
  lib=""; [ "$v" != product ] && lib="--lib=variants/$v/libckpt.so"
  for cfg in "" "--c5"; do
    echo "== $v [$cfg] rep $rep"
    timeout 600 python tools/step_timeline.py 20 $cfg $lib 2>&1 | grep -v "^library" | head -2
  done
done
done
