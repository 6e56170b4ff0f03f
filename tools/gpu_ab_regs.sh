#!/bin/bash
# K1 pair kernel at 72 registers (product) vs 80 (variant pair80): c2, c5, c3 at several chunks.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for rep in 1 2 3; do
for v in product pair80; do
  lib=""; [ "$v" != product ] && lib="--lib=variants/$v/libckpt.so"
  for cfg in "" "--c5" "--c3 --chunk=512" "--c3 --chunk=4096" "--c3 --chunk=16384"; do
    echo "== $v [$cfg] rep $rep"
    timeout 600 python tools/step_timeline.py 20 $cfg $lib 2>&1 | grep -v "^library" | head -2
  done
done
done
