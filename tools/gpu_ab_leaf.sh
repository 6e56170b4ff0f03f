#!/bin/bash
# Leaf-time A/B (fused pair path, follower off): product vs variant libraries AB_LIBS, c2 and c5.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for rep in 1 2 3; do
for v in product ${AB_LIBS}; do
  lib=""; [ "$v" != product ] && lib="--lib=variants/$v/libckpt.so"
  for cfg in ${AB_CFGS:-c2 c5}; do
    flag=""; [ "$cfg" = c5 ] && flag="--c5"
    echo "== $v $cfg rep $rep"
    CKPT_FOLLOW=${FOLLOW:-0} timeout 600 python tools/step_timeline.py 20 $flag $lib 2>&1 | grep -v "^library" | head -3
  done
done
done
