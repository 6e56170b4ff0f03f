#!/bin/bash
# c2 step/leaf A/B across variant libraries AB_LIBS (product included), alternating order, REPS reps.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
libs="product ${AB_LIBS}"
for rep in $(seq 1 ${REPS:-3}); do
  order=$libs; [ $((rep % 2)) = 0 ] && order=$(echo $libs | tr ' ' '\n' | tac | tr '\n' ' ')
  for v in $order; do
    lib=""; [ "$v" != product ] && lib="--lib=variants/$v/libckpt.so"
    printf "%-12s rep %s: " $v $rep
    timeout 600 python tools/step_timeline.py 20 ${AB_ARGS} $lib 2>&1 | grep -v "^library" | head -2 | tr '\n' ' '; echo
  done
done
