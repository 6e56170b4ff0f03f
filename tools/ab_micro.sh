#!/bin/bash
# A/B: fused_micro (leaf time of the fused pair call) for the product library and each variant.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
for rep in 1 2; do
for v in product ${VARIANTS}; do
  if [ "$v" = product ]; then lib=""; else lib="--lib variants/$v/libckpt.so"; fi
  echo "== $v (rep $rep)"
  timeout 300 python tools/fused_micro.py --quick $lib ${MICRO_ARGS} 2>&1 | grep -v "^library"
done
done
