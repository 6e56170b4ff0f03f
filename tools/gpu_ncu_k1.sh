#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
for v in ${NCU_VARIANTS:-product base}; do
  if [ "$v" = product ]; then lib=""; else lib="--lib variants/$v/libckpt.so"; fi
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:${NCU_K:-leaf_} -s ${NCU_SKIP:-2} -c 1 \
     -o gpurun_out/k1_$v python tools/one_pair.py $lib ${ONE_ARGS} > gpurun_out/ncu_$v.log 2>&1
  echo "$v rc=$?"; tail -1 gpurun_out/ncu_$v.log
done
