#!/bin/bash
# A/B of step timelines (c2 and c5) across variant libraries: AB_LIBS="name1 name2" (product first).
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
for rep in 1 2; do
for v in product ${AB_LIBS}; do
  lib=""; [ "$v" != product ] && lib="--lib=variants/$v/libckpt.so"
  for cfg in ${AB_CFGS:-c2 c5}; do
    flag=""; [ "$cfg" = c5 ] && flag="--c5"
    echo "== $v $cfg rep $rep"
    timeout 600 python tools/step_timeline.py 20 $flag $lib 2>&1 | grep -v "^library" | head -6
  done
done
done
if [ -n "$NCU_C5" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"leaf|levels|verify|compact|gather" -c 16 --csv \
  --log-file gpurun_out/c5_launches.csv python bench.py --config c5 --steps 2 --warmup 1 --no-e2e --no-cpu \
  > gpurun_out/c5_ncu_bench.log 2>&1; echo "ncu_rc=$?"
python tools/launches_md.py gpurun_out/c5_launches.csv | head -30
fi
