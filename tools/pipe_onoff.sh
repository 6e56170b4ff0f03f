#!/bin/bash
# Interleaved A/B of bench.py --pipeline on/off (fresh process per run).
# Usage: tools/pipe_onoff.sh [config] [reps] [steps]
cfg=${1:-c2}; reps=${2:-3}; steps=${3:-20}
for r in $(seq $reps); do
  for m in on off; do
    python bench.py --config $cfg --steps $steps --warmup 5 --no-e2e --no-cpu --pipeline $m \
      > gpurun_out/onoff_${cfg}_${m}_$r.json 2>/dev/null
    python -c "import json,sys;d=json.load(open(sys.argv[1]));print(sys.argv[2],sys.argv[3],'ms',d['ms_per_step'],'GB/s',d['value'],'leaf',d['roofline']['avg_launch_ms'],'clk',d['clocks']['sm_mhz'],d['clocks']['reasons'])" gpurun_out/onoff_${cfg}_${m}_$r.json $cfg $m
  done
done
