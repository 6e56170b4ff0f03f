#!/bin/bash
# A/B of the pipelined pair sequence (bench.py --pipeline on): verify-stream priority x
# programmatic launch of the leaf kernel.  Usage: tools/pipe_ab.sh [config] [reps]
cfg=${1:-c2}; reps=${2:-2}
for r in $(seq $reps); do
  for v in lo hi; do
    for k in 0 1; do
      CKPT_PIPE_VPRIO=$v CKPT_PIPE_K1PDL=$k python bench.py --config $cfg --steps 20 --warmup 5 --no-e2e --no-cpu \
        > gpurun_out/pab_${cfg}_${v}_${k}_$r.json 2>gpurun_out/pab_${cfg}_${v}_${k}_$r.err
      python - "$cfg" "$v" "$k" "$r" <<'PY'
import json, sys
c, v, k, r = sys.argv[1:]
d = json.load(open(f"gpurun_out/pab_{c}_{v}_{k}_{r}.json"))
print(c, "vprio", v, "k1pdl", k, "rep", r, "pipelined ms", d["ms_per_step"], "GB/s", d["value"],
      "| per-call ms", d["per_call"]["ms_per_step"], "| leaf ms", d["roofline"]["avg_launch_ms"],
      "| clocks", d["clocks"]["sm_mhz"], d["clocks"]["reasons"])
PY
    done
  done
done
