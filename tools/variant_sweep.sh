#!/bin/bash
# Time the bench step for each libckpt variant under variants/ (tuning only).
# usage: tools/variant_sweep.sh [config] [steps]     (env vars pass through, e.g. CKPT_PDL=0)
cfg=${1:-c2}; steps=${2:-100}
for f in variants/lib_*.so; do
  n=$(basename $f .so)
  CKPT_LIB=$f timeout 300 python bench.py --config $cfg --steps $steps --warmup 5 --no-cpu --no-e2e 2>&1 | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; ph={k: v['ms_per_step'] for k, v in d['phases_profiled_pass'].items() if isinstance(v, dict)}; print('$n $cfg', d['value'], d['ms_per_step'], r['achieved'], r['frac'], d['clocks']['sm_mhz'], ph)" || echo "$n failed"
done
