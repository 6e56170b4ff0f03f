#!/bin/bash
# usage: tools/variant_paths.sh CONFIG STEPS PATH  -- every variants/lib_*.so on one bench line each
cfg=${1:-c2}; steps=${2:-50}; pth=${3:-fused}
for f in variants/lib_*.so; do
  n=$(basename $f .so)
  CKPT_LIB=$f timeout 300 python bench.py --config $cfg --path $pth --steps $steps --warmup 5 --no-cpu --no-e2e 2>&1 | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); ph={k: v['ms_per_step'] for k, v in d['phases_profiled_pass'].items() if isinstance(v, dict)}; print('$n $cfg $pth', d['value'], d['ms_per_step'], ph)" || echo "$n failed"
done
