#!/bin/bash
# Time the bench step for each libckpt variant under variants/ (tuning only).
for f in variants/lib_*.so; do
  n=$(basename $f .so)
  CKPT_LIB=$f timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu --no-e2e 2>&1 | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$n', d['value'], r['achieved'], r['frac'], d['clocks']['sm_mhz'])" || echo "$n failed"
done
