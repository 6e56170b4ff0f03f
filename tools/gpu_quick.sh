#!/bin/bash
# Quick GPU pass: selected tests (PYTEST_K), smoke, one bench line.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout ${PYTEST_TIMEOUT:-900} python -m pytest tests -m gpu -x -q -k "${PYTEST_K}" > gpurun_out/pytest.log 2>&1; echo "pytest_rc=$?"
tail -15 gpurun_out/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke_rc=$?"
tail -3 gpurun_out/smoke.log
for cfg in ${BENCH_CFGS:-c2}; do
  timeout 900 python bench.py --config $cfg --steps 20 --warmup 5 --no-e2e --no-cpu > gpurun_out/bench_$cfg.json 2> gpurun_out/bench_$cfg.err; echo "bench_${cfg}_rc=$?"
  head -c 400 gpurun_out/bench_$cfg.json; echo
  python -c "import json;d=json.load(open('gpurun_out/bench_$cfg.json'));print({k:d[k] for k in ('value','ms_per_step')}, d['roofline']['frac'], d['phases_profiled_pass'])" 2>/dev/null
done
