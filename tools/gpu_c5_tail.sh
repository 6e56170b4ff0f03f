#!/bin/bash
# c5 post-K1 tail: per-kernel step timeline and the ncu launch list of a short c5 bench.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
if [ -n "$RUN_TESTS" ]; then
  timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/pytest.log 2>&1; echo "pytest_rc=$?"
  tail -4 gpurun_out/pytest.log
fi
timeout 600 python tools/step_timeline.py 5 --c5 > gpurun_out/c5_timeline.txt 2>&1; echo "timeline_rc=$?"
cat gpurun_out/c5_timeline.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv \
  --log-file gpurun_out/c5_launches.csv python bench.py --config c5 --steps 2 --warmup 1 --no-e2e --no-cpu \
  > gpurun_out/c5_ncu_bench.log 2>&1; echo "ncu_rc=$?"
python tools/launches_md.py gpurun_out/c5_launches.csv | head -30
