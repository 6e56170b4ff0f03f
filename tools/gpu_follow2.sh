#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
timeout 900 python -m pytest tests -m gpu -x -q -k "${PYTEST_K:-pair or fused or config2 or c4_snapshot or c5 or flagged}" > gpurun_out/pytest.log 2>&1; echo "pytest_rc=$?"
tail -3 gpurun_out/pytest.log
timeout 300 python tools/probe_follow.py variants/ftrace/libckpt.so --ftrace
timeout 600 python tools/probe_follow.py variants/ftrace/libckpt.so --ftrace --c5
for rep in 1 2; do
for f in 0 1; do
  for cfg in c2 c5; do
    flag=""; [ "$cfg" = c5 ] && flag="--c5"
    echo "== CKPT_FOLLOW=$f $cfg rep $rep"
    CKPT_FOLLOW=$f timeout 600 python tools/step_timeline.py 20 $flag 2>&1 | head -4
  done
done
done
