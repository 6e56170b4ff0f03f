#!/bin/bash
# Full GPU suite and smoke() at HEAD.  Output: gpurun_out/f/.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
O=gpurun_out/f; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; echo "tests rc=$? $(tail -1 $O/gpu_tests.log)"
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; echo "smoke rc=$? $(tail -1 $O/smoke.log)"
# compute-sanitizer is closed on the GPU pool (round 2): profiles/r2_sanitizer.md holds the last run
