timeout 1200 python -m pytest tests -m gpu -x -q -k "verify or pair or diff or compare or stream or host or saved or full or tile" > gpurun_out/pytest_ss.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_ss.log
for rep in 1 2; do python tools/step_timeline.py 20 2>&1 | head -5; done
