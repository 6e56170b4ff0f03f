timeout 900 python -m pytest tests -m gpu -x -q -k "pair or verify or diff or compare or smoke or full" > gpurun_out/pytest_t.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_t.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
python tools/step_timeline.py 10 2>&1 | head -12
