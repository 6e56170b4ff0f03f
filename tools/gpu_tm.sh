timeout 900 python -m pytest tests -m gpu -x -q -k "pair or verify or diff or compare or smoke or full or stream or host or saved" > gpurun_out/pytest_tm.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_tm.log
CKPT_TILE_GATHER=1 timeout 900 python -m pytest tests -m gpu -x -q -k "tile_compaction or compare_pair" 2>&1 | tail -1
python tools/step_timeline.py 10 2>&1 | head -5
CKPT_TILE_GATHER=1 python tools/step_timeline.py 10 2>&1 | head -5
python tools/step_timeline.py 10 2>&1 | head -5
