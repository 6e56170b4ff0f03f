set -x
timeout 900 python -m pytest tests -m gpu -x -q -k "stream" > gpurun_out/pytest_r6.log 2>&1; echo pytest=$?
timeout 600 python bench.py --steps 50 --warmup 5 --no-cpu > gpurun_out/bench_r6.json 2> gpurun_out/bench_r6.err; echo bench=$?
