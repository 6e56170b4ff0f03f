set -x
timeout 600 python bench.py --steps 50 --warmup 5 --no-cpu > gpurun_out/bench_r7.json 2> gpurun_out/bench_r7.err; echo bench=$?
timeout 600 python bench.py --config c5 --steps 20 --warmup 3 --no-cpu > gpurun_out/bench_r7_c5.json 2>> gpurun_out/bench_r7.err; echo bench=$?
