timeout 600 python bench.py --path saved --steps 50 --warmup 5 --no-cpu --no-e2e > gpurun_out/bench_saved.json 2> gpurun_out/bench_saved.err; echo rc=$?
timeout 600 python bench.py --path saved --config c5 --steps 20 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_saved_c5.json 2>> gpurun_out/bench_saved.err; echo rc=$?
