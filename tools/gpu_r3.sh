set -x
timeout 900 python -m pytest tests -m gpu -x -q -k "serialize or oracle_written or compare_saved or hash_block" > gpurun_out/pytest_persist.log 2>&1; echo pytest=$?
bash tools/variant_sweep.sh c2 100 > gpurun_out/variants.txt 2>&1
bash tools/variant_sweep.sh c2 100 >> gpurun_out/variants.txt 2>&1
timeout 600 python bench.py --config c5 --steps 30 --warmup 3 --no-cpu > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 python bench.py --config c3 --steps 30 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
