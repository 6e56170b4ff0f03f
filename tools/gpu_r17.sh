timeout 1200 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_r17.log 2>&1; echo pytest=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"leaf|levels|compact|verify|bfs" -c 12 --csv --log-file gpurun_out/launches_c3_512_r17.csv python bench.py --config c3 --chunk 512 --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"leaf|levels|compact|verify|bfs" -c 12 --csv --log-file gpurun_out/launches_c2_r17.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
timeout 600 python bench.py --config c3 --chunk 512 --steps 20 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c3_512_r17.json 2>> gpurun_out/r17.err
timeout 600 python bench.py --steps 50 --warmup 5 --no-cpu --no-e2e > gpurun_out/bench_c2_r17.json 2>> gpurun_out/r17.err
