# hash-block variant: parity tests, bench lines, launch list, ncu of the wide leaf kernel
set -x
timeout 900 python -m pytest tests -m gpu -x -q -k "hash_block" > gpurun_out/pytest_hb.log 2>&1; echo pytest=$?
for hb in 0 64 256; do
  timeout 300 python bench.py --steps 50 --warmup 5 --no-e2e --no-cpu --hash-block $hb > gpurun_out/bench_hb$hb.json 2>> gpurun_out/bench_hb.err
done
timeout 300 python bench.py --steps 50 --warmup 5 --no-e2e --no-cpu > gpurun_out/bench_hb16.json 2>> gpurun_out/bench_hb.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"leaf|levels|compact|verify|bfs" -c 60 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/b_ncu.log 2>&1; echo ncu1=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_kernel -s 6 -c 1 -f -o gpurun_out/leaf_wide_full python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --hash-block 0 > gpurun_out/b_ncu3.log 2>&1; echo ncu3=$?
