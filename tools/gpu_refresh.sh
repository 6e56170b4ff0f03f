# round-end style refresh: smoke, GPU tests, bench, ncu launch list + leaf full capture, sanitizers
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"leaf|levels|compact|verify|bfs|gather" -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/b_ncu.log 2>&1; echo ncu1=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_kernel -s 6 -c 1 -f -o gpurun_out/leaf_full python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/b_ncu2.log 2>&1; echo ncu2=$?
python tools/ncu_summary.py gpurun_out/leaf_full.ncu-rep > gpurun_out/leaf_full_summary.txt 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"levels|gather|verify" -s 8 -c 4 -f -o gpurun_out/tail_full python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/b_ncu3.log 2>&1; echo ncu3=$?
python tools/ncu_summary.py gpurun_out/tail_full.ncu-rep > gpurun_out/tail_full_summary.txt 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_run.py > gpurun_out/san_$tool.log 2>&1; echo "$tool rc=$?"
done
