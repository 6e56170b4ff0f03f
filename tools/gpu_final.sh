# final round refresh: c3 sweep, smoke, GPU tests, bench lines (c2 default + c3/c4/c5), ncu launch list + leaf
set -x
timeout 1500 python tools/sweep_c3.py --steps 10 > gpurun_out/c3_sweep.jsonl 2> gpurun_out/c3_sweep.err; echo sweep=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench=$?
timeout 600 python bench.py --config c5 --steps 20 --warmup 3 > gpurun_out/bench_c5.json 2>/dev/null; echo c5=$?
timeout 600 python bench.py --config c3 --steps 20 --warmup 3 --no-e2e > gpurun_out/bench_c3.json 2>/dev/null; echo c3=$?
timeout 900 python bench.py --config c4 --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c4.json 2>/dev/null; echo c4=$?
timeout 600 python bench.py --hash-block 0 --steps 50 --warmup 5 --no-e2e --no-cpu > gpurun_out/bench_hb_chunk.json 2>/dev/null; echo hb=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"leaf|levels|compact|verify|bfs|gather" -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/b_ncu.log 2>&1; echo ncu1=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_kernel -s 6 -c 1 -f -o gpurun_out/leaf_full python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/b_ncu2.log 2>&1; echo ncu2=$?
python tools/ncu_summary.py gpurun_out/leaf_full.ncu-rep > gpurun_out/leaf_full_summary.txt 2>&1
