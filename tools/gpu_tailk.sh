timeout 600 ncu --set full --clock-control none --import-source on -k regex:"levels|compact|verify|bfs" -s 30 -c 8 -f -o gpurun_out/tail_full python bench.py --steps 3 --warmup 5 --no-e2e --no-cpu > gpurun_out/tail_ncu.log 2>&1; echo ncu=$?
python tools/ncu_summary.py gpurun_out/tail_full.ncu-rep > gpurun_out/tail_summary.txt 2>&1
