timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_kernel -s 6 -c 1 -f -o gpurun_out/leaf_src python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu=$?
ncu -i gpurun_out/leaf_src.ncu-rep --page source --csv --print-source sass > gpurun_out/leaf_src_sass.csv 2>/dev/null
python tools/step_timeline.py 2>&1 | head -5
