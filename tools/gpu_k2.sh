timeout 900 python -m pytest tests -m gpu -x -q -k "levels or tree or pair or digest" > gpurun_out/pytest_k2.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_k2.log
python tools/levels_micro.py
python tools/step_timeline.py 2>&1 | head -5
echo "== old"; CKPT_LIB=variants/lib_lvold.so python tools/step_timeline.py 2>&1 | head -5
ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,sm__inst_issued.avg.pct_of_peak_sustained_active -k regex:levels --clock-control none -s 10 -c 2 python tools/step_timeline.py 2>&1 | grep -E "duration|inst_exec|issued" 
