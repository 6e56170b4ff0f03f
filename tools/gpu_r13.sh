CKPT_LIB=variants/lib_cap.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,32768,65536 --modes f32,f64 --reps 10 2>&1 | grep -v "^{" > gpurun_out/leaf_micro_r13.txt
CKPT_LIB=variants/lib_cap.so timeout 300 python tools/leaf_micro.py --gb 0.8 --chunks 65536 --modes f32 --reps 10 2>&1 | grep -v "^{" >> gpurun_out/leaf_micro_r13.txt
timeout 1200 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_r13.log 2>&1; echo pytest=$?
timeout 1200 python tools/sweep_c3.py --steps 10 > gpurun_out/sweep_c3_r13.jsonl 2> gpurun_out/sweep_c3_r13.md; echo sweep=$?
