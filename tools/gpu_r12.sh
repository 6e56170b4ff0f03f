for v in lat; do
  echo "== $v (LAT on)"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,16384,32768,65536 --modes f32,f64 --reps 10 2>&1 | grep -v "^{"
  CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 0.8 --chunks 8192,65536 --modes f32 --reps 10 2>&1 | grep -v "^{"
  echo "== $v (LAT off)"; CKPT_LEAF_LAT=0 CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,16384,32768,65536 --modes f32,f64 --reps 10 2>&1 | grep -v "^{"
  CKPT_LEAF_LAT=0 CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 0.8 --chunks 8192,65536 --modes f32 --reps 10 2>&1 | grep -v "^{"
done > gpurun_out/leaf_micro_r12.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_r12.log 2>&1; echo pytest=$?
