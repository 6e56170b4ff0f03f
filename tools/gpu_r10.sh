set -x
for v in base few1; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 16384,32768,65536 --modes f32,f64 --reps 10 2>&1 | grep -v "^{"
  echo "== $v 0.8GB"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 0.8 --chunks 4096,65536 --modes f32 --reps 10 2>&1 | grep -v "^{"
done > gpurun_out/leaf_micro_r10.txt
timeout 1200 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_r10.log 2>&1; echo pytest=$?
