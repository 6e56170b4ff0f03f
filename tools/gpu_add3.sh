for rep in 1 2; do for v in base add3; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,512 --modes f32,f64 --reps 20 2>&1 | grep -v "^{"
done; done
bash tools/gpu_ab.sh "base add3" 2 | grep -E "==|steps|leaf "
