for rep in 1 2; do for v in base h1 h2; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096 --modes f32 --reps 20 2>&1 | grep -v "^{"
done; done
bash tools/gpu_ab.sh "base h1 h2" 2 | grep -E "==|steps"
