set -x
for v in base prefetch base prefetch; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 512,4096,65536 --modes f32,f64 --reps 10 2>&1 | grep -v "^{"
done > gpurun_out/leaf_micro_r9.txt
bash tools/variant_sweep.sh c2 100 > gpurun_out/variants_r9.txt 2>&1
bash tools/variant_sweep.sh c2 100 >> gpurun_out/variants_r9.txt 2>&1
