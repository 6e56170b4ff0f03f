for v in few1 look look_m1 minb1; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,32768,65536 --modes f32,f64 --reps 10 2>&1 | grep -v "^{"
  CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 0.8 --chunks 65536 --modes f32 --reps 10 2>&1 | grep -v "^{"
done > gpurun_out/leaf_micro_r11.txt 2>&1
bash tools/variant_sweep.sh c2 100 > gpurun_out/variants_r11.txt 2>&1
