# K1 two chains per lane at 16 warps/SM (64-byte stages), single-tree builds only; usage: bash tools/gpu_ch2.sh
for v in ch2s64 ch2s64w4; do
  CKPT_LIB=variants/lib_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "tree_bit_exact and not hash_block" > gpurun_out/ch2_pytest_$v.log 2>&1; echo $v pytest=$?; tail -1 gpurun_out/ch2_pytest_$v.log
done
for rep in 1 2; do for v in base ch2s64 ch2s64w4; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,512 --modes f32,f64 --reps 30 2>&1 | grep -v "^{"
done; done
