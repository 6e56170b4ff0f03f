# K1 staging geometry A/B (segment bytes x ring depth); usage: bash tools/gpu_seg.sh
set -x
bash tools/gpu_var.sh "base s256x1 s256x1u1 s64x3" > gpurun_out/seg_micro.log 2>&1
for v in s256x1 s256x1u1; do
  CKPT_LIB=variants/lib_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "compare_pair or tree_bit_exact or hash_block" > gpurun_out/seg_pytest_$v.log 2>&1; echo $v pytest=$?
done
bash tools/variant_sweep.sh c2 100 > gpurun_out/seg_c2.log 2>&1
bash tools/variant_sweep.sh c3 30 > gpurun_out/seg_c3.log 2>&1
cat gpurun_out/seg_micro.log gpurun_out/seg_c2.log gpurun_out/seg_c3.log
