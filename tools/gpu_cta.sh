# K1 CTA shape A/B (warps per CTA at 24 warps/SM); usage: bash tools/gpu_cta.sh
set -x
bash tools/gpu_var.sh "base w4 w6 w12" > gpurun_out/cta_micro.log 2>&1
for v in w4 w6 w12; do
  CKPT_LIB=variants/lib_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "compare_pair or tree_bit_exact" > gpurun_out/cta_pytest_$v.log 2>&1; echo $v pytest=$?
done
bash tools/variant_sweep.sh c2 100 > gpurun_out/cta_c2.log 2>&1
bash tools/variant_sweep.sh c3 30 > gpurun_out/cta_c3.log 2>&1
cat gpurun_out/cta_micro.log gpurun_out/cta_c2.log gpurun_out/cta_c3.log
