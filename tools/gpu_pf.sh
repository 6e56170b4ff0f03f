# K1 staging L2 prefetch-size hint A/B; usage: bash tools/gpu_pf.sh
set -x
bash tools/gpu_var.sh "base pf256 pf64 pf0" > gpurun_out/pf_micro.log 2>&1
bash tools/variant_sweep.sh c2 100 > gpurun_out/pf_c2.log 2>&1
bash tools/variant_sweep.sh c3 30 > gpurun_out/pf_c3.log 2>&1
cat gpurun_out/pf_micro.log gpurun_out/pf_c2.log gpurun_out/pf_c3.log
