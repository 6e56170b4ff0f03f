# leaf-kernel A/B of tuning variants (variants/lib_*.so); usage: bash tools/gpu_var.sh "v1 v2 ..." [ncu_variant]
vs=${1:-"base mix"}
for rep in 1 2; do for v in $vs; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096 --modes f32 --reps 30 2>&1 | grep -v "^{"
done; done
M=sm__inst_executed.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_issued.avg.pct_of_peak_sustained_active,sm__cycles_elapsed.avg.per_second,gpu__time_duration.sum,smsp__average_warp_latency_issue_stalled_math_pipe_throttle.ratio,smsp__average_warp_latency_issue_stalled_dispatch_stall.ratio,smsp__average_warp_latency_issue_stalled_wait.ratio,smsp__average_warp_latency_issue_stalled_not_selected.ratio
for v in ${2:-}; do
  CKPT_LIB=variants/lib_$v.so timeout 600 ncu --metrics $M --clock-control none -k regex:leaf_kernel -s 3 -c 1 --csv python tools/leaf_micro.py --gb 3.2 --chunks 4096 --modes f32 --reps 2 > gpurun_out/ncu_$v.csv 2>&1
done
