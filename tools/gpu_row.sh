for rep in 1 2; do for v in base row; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096 --modes f32,f64 --reps 30 2>&1 | grep -v "^{"
done; done
bash tools/gpu_ab.sh "base row" 1
M=lts__t_sectors_srcunit_tex_op_read.sum,dram__bytes_read.sum,gpu__time_duration.sum,sm__inst_issued.avg.pct_of_peak_sustained_active
for v in base row; do CKPT_LIB=variants/lib_$v.so ncu --metrics $M --clock-control none -k regex:leaf_kernel -s 3 -c 1 python tools/leaf_micro.py --gb 3.2 --chunks 4096 --modes f32 --reps 2 2>&1 | grep -E "lts__|dram__|duration|issued"; done
