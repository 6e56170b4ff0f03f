#!/bin/bash
# Round-2 measurement pass: bench lines per workload, K1 pipe balance and traffic (ncu), launch list.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out/m
O=gpurun_out/m
timeout 900 python bench.py --steps 200 --warmup 10 > $O/bench_c2_200.json 2> $O/bench_c2_200.err; echo "c2_200 rc=$?"
timeout 900 python bench.py --config c5 --steps 20 --warmup 5 --no-cpu > $O/bench_c5.json 2> $O/bench_c5.err; echo "c5 rc=$?"
timeout 900 python bench.py --config c3 --steps 20 --warmup 5 --no-cpu > $O/bench_c3.json 2> $O/bench_c3.err; echo "c3 rc=$?"
timeout 1500 python bench.py --config c4 --snapshots all --steps 5 --warmup 3 --no-e2e --no-cpu > $O/bench_c4_all.json 2> $O/bench_c4_all.err; echo "c4_all rc=$?"
M=gpu__time_duration.sum,sm__cycles_elapsed.avg,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active
M=$M,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmalite_cycles_active.avg.pct_of_peak_sustained_active
M=$M,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active
M=$M,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_xu_cycles_active.avg.pct_of_peak_sustained_active
M=$M,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_fmalite.sum,sm__inst_executed_pipe_alu.sum
M=$M,sm__inst_executed_pipe_fp64.sum,sm__inst_executed_pipe_xu.sum,sm__inst_executed_pipe_lsu.sum,sm__inst_executed_pipe_uniform.sum
M=$M,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_active.avg
timeout 600 ncu --metrics $M --clock-control none -k regex:leaf_ -s 2 -c 1 --csv --log-file $O/k1_pipes.csv python tools/one_pair.py > $O/k1_pipes.log 2>&1; echo "pipes rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 40 -c 60 --csv --log-file $O/launches.csv python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu > $O/launches.log 2>&1; echo "launches rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:leaf_ -s 2 -c 1 -o $O/k1_full python tools/one_pair.py > $O/k1_full.log 2>&1; echo "k1full rc=$?"
for f in $O/bench_*.json; do echo "== $f"; head -c 300 $f; echo; done
