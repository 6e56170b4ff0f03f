#!/bin/bash
# Captures at the current HEAD: configs[2] sweep, K1 pipe counters + full ncu report of one c2 pair
# launch, and the launch list of a bench run (ncu, serialised, cold).  Output: gpurun_out/h/.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
O=gpurun_out/h; mkdir -p $O
timeout 900 python tools/sweep_c3.py --steps 5 > $O/c3_sweep.jsonl 2> $O/c3_sweep.md; echo "sweep rc=$?"
M=gpu__time_duration.sum,sm__cycles_elapsed.avg,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active
M=$M,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmalite_cycles_active.avg.pct_of_peak_sustained_active
M=$M,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active
M=$M,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fp64.sum,sm__inst_executed_pipe_xu.sum
M=$M,dram__bytes_read.sum,dram__bytes_write.sum,launch__registers_per_thread
timeout 600 ncu --metrics $M --clock-control none -k regex:leaf_ -s 2 -c 1 --csv --log-file $O/k1_pipes.csv python tools/one_pair.py > $O/k1_pipes.log 2>&1; echo "pipes rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 40 -c 60 --csv --log-file $O/launches.csv python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu > $O/launches.log 2>&1; echo "launches rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:leaf_ -s 2 -c 1 -o $O/k1_full python tools/one_pair.py > $O/k1_full.log 2>&1; echo "k1full rc=$?"
