#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out/m
O=gpurun_out/m
timeout 1500 python bench.py --config c4 --snapshots all --steps 5 --warmup 3 --no-e2e --no-cpu > $O/bench_c4_all.json 2> $O/bench_c4_all.err; echo "c4_all rc=$?"; tail -3 $O/bench_c4_all.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"leaf|levels|compact|verify|bfs|tile" -c 40 --csv --log-file $O/launches.csv python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu > $O/launches.log 2>&1; echo "launches rc=$?"
timeout 1500 python tools/sweep_c3.py --steps 5 > $O/c3_sweep.jsonl 2> $O/c3_sweep.md; echo "sweep rc=$?"
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_c2_20.json 2> $O/bench_c2_20.err; echo "c2_20 rc=$?"
for f in $O/bench_c4_all.json $O/bench_c2_20.json; do echo "== $f"; head -c 300 $f; echo; done
