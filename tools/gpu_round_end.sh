#!/bin/bash
# Round-end measurement pass at HEAD: bench lines per workload and the ncu launch lists of the
# c2 and c5 bench steps (serialised, cold).  Output: gpurun_out/e/.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
O=gpurun_out/e; mkdir -p $O
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_c2_20.json 2> $O/bench_c2_20.err; echo "c2_20 rc=$?"
timeout 900 python bench.py --steps 200 --warmup 10 --no-e2e --no-cpu > $O/bench_c2_200.json 2> $O/bench_c2_200.err; echo "c2_200 rc=$?"
timeout 900 python bench.py --config c5 --steps 20 --warmup 5 --no-cpu > $O/bench_c5.json 2> $O/bench_c5.err; echo "c5 rc=$?"
timeout 900 python bench.py --config c3 --steps 20 --warmup 5 --no-cpu > $O/bench_c3.json 2> $O/bench_c3.err; echo "c3 rc=$?"
timeout 1500 python bench.py --config c4 --snapshots all --steps 5 --warmup 3 --no-e2e --no-cpu > $O/bench_c4_all.json 2> $O/bench_c4_all.err; echo "c4_all rc=$?"
K="regex:leaf|levels|compact|verify|bfs|tile"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 40 --csv --log-file $O/launches_c2.csv python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu > $O/launches_c2.log 2>&1; echo "launches c2 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 30 --csv --log-file $O/launches_c5.csv python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/launches_c5.log 2>&1; echo "launches c5 rc=$?"
for f in $O/bench_*.json; do echo "== $f"; python -c "import json,sys;d=json.load(open(sys.argv[1]));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['clocks'])" $f; done
