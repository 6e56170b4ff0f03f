#!/bin/bash
# What the driver runs at round end, in order: build, GPU suite, smoke, reference arm, our arm.
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
O=gpurun_out/d; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; echo "tests rc=$? $(tail -1 $O/gpu_tests.log)"
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; echo "smoke rc=$? $(tail -1 $O/smoke.log)"
t0=$(date +%s); timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $O/ref.json 2> $O/ref.err; echo "ref rc=$? wall $(( $(date +%s) - t0 )) s"
t0=$(date +%s); timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $O/ours.json 2> $O/ours.err; echo "ours rc=$? wall $(( $(date +%s) - t0 )) s"
wc -l $O/ref.json $O/ours.json
python -c "import json;d=json.load(open('$O/ours.json'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['clocks'],d['e2e']['value'],d['e2e'].get('saved_tree',{}).get('value'))"
python -c "import json;d=json.load(open('$O/ref.json'));print(d['value'],d['ms_per_step'],d['cpu_baseline']['cores'])"
