for c in c2 c5 c3; do for pth in fused unfused; do
python bench.py --config $c --path $pth --steps 30 --warmup 5 --no-cpu --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['name'], d['config']['path'], d['value'], d['ms_per_step'], d['roofline']['achieved'], {k: v['ms_per_step'] for k, v in d['phases_profiled_pass'].items() if isinstance(v, dict)}, d['flagged_chunks_per_gpu'], d['diff_elems_per_gpu'])"
done; done
