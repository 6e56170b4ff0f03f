timeout 1200 python -m pytest tests -m gpu -x -q -k "tree or pair or leaf or special or exhaustive or hash_block or c3 or f64 or verify" 2>&1 | tail -1
timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,512,65536 --modes f32,f64 --reps 20 2>&1 | grep -v "^{"
timeout 600 python bench.py --config c3 --steps 20 --warmup 3 --no-cpu --no-e2e 2>&1 | tail -1 | cut -c1-150
python tools/step_timeline.py 20 2>&1 | head -2
