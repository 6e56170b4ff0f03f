for v in new lvold; do
  L=""; [ $v = lvold ] && L=variants/lib_lvold.so
  echo "== $v c3 C=512"; CKPT_LIB=${L:-paper_conf_middleware_tanaabcrtn24_b200/libckpt.so} timeout 600 python bench.py --config c3 --chunk 512 --eps 1e-6 --steps 10 --warmup 3 --no-cpu --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['phases_profiled_pass'])"
  echo "== $v c3 C=4096"; CKPT_LIB=${L:-paper_conf_middleware_tanaabcrtn24_b200/libckpt.so} timeout 600 python bench.py --config c3 --chunk 4096 --eps 1e-6 --steps 10 --warmup 3 --no-cpu --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['phases_profiled_pass'])"
done
timeout 600 python bench.py --config c5 --steps 20 --warmup 3 > gpurun_out/bench_c5.json 2>/dev/null; tail -1 gpurun_out/bench_c5.json | cut -c1-300
timeout 600 python bench.py --config c3 --steps 20 --warmup 3 --no-e2e > gpurun_out/bench_c3.json 2>/dev/null; tail -1 gpurun_out/bench_c3.json | cut -c1-300
