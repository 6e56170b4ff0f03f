timeout 1200 python -m pytest tests -m gpu -x -q -k "pair or stream or saved or c4 or c5" > gpurun_out/pytest_r18.log 2>&1; echo pytest=$?
for rep in 1 2; do
for v in fences acqrel; do
  CKPT_LIB=variants/lib_$v.so timeout 300 python bench.py --config c3 --chunk 512 --steps 20 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v c3/512', d['value'], d['phases_profiled_pass']['leaf'])"
  CKPT_LIB=variants/lib_$v.so timeout 300 python bench.py --steps 50 --warmup 5 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v c2', d['value'], d['phases_profiled_pass']['leaf'])"
done; done > gpurun_out/acqrel_r18.txt
