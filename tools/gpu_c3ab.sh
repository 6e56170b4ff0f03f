for v in prev fast; do
  echo "== $v c3 C=512"; CKPT_LIB=variants/lib_$v.so timeout 600 python bench.py --config c3 --chunk 512 --eps 1e-6 --steps 10 --warmup 3 --no-cpu --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['phases_profiled_pass'])"
done
timeout 600 python -m pytest tests -m gpu -x -q -k "levels or tree or pair or digests" 2>&1 | tail -1
