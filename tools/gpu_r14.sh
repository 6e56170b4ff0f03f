for c in 512 4096; do
  timeout 600 python bench.py --config c3 --chunk $c --steps 20 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c3_$c.json 2>> gpurun_out/r14.err
done
timeout 600 python bench.py --config c2 --chunk 512 --steps 20 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c2_512.json 2>> gpurun_out/r14.err
