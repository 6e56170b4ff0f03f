timeout 600 python -m pytest tests -m gpu -x -q -k "digests or dist" 2>&1 | tail -2
CKPT_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu --no-e2e 2>&1 | tail -1 | cut -c1-250
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu --no-e2e 2>&1 | tail -1 | cut -c1-200
