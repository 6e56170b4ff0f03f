"""One rank of the NCCL multi-GPU test (tests/test_gpu_nccl.py), launched by torch.distributed.run.

Every rank compares its own HACC-shaped checkpoint pair (arrays sharded by rank, P:287-291,
P:1303-1304) through dist.compare_runs with the C1/C2 exchange over NCCL, then its shard of ONE
large array through dist.compare_sharded_array, and saves its inputs and results for the
parent test, which checks them against the oracle and the single-GPU result.

usage: nccl_worker.py OUT_DIR
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_middleware_tanaabcrtn24_b200 as ck  # noqa: E402
from paper_conf_middleware_tanaabcrtn24_b200 import dist as ckd  # noqa: E402
import synth  # noqa: E402

CHUNK, EPS = 4096, 1e-6
N_PART = (1 << 17) + 7          # particles per rank (ragged last chunk)
N_BIG = (1 << 21) + 3           # elements of the sharded array


def main():
    out = sys.argv[1]
    rank = int(os.environ["RANK"])
    world = int(os.environ["WORLD_SIZE"])
    local = int(os.environ["LOCAL_RANK"])
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    ck.lib()

    pair = synth.rank_pair(rank, N_PART, seed_base=77, device="cuda")
    res = ckd.compare_runs(pair.a, pair.b, CHUNK, EPS, exchange=True, keep_trees=True)
    torch.cuda.synchronize()

    # one array larger than a GPU's share: every rank draws the same array and keeps its shard
    a = synth.uniform(91, N_BIG, "cuda") * 2.0 - 1.0
    b = a.clone()
    hit = torch.arange(0, N_BIG, 4099, device="cuda")
    b[hit] += 3 * EPS
    lo, hi, _, _ = ckd.array_shard(N_BIG, 4, CHUNK, world, rank)
    sh = ckd.compare_sharded_array(a[lo:hi].contiguous(), b[lo:hi].contiguous(), N_BIG, CHUNK, EPS,
                                   exchange=True)
    torch.cuda.synchronize()

    np.savez(os.path.join(out, f"rank{rank}.npz"),
             a=np.stack([t.cpu().numpy() for t in pair.a]),
             b=np.stack([t.cpu().numpy() for t in pair.b]),
             chunks=res.chunks.cpu().numpy() + res.chunk_offset,
             idx=res.idx.cpu().numpy() + res.elem_offset,
             counts=res.counts.cpu().numpy(),
             root_a=np.frombuffer(res.root_a, np.uint8), root_b=np.frombuffer(res.root_b, np.uint8),
             big_a=a.cpu().numpy() if rank == 0 else np.zeros(0, np.float32),
             big_b=b.cpu().numpy() if rank == 0 else np.zeros(0, np.float32),
             sh_chunks=sh.chunks.cpu().numpy() + sh.chunk_offset,
             sh_idx=sh.idx.cpu().numpy() + sh.elem_offset,
             sh_counts=sh.counts.cpu().numpy(),
             sh_root_a=np.frombuffer(sh.root_a, np.uint8), sh_root_b=np.frombuffer(sh.root_b, np.uint8),
             nccl=np.array(str(torch.cuda.nccl.version())), world=np.array(world))
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
