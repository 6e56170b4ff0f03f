"""Multi-process GPU tests of the multi-GPU driver (paper_conf_middleware_tanaabcrtn24_b200.dist):
two ranks share cuda:0 over the gloo backend (the GPU box has one GPU), so the collectives,
the shard bookkeeping and the top tree run for real with libckpt compute on both ranks.
Roots and counts must equal the single-process results (reading R15)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from paper_conf_middleware_tanaabcrtn24_b200 import dist as ckd
        # (1) checkpoint arrays sharded by rank
        pair = synth.c5_pair(n_ranks=1, n_particles=(1 << 16) + 40, seed=97, device="cuda")
        lo, hi = ckd.shard_range(len(pair.a), world, rank)
        r1 = ckd.compare_runs(pair.a[lo:hi], pair.b[lo:hi], 4096, pair.eps)
        # (2) one array sharded into exact subtrees
        big = synth.c3_pair(n=(1 << 20) + 33, seed=98, device="cuda", n_clusters=20, mean_len=300)
        alo, ahi, _, _ = ckd.array_shard(big.a[0].numel(), 8, 2048, world, rank)
        r2 = ckd.compare_sharded_array(big.a[0][alo:ahi], big.b[0][alo:ahi], big.a[0].numel(), 2048,
                                       big.eps)
        q.put((rank, r1.root_a, r1.root_b, r1.counts.cpu().tolist(),
               (r1.chunks + r1.chunk_offset).cpu().numpy(), (r1.idx + r1.elem_offset).cpu().numpy(),
               r2.root_a, r2.root_b, r2.counts.cpu().tolist(),
               (r2.chunks + r2.chunk_offset).cpu().numpy(), (r2.idx + r2.elem_offset).cpu().numpy()))
    finally:
        dist.destroy_process_group()


def test_two_ranks_on_one_gpu_match_single_process():
    import paper_conf_middleware_tanaabcrtn24_b200 as ck
    import synth
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted([q.get(timeout=300) for _ in range(2)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    # single-process references
    pair = synth.c5_pair(n_ranks=1, n_particles=(1 << 16) + 40, seed=97, device="cuda")
    ch, ix, nc, nd, ra, rb = ck.compare(pair.a, pair.b, 4096, pair.eps)
    big = synth.c3_pair(n=(1 << 20) + 33, seed=98, device="cuda", n_clusters=20, mean_len=300)
    ch2, ix2, nc2, nd2, ra2, rb2 = ck.compare(big.a, big.b, 2048, big.eps)
    for rank, a1, b1, c1, chunks1, idx1, a2, b2, c2, chunks2, idx2 in out:
        assert (a1, b1) == (ra, rb) and c1 == [nc, nd]
        assert (a2, b2) == (ra2, rb2) and c2 == [nc2, nd2]
    assert np.array_equal(np.concatenate([o[4] for o in out]), ch.cpu().numpy())
    assert np.array_equal(np.concatenate([o[5] for o in out]), ix.cpu().numpy())
    assert np.array_equal(np.concatenate([o[9] for o in out]), ch2.cpu().numpy())
    assert np.array_equal(np.concatenate([o[10] for o in out]), ix2.cpu().numpy())
