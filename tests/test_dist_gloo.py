"""Multi-process (world_size 2, gloo, CPU) tests of the multi-GPU driver's host logic.

The collectives C1 (all-gather of array roots) and C2 (all-reduce of counts)
run here on CPU tensors; the per-array roots come from the oracle (test-only),
so the checkpoint root can be checked to be independent of the rank count
(reading R15)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_middleware_tanaabcrtn24_b200 import dist as ckd


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _arrays(n_arrays=7):
    rng = np.random.default_rng(123)
    return [rng.uniform(-1, 1, int(rng.integers(1, 20000))).astype(np.float32)
            for _ in range(n_arrays)]


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        arrays = _arrays()
        lo, hi = ckd.shard_range(len(arrays), world, rank)
        mine = arrays[lo:hi]
        roots = np.stack([oracle.levels(oracle.leaves(a, 256, 1e-4))[-1] for a in mine])
        gathered = ckd.gather_roots(torch.from_numpy(roots))
        top = oracle.levels(gathered.numpy())[-1].tobytes()
        sizes = ckd.gather_counts([sum(oracle.n_chunks(a.size, 0, 256) for a in mine),
                                   sum(a.size for a in mine)])
        counts = torch.tensor([rank + 1, 10 * (rank + 1)], dtype=torch.int64)
        ckd.allreduce_counts(counts)
        q.put((rank, top, gathered.numpy().tobytes(), sizes.tolist(), counts.tolist()))
    finally:
        dist.destroy_process_group()


def _run(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out)


def test_shard_range_covers_all_items_in_rank_order():
    for n in (1, 5, 7, 64, 1000):
        for world in (1, 2, 3, 4, 8):
            spans = [ckd.shard_range(n, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == n
            for (a, b), (c, d) in zip(spans, spans[1:]):
                assert b == c and a <= b
            assert max(b - a for a, b in spans) - min(b - a for a, b in spans) <= 1


@pytest.mark.parametrize("world", [1, 2])
def test_root_is_independent_of_rank_count_gloo(world):
    import oracle
    arrays = _arrays()
    ref = oracle.build_checkpoint(arrays, 256, 1e-4)
    res = _run(world)
    for rank, top, gathered, sizes, counts in res:
        assert top == ref.root
        assert np.frombuffer(gathered, np.uint8).reshape(-1, 16).tolist() == ref.array_roots.tolist()
        assert counts == [sum(r + 1 for r in range(world)), sum(10 * (r + 1) for r in range(world))]
        tot_chunks = sum(s[0] for s in sizes)
        assert tot_chunks == sum(ref.n_leaves)
        assert sum(s[1] for s in sizes) == sum(a.size for a in arrays)


# ------------------------------------------- one array sharded over GPUs ----

@pytest.mark.parametrize("world", [1, 2, 3, 4, 5, 8])
@pytest.mark.parametrize("n", [1, 100, 4096, 100_003, 262_144])
def test_array_shard_subtree_roots_give_the_single_gpu_root(world, n):
    # pins the subtree property array_shard relies on, with the oracle standing in for the GPU
    import oracle
    rng = np.random.default_rng(n + world)
    a = rng.uniform(-1, 1, n).astype(np.float32)
    C = 512
    ref = oracle.levels(oracle.leaves(a, C, 1e-5))[-1]
    roots, spans = [], []
    for r in range(world):
        lo, hi, c_lo, k = ckd.array_shard(n, 4, C, world, r)
        spans.append((lo, hi))
        if hi > lo:
            assert c_lo == r << k and lo == c_lo * (C // 4)
            roots.append(oracle.levels(oracle.leaves(a[lo:hi], C, 1e-5))[-1])
    assert spans[0][0] == 0 and max(h for _, h in spans) == n
    for (a0, b0), (a1, b1) in zip(spans, spans[1:]):
        assert b0 == a1 or (a1 == b1 == n)
    top = oracle.levels(np.stack(roots))[-1]
    assert top.tobytes() == ref.tobytes()


def _shard_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        rng = np.random.default_rng(7)
        a = rng.uniform(-1, 1, 70_001).astype(np.float32)
        lo, hi, _, _ = ckd.array_shard(a.size, 4, 1024, world, rank)
        root = oracle.levels(oracle.leaves(a[lo:hi], 1024, 1e-5))[-1:]
        gathered = ckd.gather_roots(torch.from_numpy(root.copy()))
        q.put((rank, oracle.levels(gathered.numpy())[-1].tobytes()))
    finally:
        dist.destroy_process_group()


def test_array_shard_root_over_gloo_world2():
    import oracle
    rng = np.random.default_rng(7)
    a = rng.uniform(-1, 1, 70_001).astype(np.float32)
    ref = oracle.levels(oracle.leaves(a, 1024, 1e-5))[-1].tobytes()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(top == ref for _, top in out)
