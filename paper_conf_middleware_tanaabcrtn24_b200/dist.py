"""Multi-GPU driver: one process per GPU, checkpoint arrays sharded by rank.

The paper compares each checkpoint pair on a dedicated GPU, independently
(P:287-291): HACC writes one checkpoint per rank
(P:1303-1304), so the arrays shard naturally and no checkpoint byte crosses
GPUs -- the same array index of run A and run B lives on the same GPU.

The only exchanges (NCCL over NVLink/NVSwitch through torch.distributed):
  C1  all-gather of the array roots (16 B each) so every rank builds the same
      top levels over all arrays -> a checkpoint root independent of the GPU
      count (reading R15);
  C2  all-reduce(SUM) of {flagged chunks, differing elements}.
Both messages are < 1 KB: latency-bound, not bandwidth-bound.

The helpers below are backend-agnostic (gloo on CPU tensors in the tests,
NCCL on CUDA tensors in production); compute always goes through libckpt.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Optional, Sequence, Tuple

import torch
import torch.distributed as dist


def shard_range(n_items: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous block [lo, hi) of n_items owned by `rank` (ranks -> GPUs in blocks)."""
    base, extra = divmod(n_items, world)
    lo = rank * base + min(rank, extra)
    hi = lo + base + (1 if rank < extra else 0)
    return lo, hi


def gather_counts(local: Sequence[int], group=None, device="cpu") -> torch.Tensor:
    """All-gather a small int64 vector from every rank -> (world, len(local))."""
    world = dist.get_world_size(group)
    t = torch.tensor(list(local), dtype=torch.int64, device=device)
    out = torch.empty((world, t.numel()), dtype=torch.int64, device=device)
    dist.all_gather_into_tensor(out.view(-1), t, group=group)
    return out


def gather_roots(local_roots: torch.Tensor, group=None) -> torch.Tensor:
    """C1: all-gather (n_local, 16) uint8 root digests in rank order -> (n_total, 16)."""
    world = dist.get_world_size(group)
    n_local = local_roots.shape[0]
    counts = gather_counts([n_local], group, local_roots.device).view(-1).tolist()
    m = max(counts)
    buf = torch.zeros((m, 16), dtype=torch.uint8, device=local_roots.device)
    buf[:n_local] = local_roots
    out = torch.empty((world * m, 16), dtype=torch.uint8, device=local_roots.device)
    dist.all_gather_into_tensor(out.view(-1), buf.view(-1), group=group)
    parts = [out[r * m: r * m + counts[r]] for r in range(world)]
    return torch.cat(parts, 0)


def allreduce_counts(counts: torch.Tensor, group=None) -> torch.Tensor:
    """C2: element-wise SUM of int64 counters over ranks (in place)."""
    dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return counts


@dataclass
class RunComparison:
    root_a: Optional[bytes]            # checkpoint roots over ALL arrays (identical on every rank)
    root_b: Optional[bytes]
    chunks: torch.Tensor               # local flagged chunk ids (local numbering)
    idx: torch.Tensor                  # local differing element ids (local numbering)
    chunk_offset: int                  # add to local ids for global numbering
    elem_offset: int
    counts: torch.Tensor               # device int64 [2]: global {n_chunks, n_diff} after C2
    trees: tuple = ()


def compare_runs(arrays_a: Sequence[torch.Tensor], arrays_b: Sequence[torch.Tensor],
                 chunk_bytes: int, eps: float, group=None, read_roots: bool = True,
                 keep_trees: bool = False, exchange: Optional[bool] = None) -> RunComparison:
    """Compare this rank's arrays of run A and run B (steps 1-4) and join the ranks.

    exchange: run C1/C2 (default: when torch.distributed is initialised with world size > 1;
    True also at world size 1, e.g. to exercise the NCCL path on one GPU)."""
    from . import tree_build, tree_diff_async, tree_from_digests_batch, verify_async

    TA = tree_build(list(arrays_a), chunk_bytes, eps)
    TB = tree_build(list(arrays_b), chunk_bytes, eps)
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    chunks = torch.empty(max(TA.n_leaves, 1), dtype=torch.int64, device="cuda")
    n_elems = sum(t.numel() for t in arrays_a)
    idx = torch.empty(max(n_elems, 1), dtype=torch.int64, device="cuda")
    tree_diff_async(TA, TB, chunks, counts[0:1])
    verify_async(list(arrays_a), list(arrays_b), chunks, counts[0:1], chunk_bytes, eps, idx,
                 counts[1:2])
    initialised = dist.is_available() and dist.is_initialized()
    distributed = initialised and (dist.get_world_size(group) > 1 if exchange is None else exchange)
    chunk_off = elem_off = 0
    local = counts.clone()
    if distributed:
        # two collectives: a fixed-size header (array count, sizes, counts), then the roots
        # of both runs padded to the largest array count; the counts are summed locally and
        # both top trees are built by one levels launch
        world = dist.get_world_size(group)
        r = dist.get_rank(group)
        na = len(arrays_a)
        hdr = torch.stack([torch.tensor([na, TA.n_leaves, n_elems], dtype=torch.int64,
                                        device="cuda"), counts.new_zeros(3)]).view(-1)
        hdr[3:5] = counts
        hdrs = torch.empty((world, 6), dtype=torch.int64, device="cuda")
        dist.all_gather_into_tensor(hdrs.view(-1), hdr, group=group)
        h = hdrs.cpu()
        nas = h[:, 0].tolist()
        m = max(nas)
        send = torch.zeros((2 * m, 16), dtype=torch.uint8, device="cuda")
        TA.array_roots(out=send[:na])
        TB.array_roots(out=send[m:m + na])
        recv = torch.empty((world, 2 * m, 16), dtype=torch.uint8, device="cuda")
        dist.all_gather_into_tensor(recv.view(-1), send.view(-1), group=group)
        ra = torch.cat([recv[k, :nas[k]] for k in range(world)], 0)
        rb = torch.cat([recv[k, m:m + nas[k]] for k in range(world)], 0)
        top_a, top_b = tree_from_digests_batch(torch.cat([ra, rb], 0), [ra.shape[0], rb.shape[0]])
        chunk_off = int(h[:r, 1].sum().item()) if r else 0
        elem_off = int(h[:r, 2].sum().item()) if r else 0
        counts.copy_(hdrs[:, 3:5].sum(0))
    else:
        top_a, top_b = TA, TB
    ra = top_a.root() if read_roots else None
    rb = top_b.root() if read_roots else None
    nl = local.cpu().tolist() if read_roots else [chunks.numel(), idx.numel()]
    res = RunComparison(ra, rb, chunks[: nl[0]], idx[: nl[1]], chunk_off, elem_off, counts,
                        (TA, TB, top_a, top_b) if keep_trees else ())
    return res


# ---------------------------------------------------------------------------
# one array larger than a GPU's share (optional row)
# ---------------------------------------------------------------------------

def array_shard(n_elems: int, elem_bytes: int, chunk_bytes: int, world: int,
                rank: int) -> Tuple[int, int, int, int]:
    """Split ONE array over `world` GPUs so that every shard is an exact subtree of the
    single-GPU tree (level-ordered layout with odd-node promotion, reading R13).

    Shards are blocks of 2^k chunks, 2^k = the smallest power of two >= ceil(L / world): GPU g
    owns chunks [g*2^k, min(L, (g+1)*2^k)).  Node j of level l covers leaves
    [j*2^l, (j+1)*2^l), and a block starts at an even index on every level below k, so the
    pairing and the promotion of the last odd node are the same in the shard's own tree as in the
    global one; the shard root is global node (k, g).  The tree over the gathered shard roots
    (ckpt_tree_from_digests) is therefore levels k.. of the global tree and its root the
    single-GPU root.  Returns (elem_lo, elem_hi, chunk_lo, k); an empty shard has lo == hi."""
    L = -(-n_elems * elem_bytes // chunk_bytes)
    per = -(-L // world)
    k = max(0, (per - 1).bit_length())
    c_lo = min(L, rank << k)
    c_hi = min(L, (rank + 1) << k)
    per_elems = chunk_bytes // elem_bytes
    return min(n_elems, c_lo * per_elems), min(n_elems, c_hi * per_elems), c_lo, k


def compare_sharded_array(a_local: torch.Tensor, b_local: torch.Tensor, n_total: int,
                          chunk_bytes: int, eps: float, group=None,
                          exchange: Optional[bool] = None) -> RunComparison:
    """Compare this GPU's shard (array_shard) of ONE large array of run A and run B.

    Every rank builds its subtree, C1 all-gathers the shard roots (empty shards send none) and
    every rank builds the same top levels -> the single-GPU root; C2 all-reduces the counts.
    Local ids are shifted to global ones with chunk_offset / elem_offset."""
    from . import compare_pair_async, tree_from_digests
    initialised = dist.is_available() and dist.is_initialized()
    world = dist.get_world_size(group) if initialised else 1
    rank = dist.get_rank(group) if world > 1 else 0
    collect = initialised and (world > 1 if exchange is None else exchange)
    lo, hi, c_lo, _ = array_shard(n_total, a_local.element_size(), chunk_bytes, world, rank)
    if a_local.numel() != hi - lo or b_local.numel() != hi - lo:
        raise ValueError(f"rank {rank} must hold elements [{lo}, {hi}) of the array")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    chunks = torch.empty(max(1, -(-(hi - lo) * a_local.element_size() // chunk_bytes)),
                         dtype=torch.int64, device="cuda")
    idx = torch.empty(max(1, hi - lo), dtype=torch.int64, device="cuda")
    if hi > lo:
        TA, TB = compare_pair_async([a_local], [b_local], chunk_bytes, eps, chunks, idx, counts)
        ra, rb = TA.array_roots(), TB.array_roots()
    else:
        TA = TB = None
        ra = rb = torch.zeros((0, 16), dtype=torch.uint8, device="cuda")
    local = counts.clone()
    if collect:
        roots_a, roots_b = gather_roots(ra, group), gather_roots(rb, group)
        allreduce_counts(counts, group)
    else:
        roots_a, roots_b = ra, rb
    top_a, top_b = tree_from_digests(roots_a), tree_from_digests(roots_b)
    nl = local.cpu().tolist()
    return RunComparison(top_a.root(), top_b.root(), chunks[: nl[0]], idx[: nl[1]], c_lo, lo,
                         counts, (TA, TB, top_a, top_b))
