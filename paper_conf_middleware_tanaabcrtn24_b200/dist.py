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
                 keep_trees: bool = False) -> RunComparison:
    """Compare this rank's arrays of run A and run B (steps 1-4) and join the ranks.

    With torch.distributed uninitialised (or world size 1) no collective runs."""
    from . import tree_build, tree_diff_async, tree_from_digests, verify_async

    TA = tree_build(list(arrays_a), chunk_bytes, eps)
    TB = tree_build(list(arrays_b), chunk_bytes, eps)
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    chunks = torch.empty(max(TA.n_leaves, 1), dtype=torch.int64, device="cuda")
    n_elems = sum(t.numel() for t in arrays_a)
    idx = torch.empty(max(n_elems, 1), dtype=torch.int64, device="cuda")
    tree_diff_async(TA, TB, chunks, counts[0:1])
    verify_async(list(arrays_a), list(arrays_b), chunks, counts[0:1], chunk_bytes, eps, idx,
                 counts[1:2])
    distributed = dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1
    chunk_off = elem_off = 0
    local = counts.clone()
    if distributed:
        roots_a = gather_roots(TA.array_roots(), group)
        roots_b = gather_roots(TB.array_roots(), group)
        top_a, top_b = tree_from_digests(roots_a), tree_from_digests(roots_b)
        sizes = gather_counts([TA.n_leaves, n_elems], group, "cuda")
        r = dist.get_rank(group)
        chunk_off = int(sizes[:r, 0].sum().item()) if r else 0
        elem_off = int(sizes[:r, 1].sum().item()) if r else 0
        allreduce_counts(counts, group)
    else:
        top_a, top_b = TA, TB
    ra = top_a.root() if read_roots else None
    rb = top_b.root() if read_roots else None
    nl = local.cpu().tolist() if read_roots else [chunks.numel(), idx.numel()]
    res = RunComparison(ra, rb, chunks[: nl[0]], idx[: nl[1]], chunk_off, elem_off, counts,
                        (TA, TB, top_a, top_b) if keep_trees else ())
    return res
