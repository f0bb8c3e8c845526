"""Multi-GPU campaign sharding (DESIGN §1 row e).

A campaign is a set of independent injections decoded from (seed, n) alone, so rank r of W takes
the contiguous index range shard(N, r, W) and the only collective is one all-reduce(SUM) of the
int64 outcome counters [3][5] (plus the optional per-site counters [3][64][5]).  Counters are
therefore identical for every W (sharding invariance).  Backend: NCCL over NVLink on the GPU
box; gloo for the CPU tests of this host logic.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard(n_total: int, rank: int, world: int, first: int = 0) -> tuple[int, int]:
    """Contiguous [first, first + count) slice of rank `rank` (the first n_total % world ranks get one more)."""
    base, extra = divmod(n_total, world)
    start = first + rank * base + min(rank, extra)
    return start, base + (1 if rank < extra else 0)


def step_slice(step: int, rank: int, world: int, per_rank: int, first: int = 0) -> tuple[int, int]:
    """Weak-scaling bench slices: step s of rank r covers [first + (s*W + r)*per_rank, +per_rank)."""
    return first + (step * world + rank) * per_rank, per_rank


def all_reduce_counts(counts: torch.Tensor, group=None) -> torch.Tensor:
    """SUM the outcome counters over ranks in place (no-op without an initialised process group)."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return counts


def all_reduce_max(t: torch.Tensor, group=None) -> torch.Tensor:
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return t


def check_identical(t: torch.Tensor, group=None) -> bool:
    """C4: every rank holds the same tensor (ranges / golden hash) — MIN == MAX across ranks."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return True
    lo, hi = t.clone(), t.clone()
    dist.all_reduce(lo, op=dist.ReduceOp.MIN, group=group)
    dist.all_reduce(hi, op=dist.ReduceOp.MAX, group=group)
    return bool(torch.equal(lo, hi))
