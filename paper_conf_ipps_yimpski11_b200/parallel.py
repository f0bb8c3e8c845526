"""Multi-GPU sharding (DESIGN §1 row e): campaigns and single runs.

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


def part_slice(units: int, granule: int, rank: int, world: int) -> tuple[int, int]:
    """Single-run shard of rank r: a contiguous run of partition units, cut on `granule` multiples
    (CP rows come in blocks of `by`); the slices of all ranks partition [0, units)."""
    blocks = (units + granule - 1) // granule
    b0, nb = shard(blocks, rank, world)
    return min(b0 * granule, units), min((b0 + nb) * granule, units)


def run_single_sharded(hk, dev, ranges, rank: int, world: int, variant=None, group=None):
    """One protected single run split over the ranks: rank r computes its part
    (hauberk_run_part); CP rows / MRI-Q voxels are assembled on every rank by an all-gather of the
    parts (exact), TPACF's partial histograms by one all-reduce(SUM).  Returns (output, alarm, fail)
    with the control-block alarm / fail bits OR-ed over the ranks.  `hk` is the binding module."""
    variant = hk.HK_FT if variant is None else variant
    units, gran = hk.part_units(dev)
    b, e = part_slice(units, gran, rank, world)
    cb = hk.new_control(dev.output()[0].device if isinstance(dev.output(), tuple) else dev.output().device)
    hk.run_part(dev, b, e, variant, ranges, cb)
    words = cb.view(torch.int32)[:2].clone()  # alarm, fail
    multi = dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1
    if dev.bench == 2:
        hist = dev.output()
        if multi:
            dist.all_reduce(hist, op=dist.ReduceOp.SUM, group=group)
        out = hist
    else:
        flat = [dev.output()] if dev.bench == 0 else list(dev.output())
        row = dev.nx if dev.bench == 0 else 1  # elements per unit
        if multi:
            spans = [part_slice(units, gran, r, world) for r in range(world)]
            width = max(q - p for p, q in spans) * row
            for t in flat:
                v = t.view(-1)
                mine = torch.zeros(width, dtype=v.dtype, device=v.device)
                mine[: (e - b) * row] = v[b * row: e * row]
                got = [torch.empty_like(mine) for _ in range(world)]
                dist.all_gather(got, mine, group=group)
                for r, (p, q) in enumerate(spans):
                    v[p * row: q * row] = got[r][: (q - p) * row]
        out = dev.output()
    if multi:
        allw = [torch.empty_like(words) for _ in range(dist.get_world_size(group))]
        dist.all_gather(allw, words, group=group)
        words = torch.stack(allw)
    w = words.view(-1, 2).cpu()
    alarm = fail = 0
    for a, f in w.tolist():
        alarm |= a & 0xFFFFFFFF
        fail |= f & 0xFFFFFFFF
    return out, alarm, fail
