"""Host logic of the multi-GPU campaign on CPU: contiguous shards, weak-scaling
step slices, and the counters all-reduce over a world-size-2 gloo group.  The per-shard campaigns
run in the CPU oracle (test infrastructure); the reduction/sharding code is the product's."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_yimpski11_b200 import parallel as par


@pytest.mark.parametrize("n,w", [(0, 1), (1, 2), (10, 3), (1000, 8), (1000003, 7)])
def test_shards_partition_the_index_range(n, w):
    spans = [par.shard(n, r, w, first=5) for r in range(w)]
    covered = []
    for s, c in spans:
        covered.extend(range(s, s + c))
    assert covered == list(range(5, 5 + n))
    sizes = [c for _, c in spans]
    assert max(sizes) - min(sizes) <= 1


def test_step_slices_are_disjoint_across_ranks_and_steps():
    seen = set()
    for s in range(4):
        for r in range(3):
            a, c = par.step_slice(s, r, 3, 10)
            idx = set(range(a, a + c))
            assert not (idx & seen)
            seen |= idx
    assert seen == set(range(120))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, total, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle as O
    import workloads as W
    probs = [W.cp_small(), W.mriq_problem(4, 23, n_vox=60), W.tpacf_small(n=60, n_rand=1)]
    R = [O.profile_ranges(b, probs[b]) for b in range(3)]
    first, cnt = par.shard(total, rank, world)
    c, _ = O.campaign(-1, probs, R, seed=777, first=first, count=cnt, mode=1, records=False)
    t = torch.from_numpy(c.copy())
    par.all_reduce_counts(t)
    same = par.check_identical(torch.tensor([float(R[0].det[0].lo[0]), float(R[0].det[0].hi[0])], dtype=torch.float64))
    differ = par.check_identical(torch.tensor([float(rank)]))
    m = torch.tensor([float(rank + 1)])
    par.all_reduce_max(m)
    if rank == 0:
        q.put((t.numpy().tolist(), same, differ, float(m.item())))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_counters_equal_single_process():
    import oracle as O
    import workloads as W
    total = 301
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, total, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    probs = [W.cp_small(), W.mriq_problem(4, 23, n_vox=60), W.tpacf_small(n=60, n_rand=1)]
    R = [O.profile_ranges(b, probs[b]) for b in range(3)]
    c, _ = O.campaign(-1, probs, R, seed=777, first=0, count=total, mode=1, records=False)
    counts, same, differ, mx = res
    assert np.array_equal(np.array(counts), c)
    assert same is True and differ is False and mx == 2.0


# ---- single-run sharding host logic: part slices + assembly over a gloo group
@pytest.mark.parametrize("units,gran,w", [(512, 16, 1), (512, 16, 3), (64, 16, 8), (32768, 1, 7), (72, 1, 5), (5, 1, 8)])
def test_part_slices_partition_the_units_on_granule_boundaries(units, gran, w):
    spans = [par.part_slice(units, gran, r, w) for r in range(w)]
    pos = 0
    for b, e in spans:
        assert b == pos and e >= b
        assert b % gran == 0 and (e % gran == 0 or e == units)
        pos = e
    assert pos == units


class _FakeHK:
    """Stand-in for the binding: run_part writes a known function of the global unit index into
    the part (CP rows, MRI-Q voxels) or adds per-row counts into a zeroed hist (TPACF), with the
    library's zeroing rules; the control block gets alarm bit (1 << rank) on rank 1 only."""
    HK_FT = 1

    def __init__(self, rank):
        self.rank = rank

    def part_units(self, dev):
        return {0: (dev.ny, dev.by), 1: (dev.n, 1), 2: (dev.rows, 1)}[dev.bench]

    def new_control(self, device):
        return torch.zeros(24, dtype=torch.int32, device=device)

    def run_part(self, dev, b, e, variant, ranges, cb):
        if dev.bench == 0:
            y = torch.arange(b, e, dtype=torch.float32)[:, None]
            x = torch.arange(dev.nx, dtype=torch.float32)[None, :]
            dev.grid[b:e] = 1000 * y + x
        elif dev.bench == 1:
            v = torch.arange(b, e, dtype=torch.float32)
            dev.qr[b:e], dev.qi[b:e] = v * 0.5, -v
        else:
            dev.hist.zero_()
            for r in range(b, e):
                dev.hist[r % dev.hist.shape[0], r % dev.hist.shape[1]] += r + 1
        if self.rank == 1:
            cb[0] = 2


class _Dev:
    def __init__(self, bench):
        self.bench = bench
        self.nx, self.ny, self.by = 8, 64, 16
        self.n, self.rows = 37, 23
        self.grid = torch.full((self.ny, self.nx), float("nan"))
        self.qr, self.qi = torch.full((self.n,), float("nan")), torch.full((self.n,), float("nan"))
        self.hist = torch.zeros((3, 5), dtype=torch.int64)

    def output(self):
        return {0: self.grid, 1: (self.qr, self.qi), 2: self.hist}[self.bench]


def _expected(bench):
    d = _Dev(bench)
    _FakeHK(0).run_part(d, 0, _FakeHK(0).part_units(d)[0], 1, None, torch.zeros(24, dtype=torch.int32))
    return d.output()


def _single_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    res = []
    for bench in range(3):
        d = _Dev(bench)
        out, alarm, fail = par.run_single_sharded(_FakeHK(rank), d, None, rank, world)
        outs = [out] if bench != 1 else list(out)
        res.append(([o.clone() for o in outs], alarm, fail))
    if rank == 0:
        q.put(res)
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world3_single_run_sharding_assembles_the_whole_output():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_single_worker, args=(r, 3, port, q)) for r in range(3)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for bench in range(3):
        outs, alarm, fail = res[bench]
        exp = _expected(bench)
        exp = [exp] if bench != 1 else list(exp)
        for o, e in zip(outs, exp):
            assert torch.equal(o, e), bench
        assert alarm == 2 and fail == 0
