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
    probs = [W.cp_small(), W.mriq_problem(4, 23, n_vox=60), W.tpacf_small(n=60, n_rand=1, chunk=16)]
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
    probs = [W.cp_small(), W.mriq_problem(4, 23, n_vox=60), W.tpacf_small(n=60, n_rand=1, chunk=16)]
    R = [O.profile_ranges(b, probs[b]) for b in range(3)]
    c, _ = O.campaign(-1, probs, R, seed=777, first=0, count=total, mode=1, records=False)
    counts, same, differ, mx = res
    assert np.array_equal(np.array(counts), c)
    assert same is True and differ is False and mx == 2.0
