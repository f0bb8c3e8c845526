"""Sweep CP-L (config 4) launch shapes: BASE / FT device time per shape (CUDA events via the library hook)."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as W
from paper_conf_ipps_yimpski11_b200 import hauberk as hk
dev = torch.device("cuda", 0)
flush = torch.empty(128 * 1024 * 1024, dtype=torch.float32, device=dev)
for (bx, by, u) in [(16, 16, 8), (32, 4, 8), (32, 8, 4), (32, 4, 4), (16, 16, 4), (32, 8, 2), (64, 4, 2), (32, 2, 8), (64, 2, 4), (16, 8, 8), (32, 4, 2), (128, 2, 2)]:
    p = W.cp_config4(bx=bx, by=by, unroll=u)
    d = hk.CPDevice.from_problem(p, dev)
    R = hk.profile_ranges(d)
    cb = hk.new_control(dev)
    hk.timing_enable(True)
    t = {0: [], 1: []}
    for rep in range(8):
        for v in (0, 1):
            flush.zero_()
            hk.run(d, v, R, cb)
            torch.cuda.synchronize()
            ms, n, w = hk.timing_read(0, 0)
            if rep >= 2:
                t[v].append(ms)
    hk.timing_enable(False)
    b, f = statistics.median(t[0]), statistics.median(t[1])
    mufu = w / (f * 1e-3) / (148 * 16 * 1.965e9)
    print(f"bx={bx:3d} by={by:2d} U={u}  base {b:.3f} ms  ft {f:.3f} ms  overhead {100*(f/b-1):5.2f}%  ft-xu-frac {mufu:.3f}", flush=True)
