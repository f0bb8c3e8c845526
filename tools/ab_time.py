"""A/B device timing of the hot kernels for one library build (HAUBERK_LIB selects the .so).

  HAUBERK_LIB=_ab/x/libhauberk.so python tools/ab_time.py [--fi N] [cp mriq tpacf]

Prints, per benchmark at its BASELINE config (cfg4 CP-L, cfg2 MRI-Q, cfg3 TPACF), the median
BASE / FT kernel time (CUDA events on the launching stream, library timing hook, L2 flushed
before every launch) and, with --fi N, the device time per replica of an N-injection
replica-mode campaign on that benchmark's campaign shape (cfg1 / cfg2 / cfg3).
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_yimpski11_b200 import hauberk as hk  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("which", nargs="*", default=["cp", "mriq", "tpacf"])
ap.add_argument("--fi", type=int, default=0)
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--cp", default="16,16,8", help="bx,by,unroll for cfg4")
a = ap.parse_args()
dev = torch.device("cuda", 0)
flush = torch.empty(128 * 1024 * 1024, dtype=torch.float32, device=dev)
tag = os.environ.get("HAUBERK_LIB", "default")
XU = 148 * 16 * 1.965e9
for name in a.which:
    if name == "cp":
        bx, by, u = (int(x) for x in a.cp.split(","))
        d = hk.CPDevice.from_problem(W.cp_config4(bx=bx, by=by, unroll=u), dev)
        ops = 1.0
    elif name == "mriq":
        d = hk.MRIQDevice.from_problem(W.mriq_config2(), dev)
        ops = 2.0
    else:
        d = hk.TPACFDevice.from_problem(W.tpacf_config3(), dev)
        ops = 0.0
    R = hk.profile_ranges(d)
    cb = hk.new_control(dev)
    hk.timing_enable(True)
    t = {0: [], 1: []}
    w = 0
    for rep in range(a.reps + 2):
        for v in (hk.HK_BASE, hk.HK_FT):
            flush.zero_()
            hk.run(d, v, R, cb)
            torch.cuda.synchronize()
            ms, n, w = hk.timing_read(d.bench, 0)
            if rep >= 2:
                t[v].append(ms)
    hk.timing_enable(False)
    assert hk.read_control(cb).alarm == 0
    b, f = statistics.median(t[0]), statistics.median(t[1])
    xu = f" xu-frac {w * ops / (f * 1e-3) / XU:.3f}" if ops else f" Gpairs/s {w / (f * 1e-3) / 1e9:.0f}"
    print(f"[{tag}] {name:5s} base {b * 1e3:9.2f} us  ft {f * 1e3:9.2f} us  overhead {100 * (f / b - 1):6.2f}%{xu}", flush=True)
    if a.fi:
        probs = {"cp": W.cp_config1(), "mriq": W.mriq_config2(), "tpacf": W.tpacf_config3()}
        b_i = {"cp": 0, "mriq": 1, "tpacf": 2}[name]
        mk = [hk.CPDevice, hk.MRIQDevice, hk.TPACFDevice][b_i]
        dd = mk.from_problem(probs[name], dev)
        RR = hk.profile_ranges(dd)
        counts = torch.zeros((3, 5), dtype=torch.int64, device=dev)
        dl, rl = [None] * 3, [None] * 3
        dl[b_i], rl[b_i] = dd, RR
        with hk.CampaignSession(b_i, dl, rl, 0x4841554245524B05) as s:
            s.run(10_000_000, min(a.fi, 500), counts)  # warm-up
            torch.cuda.synchronize()
            hk.timing_enable(True)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            s.run(0, a.fi, counts)
            e1.record()
            torch.cuda.synchronize()
            ms, nl, work = hk.timing_read(b_i, 1)
            hk.timing_enable(False)
        print(f"[{tag}] {name:5s} FI: {a.fi} inj, step {e0.elapsed_time(e1):8.2f} ms, fi kernels {ms:8.2f} ms "
              f"({nl} launches) = {1e3 * ms / a.fi:7.2f} us/replica, {a.fi / (e0.elapsed_time(e1) * 1e-3):9.0f} inj/s", flush=True)
