"""Device time per single run (hauberk_run_*) of the benchmark kernels at their BASELINE configs.

  python tools/single_time.py [cp|mriq|tpacf ...] [--reps 30]

Per variant (BASE, FT_NL, FT_L, FT): the median kernel-only time (library CUDA events around the
main kernel) and the median per-call time of 20 back-to-back calls (table / pre-pass kernels and
memsets included), L2 flushed before each measurement; algorithmic op rate vs the pipe peak.
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
ap.add_argument("which", nargs="*", default=["mriq", "tpacf"])
ap.add_argument("--reps", type=int, default=30)
a = ap.parse_args()
dev = torch.device("cuda", 0)
flush = torch.empty(128 * 1024 * 1024, dtype=torch.float32, device=dev)
OPS = {"cp": (1.0, 148 * 16 * 1965e6), "mriq": (2.0, 148 * 16 * 1965e6), "tpacf": (11.0, 148 * 128 * 1965e6)}
for name in a.which:
    d = {"cp": lambda: hk.CPDevice.from_problem(W.cp_config4(bx=16, by=16, unroll=8), dev),
         "mriq": lambda: hk.MRIQDevice.from_problem(W.mriq_config2(), dev),
         "tpacf": lambda: hk.TPACFDevice.from_problem(W.tpacf_config3(), dev)}[name]()
    R = hk.profile_ranges(d)
    cb = hk.new_control(dev)
    for v, vn in ((hk.HK_BASE, "BASE"), (hk.HK_FT_NL, "FT_NL"), (hk.HK_FT_L, "FT_L"), (hk.HK_FT, "FT")):
        hk.timing_enable(True)
        ks, work = [], 0.0
        for r in range(a.reps):
            flush.zero_()
            hk.run(d, v, R, cb)
            torch.cuda.synchronize()
            ms, n, w = hk.timing_read(d.bench, 0)
            if r >= 2:
                ks.append(ms)
                work = w
        hk.timing_enable(False)
        calls = []
        for r in range(8):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20):
                hk.run(d, v, R, cb)
            e1.record()
            torch.cuda.synchronize()
            if r >= 1:
                calls.append(e0.elapsed_time(e1) / 20)
        km, cm = statistics.median(ks), statistics.median(calls)
        ops, peak = OPS[name]
        print(f"{name:6s} {vn:6s} kernel {km * 1e3:8.2f} us  per-call {cm * 1e3:8.2f} us  frac {work * ops / (km * 1e-3) / peak:.4f}  "
              f"alarm {hk.read_control(cb).alarm}", flush=True)
