"""Mixed-campaign step timing (config-5 mix, replica mode) for one library build.

  HAUBERK_LIB=_ab/x/libhauberk.so HK_CONCURRENT=1 python tools/conc_time.py [--n 3000] [--steps 5]

Prints the device time per step of N injections (CUDA events on the campaign stream, L2 not
flushed) and the outcome counters, so builds / stream modes can be compared for speed and for
identical classification.
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
ap.add_argument("--n", type=int, default=3000)
ap.add_argument("--steps", type=int, default=5)
ap.add_argument("--batch", type=int, default=0)
ap.add_argument("--timing", action="store_true", help="also print the per-class kernel device time per step")
a = ap.parse_args()
dev = torch.device("cuda", 0)
devs = [hk.CPDevice.from_problem(W.cp_config1(), dev), hk.MRIQDevice.from_problem(W.mriq_config2(), dev),
        hk.TPACFDevice.from_problem(W.tpacf_config3(), dev)]
ranges = [hk.profile_ranges(d) for d in devs]
counts = torch.zeros((3, 5), dtype=torch.int64, device=dev)
tag = (f"{os.environ.get('HAUBERK_LIB', 'default')} conc={os.environ.get('HK_CONCURRENT', '-')} "
       f"prio={os.environ.get('HK_CONC_PRIO', '-')} batch={a.batch}")
with hk.CampaignSession(-1, devs, ranges, 0x4841554245524B05, batch=a.batch) as s:
    s.run(50_000_000, a.n, counts)  # warm-up (other indices)
    torch.cuda.synchronize()
    counts.zero_()
    ts = []
    hk.timing_enable(a.timing)
    for k in range(a.steps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        s.run(k * a.n, a.n, counts)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
if a.timing:
    for b in range(3):
        for cls in (1, 3):
            ms, n, w = hk.timing_read(b, cls)
            if n:
                print(f"  bench {b} cls {cls}: {ms / a.steps:8.2f} ms/step over {n / a.steps:.1f} launches/step "
                      f"({ms / n:.3f} ms per launch, work {w / a.steps:.3g}/step)")
    hk.timing_enable(False)
med = statistics.median(ts)
print(f"[{tag}] step {med:8.2f} ms (min {min(ts):.2f} max {max(ts):.2f}) -> {a.n / med * 1e3:9.0f} inj/s  "
      f"counts {counts.cpu().tolist()}", flush=True)
