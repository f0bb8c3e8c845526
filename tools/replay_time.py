"""Time the replay-mode (campaign mode 1) config-5 campaign: N injections, repeated, CUDA events."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_yimpski11_b200 import hauberk as hk  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
dev = torch.device("cuda", 0)
probs = [W.cp_config1(), W.mriq_config2(), W.tpacf_config3()]
devs = [hk.CPDevice.from_problem(probs[0], dev), hk.MRIQDevice.from_problem(probs[1], dev),
        hk.TPACFDevice.from_problem(probs[2], dev)]
ranges = [hk.profile_ranges(d) for d in devs]
with hk.CampaignSession(-1, devs, ranges, 0x4841554245524B05, mode=1) as sr:
    for rep in range(4):
        c = torch.zeros((3, 5), dtype=torch.int64, device=dev)
        torch.cuda.synchronize()
        hk.timing_enable(True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        sr.run(0, n, c)
        e1.record()
        torch.cuda.synchronize()
        t = [hk.timing_read(b, 1) for b in range(3)]
        hk.timing_enable(False)
        print(f"rep {rep}: {n} replays in {e0.elapsed_time(e1):.2f} ms; per-bench timed kernels (ms, launches): "
              f"{[(round(x[0], 3), x[1]) for x in t]}; counts {c.sum().item()}", flush=True)
