"""One fused MRI-Q + TPACF replica launch of a mixed config-5 campaign slice (for ncu -k regex:mix_fi_kernel).

  python tools/profile_mix.py [n_injections]   (default 600: 200 each of CP-s / MRI-Q / TPACF)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_yimpski11_b200 import hauberk as hk  # noqa: E402

dev = torch.device("cuda", 0)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 600
devs = [hk.CPDevice.from_problem(W.cp_config1(), dev), hk.MRIQDevice.from_problem(W.mriq_config2(), dev),
        hk.TPACFDevice.from_problem(W.tpacf_config3(), dev)]
ranges = [hk.profile_ranges(d) for d in devs]
counts = torch.zeros((3, 5), dtype=torch.int64, device=dev)
with hk.CampaignSession(-1, devs, ranges, 0x4841554245524B05) as S:
    S.run(0, n, counts)
    torch.cuda.synchronize()
print("mixed", counts.tolist())
