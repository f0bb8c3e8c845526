"""A short campaign slice per benchmark (for ncu -k regex:fi_kernel)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as W
from paper_conf_ipps_yimpski11_b200 import hauberk as hk
dev = torch.device("cuda", 0)
which = sys.argv[1:] or ["mriq", "tpacf"]
for name in which:
    b = {"cp": 0, "mriq": 1, "tpacf": 2}[name]
    p = [W.cp_config1, W.mriq_config2, W.tpacf_config3][b]()
    d = [hk.CPDevice, hk.MRIQDevice, hk.TPACFDevice][b].from_problem(p, dev)
    R = hk.profile_ranges(d)
    devs = [None, None, None]; rng = [None, None, None]
    devs[b] = d; rng[b] = R
    counts = torch.zeros((3, 5), dtype=torch.int64, device=dev)
    with hk.CampaignSession(b, devs, rng, 0x4841554245524B05) as S:
        S.run(0, 512, counts)
        torch.cuda.synchronize()
    print(name, counts[b].tolist())
