"""Small end-to-end pass for compute-sanitizer (memcheck / racecheck / synccheck): every benchmark's
BASE/FT/FT_NL/FT_L/PROFILE runs plus replica and replay campaigns (the FI kernels model crashes by
suppressing the access, so no real out-of-bounds access may appear)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as W
from paper_conf_ipps_yimpski11_b200 import hauberk as hk
dev = torch.device("cuda", 0)
probs = [W.cp_small(), W.mriq_small(), W.tpacf_small(n=300, n_rand=2)]
devs = [hk.CPDevice.from_problem(probs[0], dev), hk.MRIQDevice.from_problem(probs[1], dev), hk.TPACFDevice.from_problem(probs[2], dev)]
R = [hk.profile_ranges(d) for d in devs]
for b, d in enumerate(devs):
    cb = hk.new_control(dev)
    for v in (hk.HK_BASE, hk.HK_FT, hk.HK_FT_NL, hk.HK_FT_L):
        hk.run(d, v, R[b], cb)
torch.cuda.synchronize()
counts = torch.zeros((3, 5), dtype=torch.int64, device=dev)
for mode in (0, 1):
    hk.inject_campaign(-1, devs, R, 0xC0FFEE, 0, 240 if mode == 0 else 3000, counts, mode=mode)
torch.cuda.synchronize()
print("sanitize smoke ok", counts.cpu().tolist())
