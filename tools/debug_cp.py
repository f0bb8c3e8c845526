import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as W
from paper_conf_ipps_yimpski11_b200 import hauberk as hk
p = W.cp_problem(37, 64, 32, seed=7, bx=16, by=8, unroll=int(sys.argv[1]) if len(sys.argv) > 1 else 1)
d = hk.CPDevice.from_problem(p, "cuda")
R = hk.profile_ranges(d, maxvar=p.unroll)
print("ranges", R.as_list())
for v in (hk.HK_BASE, hk.HK_FT_NL, hk.HK_FT_L, hk.HK_FT):
    cb = hk.new_control("cuda")
    hk.run(d, v, R, cb)
    torch.cuda.synchronize()
    c = hk.read_control(cb)
    print(v, hex(c.alarm), c.fail, c.n_alarm_warps, hex(c.first_thread), list(c.outlier_min_ord)[:2], cb.cpu().numpy()[:8])
