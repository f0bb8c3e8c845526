"""One FT launch of each benchmark kernel at its BASELINE config (for ncu -k regex:...)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as W
from paper_conf_ipps_yimpski11_b200 import hauberk as hk
dev = torch.device("cuda", 0)
which = [a for a in sys.argv[1:] if not a.startswith("--v=")] or ["cp", "mriq", "tpacf"]
variants = [int(a[4:]) for a in sys.argv[1:] if a.startswith("--v=")]  # e.g. --v=1 --v=3 (default BASE, FT)
for name in which:
    if name == "cp":
        d = hk.CPDevice.from_problem(W.cp_config4(bx=16, by=16, unroll=8), dev)
    elif name == "mriq":
        d = hk.MRIQDevice.from_problem(W.mriq_config2(), dev)
    else:
        d = hk.TPACFDevice.from_problem(W.tpacf_config3(), dev)
    R = hk.profile_ranges(d)
    cb = hk.new_control(dev)
    for v in (variants or (hk.HK_BASE, hk.HK_FT)):
        hk.run(d, v, R, cb)
    torch.cuda.synchronize()
    print(name, "ok")
