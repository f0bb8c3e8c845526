"""Per-CTA trace of one TPACF single run (a build with -DHK_TP_SR_TRACE, via HAUBERK_LIB):
SM, start/end (globaltimer ns) and piece of every CTA -> per-SM busy time and the CTA spread."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_yimpski11_b200 import hauberk as hk  # noqa: E402

dev = torch.device("cuda", 0)
d = hk.TPACFDevice.from_problem(W.tpacf_config3(), dev)
R = hk.profile_ranges(d)
cb = hk.new_control(dev)
v = int(sys.argv[1]) if len(sys.argv) > 1 else hk.HK_FT
for _ in range(5):
    hk.run(d, v, R, cb)
torch.cuda.synchronize()
buf = np.zeros((4096, 4), dtype=np.uint64)
assert hk.lib().hk_debug_trace(buf.ctypes.data_as(ctypes.c_void_p)) == 0
n = int((buf[:, 2] > 0).sum())
b = buf[:n].astype(np.int64)
t0 = b[:, 1].min()
st, en = (b[:, 1] - t0) / 1e3, (b[:, 2] - t0) / 1e3
dur = en - st
print(f"CTAs {n}; kernel span {en.max():.1f} us; CTA duration min/med/max {dur.min():.1f}/{np.median(dur):.1f}/{dur.max():.1f} us; "
      f"start spread {st.max():.1f} us")
sm = b[:, 0]
per = np.bincount(sm, minlength=148)
print("CTAs per SM: min", per.min(), "max", per.max(), "hist", np.bincount(per))
busy = np.array([en[sm == k].max() if (sm == k).any() else 0 for k in range(148)])
print(f"SM end time min/med/max {busy.min():.1f}/{np.median(busy):.1f}/{busy.max():.1f} us")
row = b[:, 3] >> 32
for q in (0.0, 0.5, 0.9, 1.0):
    i = np.argsort(dur)[min(n - 1, int(q * (n - 1)))]
    print(f"  q{q:.1f}: dur {dur[i]:.1f} us row {row[i]} piece {(b[i, 3] >> 16) & 0xffff}/{b[i, 3] & 0xffff} sm {sm[i]} start {st[i]:.1f}")
slow = np.argsort(-dur)[:10]
print("slowest rows:", row[slow].tolist(), "pieces:", ((b[slow, 3] >> 16) & 0xffff).tolist(), [round(x, 1) for x in dur[slow]])
print("mean dur by h:", {int(h): round(float(dur[(row // 8) == h].mean()), 1) for h in range(9)})
rank = np.arange(n) // 148
print("mean dur by launch rank (blockIdx // 148):", {int(k): round(float(dur[rank == k].mean()), 1) for k in range(int(rank.max()) + 1)})
