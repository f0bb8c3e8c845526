"""MRI-Q single-run kernel: XU efficiency per resident warp count (BASE, library timing hook).

  HAUBERK_LIB=_ab/x/libhauberk.so python tools/mq_warp_eff.py [n_vox ...]

For each voxel count (config-2 k-space, 3,072 samples) prints the median kernel time and the
fraction of the per-SM-sub-partition MUFU bound ceil(warps / 592) * numK * 16 cycles at 1,965 MHz
(a warp's MUFU.SIN + MUFU.COS take 16 issue cycles of the sub-partition's XU), i.e. how well the
resident warps keep the XU busy independent of wave quantisation.
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_yimpski11_b200 import hauberk as hk  # noqa: E402

dev = torch.device("cuda", 0)
flush = torch.empty(128 * 1024 * 1024, dtype=torch.float32, device=dev)
counts = [int(a) for a in sys.argv[1:]] or [148 * 4 * 32, 2 * 148 * 4 * 32, 32768]
for nv in counts:
    d = hk.MRIQDevice.from_problem(W.mriq_problem(32, 3072, n_vox=nv), dev)
    R = hk.profile_ranges(d)
    cb = hk.new_control(dev)
    hk.timing_enable(True)
    ks = []
    for r in range(12):
        flush.zero_()
        hk.run(d, hk.HK_BASE, R, cb)
        torch.cuda.synchronize()
        ms, _, _ = hk.timing_read(d.bench, 0)
        if r >= 2:
            ks.append(ms)
    hk.timing_enable(False)
    km = statistics.median(ks)
    warps = (nv + 31) // 32
    bound_us = -(-warps // 592) * 3072 * 16 / 1965.0
    print(f"{os.environ.get('HAUBERK_LIB', 'default')} n_vox {nv:6d} warps {warps:5d} kernel {km * 1e3:7.2f} us "
          f"bound {bound_us:6.2f} us  eff {bound_us / (km * 1e3):.3f}", flush=True)
