"""HAUBERK error recovery (PAPER §VI) on top of the C ABI.

* Re-execution diagnosis of an alarm (Fig. 11): re-run the protected kernel; an
  identical output with the same alarm is a FALSE ALARM (ranges are extended to the recorded
  outliers, A11 L1309-1313, and stored as part of the on-line learning); no alarm on the re-run is
  a TRANSIENT fault (the re-run's output is taken); a different output with an alarm points to a
  PERSISTENT / intermittent fault (the paper then runs a BIST and migrates — out of scope here).
* alpha controller (L2066-2081): a detector's ranges are loosened by x10 when its false-positive
  ratio exceeds 10 % and tightened by /10 below 5 % (alpha >= 1).
* Multi-set training (L2031-2036, L2654-2662): PROFILE samples of several training inputs are
  concatenated before the threshold search (hauberk_profile_search).
* The synthetic false-positive study of Fig. 16 (L2652-2662, L2780-2820): train on k of 50
  synthetic datasets, test fault-free runs on 2 held-out ones, repeat.

Host orchestration only; every kernel runs through hauberk_run_* / hauberk_profile_*.
"""
from __future__ import annotations

import struct
from dataclasses import dataclass, field

import numpy as np
import torch

from . import hauberk as hk

OK, FALSE_ALARM, TRANSIENT, PERSISTENT, FAILED = "ok", "false_alarm", "transient", "persistent", "failed"


def ord_to_float(o: int) -> float:
    """Inverse of the R8 ordinal: o >= 0 -> bits o; o < 0 -> sign bit | -o."""
    bits = o if o >= 0 else (0x80000000 | (-o))
    return struct.unpack("<f", struct.pack("<I", bits & 0xFFFFFFFF))[0]


def extend_ranges(R: hk.Ranges, d: int, values) -> hk.Ranges:
    """A11 (L1309-1313; DESIGN R24) through hauberk_extend_ranges: make detector d's ranges include
    every value (each joins the range of its correlation class at the detector's threshold)."""
    hk.extend_ranges(R.det[d], values)
    return R


def outliers_of(cb: hk.Control, d: int):
    """The recorded outlier interval of detector d (hauberk_outliers; empty if none)."""
    return hk.outliers(cb, d)


@dataclass
class AlphaController:
    """alpha per detector set (hauberk_alpha_update): x10 above 10 % false positives, /10 below 5 %,
    never below 1 (L2066-2077)."""
    alpha: float = 1.0
    hi: float = 0.10
    lo: float = 0.05
    history: list = field(default_factory=list)

    def update(self, fp_ratio: float) -> float:
        self.alpha = hk.alpha_update(self.alpha, fp_ratio, self.hi, self.lo)
        self.history.append((fp_ratio, self.alpha))
        return self.alpha


def _outputs(dev):
    o = dev.output()
    return tuple(t.clone() for t in o) if isinstance(o, tuple) else (o.clone(),)


def _identical(a, b) -> bool:
    return all(torch.equal(x.view(torch.int32) if x.dtype == torch.float32 else x,
                           y.view(torch.int32) if y.dtype == torch.float32 else y) for x, y in zip(a, b))


@dataclass
class Diagnosis:
    verdict: str
    alarm: int
    rerun_alarm: int | None
    extended: bool
    outputs: tuple


def protected_run(dev, ranges: hk.Ranges, variant: int = hk.HK_FT, learn: bool = True) -> Diagnosis:
    """Run the protected kernel; on an alarm re-execute and diagnose (Fig. 11, hauberk_diagnose)."""
    cb = hk.new_control(dev.output()[0].device if isinstance(dev.output(), tuple) else dev.output().device)
    hk.run(dev, variant, ranges, cb)
    torch.cuda.current_stream().synchronize()
    c1 = hk.read_control(cb)
    out1 = _outputs(dev)
    if c1.alarm == 0 and c1.fail == 0:
        return Diagnosis(OK, 0, None, False, out1)
    if c1.fail:
        return Diagnosis(FAILED, c1.alarm, None, False, out1)
    hk.run(dev, variant, ranges, cb)
    torch.cuda.current_stream().synchronize()
    c2 = hk.read_control(cb)
    out2 = _outputs(dev)
    verdict = hk.diagnose(c1.alarm, c1.fail, c2.alarm, c2.fail, _identical(out1, out2))
    extended = False
    if verdict == FALSE_ALARM and learn and (c1.alarm & hk_alarm_range()):
        for d in range(ranges.n_det):
            vals = outliers_of(c1, d)
            if vals:
                extend_ranges(ranges, d, vals)
                extended = True
    keep = out1 if verdict == FALSE_ALARM else out2
    return Diagnosis(verdict, c1.alarm, c2.alarm, extended, keep)


def hk_alarm_range() -> int:
    return 4


# ------------------------------------------------------------------------------------------------
# multi-set training and the Fig. 16 false-positive study
# ------------------------------------------------------------------------------------------------
def train_ranges(devs, maxvar: int = 1, t0_exp10: int = -5, alpha: float = 1.0) -> hk.Ranges:
    """Ranges from the concatenated PROFILE samples of several training inputs."""
    per = [hk.profile_samples(d, maxvar).cpu().numpy() for d in devs]
    R = hk.Ranges()
    R.n_det = maxvar
    R.alpha = alpha
    for det in range(maxvar):
        s = np.concatenate([p[det] for p in per])
        s = s[np.isfinite(s)]  # zero-trip threads keep NaN (R19)
        R.det[det] = hk.profile_search(s, t0_exp10)
    return R


def false_positive_study(make_dev, n_sets: int = 52, n_test: int = 2, train_sizes=(1, 2, 5, 10, 20, 50),
                         repeats: int = 10, seed: int = 2011, alpha: float = 1.0, maxvar: int = 1):
    """Fig. 16 analogue: `make_dev(i)` builds the device input of synthetic dataset i.  For each
    repeat, n_test sets are held out; ranges trained on the first k of the rest; the false-positive
    ratio = fraction of fault-free test runs that alarm.  Returns {k: mean FP ratio}."""
    devs = [make_dev(i) for i in range(n_sets)]
    samples = [hk.profile_samples(d, maxvar).cpu().numpy() for d in devs]
    rng = np.random.default_rng(seed)
    fp = {k: [] for k in train_sizes}
    for _ in range(repeats):
        order = rng.permutation(n_sets)
        test, train = order[:n_test], order[n_test:]
        for k in train_sizes:
            R = hk.Ranges()
            R.n_det = maxvar
            R.alpha = alpha
            for det in range(maxvar):
                s = np.concatenate([samples[i][det] for i in train[:k]])
                R.det[det] = hk.profile_search(s[np.isfinite(s)])
            alarms = 0
            for i in test:
                cb = hk.new_control(samples_device(devs[i]))
                hk.run(devs[i], hk.HK_FT, R, cb)
                torch.cuda.current_stream().synchronize()
                alarms += hk.read_control(cb).alarm != 0
            fp[k].append(alarms / len(test))
    return {k: float(np.mean(v)) for k, v in fp.items()}


def samples_device(dev):
    o = dev.output()
    return (o[0] if isinstance(o, tuple) else o).device
