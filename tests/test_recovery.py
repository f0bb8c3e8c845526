"""Recovery (PAPER §VI; NEXT f2): range extension from outliers (A11), the alpha controller,
multi-set training through hauberk_profile_search (parity with the oracle's threshold walk), and
on the GPU the re-execution diagnosis of Fig. 11 and a small Fig. 16 false-positive study."""
import struct

import numpy as np
import pytest
import torch

import oracle as O
import workloads as W
from paper_conf_ipps_yimpski11_b200 import hauberk as hk
from paper_conf_ipps_yimpski11_b200 import recovery as rc


def _rs(lo_hi, t):
    R = hk.Ranges()
    R.n_det = 1
    R.alpha = 1.0
    R.det[0].n = len(lo_hi)
    R.det[0].t_exp10 = t
    for r, (a, b) in enumerate(lo_hi):
        R.det[0].lo[r], R.det[0].hi[r] = a, b
    return R


def test_ord_to_float_inverts_the_oracle_ordinal():
    L = O.lib()
    for v in [0.0, 1.0, -1.0, 3.5e-12, -7.25e20, 1e-45, -1e-45]:
        v = float(np.float32(v))
        assert rc.ord_to_float(L.ora_ord(v)) == v


def test_extend_ranges_widens_the_class_of_the_outlier_and_adds_missing_classes():
    R = _rs([(-3.0, -1.0), (2.0, 5.0)], -5)
    rc.extend_ranges(R, 0, [7.0, -0.5])           # pos range grows to 7; neg range grows to -0.5
    assert [(R.det[0].lo[r], R.det[0].hi[r]) for r in range(R.det[0].n)] == [(-3.0, -0.5), (2.0, 7.0)]
    rc.extend_ranges(R, 0, [1e-7])                # |v| <= 1e-5: new zero-class range between them
    got = [(R.det[0].lo[r], R.det[0].hi[r]) for r in range(R.det[0].n)]
    assert got == [(-3.0, -0.5), (float(np.float32(1e-7)),) * 2, (2.0, 7.0)]
    rc.extend_ranges(R, 0, [float("nan")])        # NaN never widens a range
    assert R.det[0].n == 3


def test_alpha_controller_follows_the_10_and_5_percent_rule():
    a = rc.AlphaController()
    assert a.update(0.3) == 10.0       # > 10 %: loosen
    assert a.update(0.2) == 100.0
    assert a.update(0.07) == 100.0     # between 5 % and 10 %: keep
    assert a.update(0.0) == 10.0       # < 5 %: tighten
    assert a.update(0.01) == 1.0
    assert a.update(0.0) == 1.0        # never below 1 (L2073-2077)


@pytest.mark.parametrize("seed", range(6))
def test_profile_search_matches_the_oracle_walk(seed):
    rng = np.random.default_rng(seed)
    mag = 10.0 ** rng.uniform(-7, 2)
    s = np.concatenate([rng.uniform(1, 9, 300) * mag, -rng.uniform(1, 3, 100) * mag,
                        rng.uniform(-1, 1, 40) * mag * 10.0 ** rng.uniform(-6, -1)]).astype(np.float32)
    g = hk.profile_search(s)
    o = O.profile_samples(s)
    assert g.t_exp10 == o.t_exp10 and g.n == o.n
    assert [(g.lo[r], g.hi[r]) for r in range(g.n)] == [(o.lo[r], o.hi[r]) for r in range(o.n)]
    with pytest.raises(hk.HauberkError):
        hk.profile_search(np.array([1.0, np.inf], dtype=np.float32))


# ---------------------------------------------------------------------------------------- GPU
@pytest.mark.gpu
def test_reexecution_diagnosis_false_alarm_then_learned():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    p = W.cp_small()
    d = hk.CPDevice.from_problem(p, "cuda")
    R = hk.profile_ranges(d)
    assert rc.protected_run(d, R).verdict == rc.OK
    # shrink the positive range so fault-free threads fall outside: a false alarm by construction
    r = R.det[0].n - 1
    mid = 0.5 * (R.det[0].lo[r] + R.det[0].hi[r])
    R.det[0].hi[r] = float(np.float32(mid))
    dg = rc.protected_run(d, R)
    assert dg.verdict == rc.FALSE_ALARM and dg.alarm & 4 and dg.extended
    # the outliers were folded back into the ranges (on-line learning, L2031-2036)
    assert rc.protected_run(d, R).verdict == rc.OK


@pytest.mark.gpu
def test_multiset_training_and_false_positive_study():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    make = lambda i: hk.MRIQDevice.from_problem(W.mriq_problem(8, 96, seed=1000 + i), "cuda")
    devs = [make(i) for i in range(3)]
    R = rc.train_ranges(devs)
    for d in devs:
        assert rc.protected_run(d, R, learn=False).verdict == rc.OK
    fp = rc.false_positive_study(make, n_sets=12, n_test=2, train_sizes=(1, 5, 10), repeats=3)
    assert fp[10] <= fp[1]
    assert all(0.0 <= v <= 1.0 for v in fp.values())
