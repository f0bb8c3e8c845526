"""Pins of the oracle's non-benchmark machinery against things other than itself
(-m "not gpu"): RNG known answers, the R8 ordinal, the profiler walk on hand-reasoned cases and
against exhaustive search, the output-correctness rules, the outcome
classes (L2377-2387) and the injection decode (brute-force enumeration, uniformity, sharding)."""
import ctypes as C
import math
import os
import struct

import numpy as np
import pytest

import oracle as O
import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _f32(x):
    return float(np.float32(x))


# ---------------------------------------------------------------- R15 SplitMix64 known answers
def test_splitmix64_known_answers():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "splitmix64.txt")) if l.strip() and not l.startswith("#")]
    L = O.lib()
    for r in rows:
        seed = int(r[0], 0)
        for m, v in enumerate(r[1:]):
            assert L.ora_splitmix(seed, m) == int(v, 0)
    # the numpy input generator implements the same stream independently
    for r in rows:
        seed = int(r[0], 0)
        got = W.splitmix64(seed, len(r) - 1)
        assert [int(x) for x in got] == [int(v, 0) for v in r[1:]]


def test_bounded_draw_is_floor_of_scaled_fraction():
    L = O.lib()
    for r in [0, 1, 2**63, 2**64 - 1, 0x123456789ABCDEF0]:
        for m in [1, 2, 3, 7, 54, 10**6, 2**40 + 3]:
            assert L.ora_bounded(r, m) == (r * m) >> 64
            assert 0 <= L.ora_bounded(r, m) < m


# ---------------------------------------------------------------- R8 ordinal ("value space")
def test_ordinal_counts_encodings():
    L = O.lib()
    assert L.ora_ord(0.0) == 0 and L.ora_ord(-0.0) == 0
    assert L.ora_ord(1.0) == 0x3F800000
    assert L.ora_ord(-1.0) == -0x3F800000
    one_up = np.nextafter(np.float32(1), np.float32(2))
    assert L.ora_ord(float(one_up)) - L.ora_ord(1.0) == 1
    # the smallest positive and negative denormals are 1 encoding away from zero
    d = float(np.array([1], dtype=np.uint32).view(np.float32)[0])
    assert L.ora_ord(d) == 1 and L.ora_ord(-d) == -1


def test_ordinal_is_monotone_and_unit_step():
    L = O.lib()
    rng = np.random.default_rng(1)
    x = np.sort(rng.standard_normal(2000).astype(np.float32) * np.float32(10.0) ** rng.integers(-30, 30, 2000).astype(np.float32))
    o = [L.ora_ord(float(v)) for v in x]
    assert all(a <= b for a, b in zip(o, o[1:]))
    for v in x[:200]:
        nv = np.nextafter(v, np.float32(np.inf))
        if np.isfinite(nv) and not (v == 0):
            assert L.ora_ord(float(nv)) - L.ora_ord(float(v)) == 1


# ---------------------------------------------------------------- profiler (R9)
def test_profiler_threshold_table():
    L = O.lib()
    for k in range(-38, 39):
        assert L.ora_threshold(k) == _f32(float(f"1e{k}"))


def test_profiler_single_positive_cluster_keeps_default_threshold():
    # all samples positive and > 1e-4: every T in a neighbourhood gives one range -> no strict improvement
    s = np.array([0.01, 0.5, 2.0, 0.3], dtype=np.float32)
    r = O.profile_samples(s)
    assert r.t_exp10 == -5 and r.n == 1
    assert (r.lo[0], r.hi[0]) == (_f32(0.01), _f32(2.0))


def test_profiler_hand_case_moves_threshold_down():
    # {-2e-6, 3e-6, 0.01, 2, -0.5}: at T=1e-5 the zero band [-2e-6, 3e-6] straddles 0 and spans ~1.8e9
    # encodings; at T=1e-6 both tiny values join the negative / positive ranges, which is far smaller;
    # T=1e-7 classifies identically (tie) so the walk stops at 1e-6.
    s = np.array([-2e-6, 3e-6, 0.01, 2.0, -0.5], dtype=np.float32)
    r = O.profile_samples(s)
    assert r.t_exp10 == -6
    assert r.n == 2
    assert (r.lo[0], r.hi[0]) == (_f32(-0.5), _f32(-2e-6))
    assert (r.lo[1], r.hi[1]) == (_f32(3e-6), _f32(2.0))
    # value-space sizes counted as encodings (R8): zero band alone at T = 1e-5
    bits = lambda v: struct.unpack("<I", struct.pack("<f", v))[0]
    zero_band = bits(_f32(3e-6)) + (bits(_f32(-2e-6)) & 0x7FFFFFFF) + 1
    assert O.profile_cost(s, -5) == zero_band + 1 + (bits(2.0) - bits(_f32(0.01)) + 1)


def test_profiler_three_points_and_empty_classes():
    s = np.array([-3.0, -2.0, 1e-9, -1e-9, 5.0, 7.0], dtype=np.float32)
    r = O.profile_samples(s)
    # three correlation points survive: negative, near-zero, positive (Fig. 10 motivation, L1479-1487)
    assert r.n == 3
    assert r.lo[0] == -3.0 and r.hi[0] == -2.0
    assert r.lo[2] == 5.0 and r.hi[2] == 7.0
    assert r.lo[1] == _f32(-1e-9) and r.hi[1] == _f32(1e-9)


@pytest.mark.parametrize("seed", range(12))
def test_profiler_walk_ends_in_local_minimum_and_matches_global_on_clustered_data(seed):
    rng = np.random.default_rng(seed)
    mag = 10.0 ** rng.uniform(-8, 3)
    parts = [rng.uniform(1, 10, 50) * mag, -rng.uniform(1, 10, 50) * mag * 0.7]
    if seed % 2:
        parts.append(rng.uniform(-1, 1, 20) * mag * 1e-4)
    s = np.concatenate(parts).astype(np.float32)
    r = O.profile_samples(s)
    k = r.t_exp10
    c = O.profile_cost(s, k)
    if k > -38:
        assert c <= O.profile_cost(s, k - 1)
    if k < 38:
        assert c <= O.profile_cost(s, k + 1)
    costs = [O.profile_cost(s, kk) for kk in range(-38, 39)]
    # splitting a cluster at T can shrink the total (non-unimodal profile); where the cost profile
    # is unimodal along the walk's direction, hill-climbing from T0 must reach the global minimum
    # (the walk stops on plateaus by the paper's rule "repeated if ... smaller than ... previous run")
    assert c == min(costs) or not _strict_path_to_global(costs)


def _strict_path_to_global(costs, k0=-5):
    """True iff costs strictly decrease from k0 to the global minimum nearest to k0."""
    m = min(costs)
    i0 = k0 + 38
    cands = [a for a, v in enumerate(costs) if v == m]
    lo = min(cands, key=lambda a: abs(a - i0))
    step = 1 if lo >= i0 else -1
    path = [costs[a] for a in range(i0, lo + step, step)]
    return all(x > y for x, y in zip(path, path[1:]))


def test_profiler_reaches_global_minimum_on_strict_path():
    # +-{1..9}e-6 straddling zero: T=1e-5 -> one zero band; 1e-6 -> zero band shrinks; 1e-7 -> two tight
    # ranges.  Costs strictly decrease from T0 to the global minimum, so the walk must find it.
    v = np.arange(1, 10) * 1e-6
    s = np.concatenate([v, -v]).astype(np.float32)
    costs = [O.profile_cost(s, kk) for kk in range(-38, 39)]
    assert _strict_path_to_global(costs)
    r = O.profile_samples(s)
    assert r.t_exp10 == -7 and r.n == 2
    assert O.profile_cost(s, r.t_exp10) == min(costs)


def test_profiler_rejects_nan():
    with pytest.raises(FloatingPointError):
        O.profile_samples(np.array([1.0, np.nan], dtype=np.float32))
    # invalid (zero-trip) samples are skipped even if NaN (R19)
    r = O.profile_samples(np.array([1.0, np.nan], dtype=np.float32), valid=np.array([1, 0], dtype=np.uint8))
    assert r.n == 1


# ---------------------------------------------------------------- correctness rules and classes
def test_mriq_rule_truth_table():
    L = O.lib()
    # tolerance Max{1e-4 * Max|GR|, 0.2% |GR_i|}
    g = np.array([1.0, 1000.0, -5.0], dtype=np.float32)
    M = L.ora_max_abs(O._p(g), 3)
    assert M == 1000.0
    def wrong(r):
        r = np.array(r, dtype=np.float32)
        w = C.c_float()
        return L.ora_fp_wrong(O._p(r), O._p(g), 3, M, C.byref(w)), w.value
    assert wrong([1.09, 1000.0, -5.0])[0] == 0          # |err| 0.09 <= 0.1
    assert wrong([1.11, 1000.0, -5.0])[0] == 1          # 0.11 > 0.1
    assert wrong([1.0, 1001.9, -5.0])[0] == 0           # 1.9 <= 2.0 (0.2 %)
    assert wrong([1.0, 1002.1, -5.0])[0] == 1
    assert wrong([np.nan, 1000.0, -5.0])[0] == 1        # R6: NaN is wrong
    assert wrong([np.inf, 1000.0, -5.0])[0] == 1


def test_tpacf_one_percent_rule_truth_table():
    L = O.lib()
    nb, nr = 2, 1
    g = np.zeros((3, nb + 2), dtype=np.int64)
    g[0, 1] = 100; g[0, 2] = 0; g[1, 1] = 50; g[2, 2] = 7
    def wrong(h):
        return L.ora_tpacf_wrong(O._p(h), O._p(g), nr, nb, None)
    h = g.copy(); h[0, 1] = 101
    assert wrong(h) == 0                   # 1 % exactly is not "more than 1 %" (L80-84)
    h = g.copy(); h[0, 1] = 102
    assert wrong(h) == 1
    h = g.copy(); h[0, 2] = 1
    assert wrong(h) == 1                   # zero golden bin: any change is wrong (R3)
    h = g.copy(); h[0, 0] += 5; h[0, 3] += 9
    assert wrong(h) == 0                   # under/overflow bins are not outputs (R4)
    # DR and RR are summed over random sets before the rule (R4)
    out = np.zeros(3 * nb, dtype=np.int64)
    L.ora_tpacf_outputs(O._p(g), nr, nb, O._p(out))
    assert list(out) == [100, 0, 0, 7, 50, 0]


def test_classifier_truth_table():
    L = O.lib()
    for fail in (1, 2):
        for wrong in (0, 1):
            for alarm in (0, 4):
                assert L.ora_classify(wrong, alarm, fail) == O.FAILURE
    assert L.ora_classify(0, 0, 0) == O.MASKED
    assert L.ora_classify(0, 8, 0) == O.DET_MASKED
    assert L.ora_classify(1, 2, 0) == O.DETECTED
    assert L.ora_classify(1, 0, 0) == O.UNDETECTED


def test_paper_outcome_bookkeeping():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "paper_outcomes.txt")) if l.strip() and not l.startswith("#")]
    parts = [float(v) for v in rows[0]]
    assert abs(sum(parts) - 100.0) < 1e-9
    masked, failure, detected, det_masked, undetected = parts
    # coverage = P(detected or masked) = 1 - undetected (L2372-2375, R2)
    assert abs((100.0 - undetected) - (masked + failure + detected + det_masked)) < 1e-9
    esc, cov = float(rows[1][1]), float(rows[1][3])
    assert abs(100.0 - esc - cov) < 1e-9


# ---------------------------------------------------------------- decode (R14)
def _enumerate_instances(bench, p):
    """Brute force: list every (thread, instance) of an ITER site in (thread, inst) order."""
    tr = O.trips(bench, p)
    out = []
    for t, n in enumerate(tr):
        out.extend((t, i) for i in range(int(n)))
    return out


def test_decode_matches_bruteforce_enumeration_tpacf():
    p = W.tpacf_small(n=70, n_rand=1)
    inst = _enumerate_instances(O.TPACF, p)
    L = O.lib()
    seed = 99
    benches, faults = O.decode(O.TPACF, [None, None, p], seed, 0, 400)
    en = [s for s in range(O.nsites(O.TPACF)) if True]
    for n, (site, thread, ins, mask) in enumerate(faults):
        r1 = L.ora_splitmix(seed, 8 * n + 1)
        r2 = L.ora_splitmix(seed, 8 * n + 2)
        r3 = L.ora_splitmix(seed, 8 * n + 3)
        assert site == en[(r1 * len(en)) >> 64]
        cls, width = O.site_info(O.TPACF, 1, site)
        if cls == 0:
            assert (thread, ins) == ((r2 * O.n_threads(O.TPACF, p)) >> 64, 0)
        else:
            assert (thread, ins) == inst[(r2 * len(inst)) >> 64]
        assert mask == 1 << ((r3 * width) >> 64)


def test_decode_is_shard_invariant_and_mixed_uses_n_mod_3():
    probs = [W.cp_small(), W.mriq_small(), W.tpacf_small()]
    b_all, f_all = O.decode(-1, probs, 7, 0, 600)
    b0, f0 = O.decode(-1, probs, 7, 0, 250)
    b1, f1 = O.decode(-1, probs, 7, 250, 350)
    assert list(b_all) == list(b0) + list(b1)
    assert f_all == f0 + f1
    assert list(b_all) == [n % 3 for n in range(600)]


def test_decode_sites_uniform_chi2():
    p = W.cp_small()
    n = 20000
    _, faults = O.decode(O.CP, [p, None, None], 2024, 0, n)
    ns = O.nsites(O.CP, p.unroll)
    counts = np.bincount([f[0] for f in faults], minlength=ns)
    exp = n / ns
    chi2 = float(((counts - exp) ** 2 / exp).sum())
    # 37 dof: p = 0.999 quantile ~ 69.3
    assert chi2 < 69.3, chi2
    bits = np.bincount([int(math.log2(f[3])) for f in faults if O.site_info(O.CP, p.unroll, f[0])[1] == 32], minlength=32)
    e = bits.sum() / 32
    assert float(((bits - e) ** 2 / e).sum()) < 61.1  # 31 dof, p = 0.999


def test_site_catalogue_sizes():
    # 22 + 4U CP sites (38 at U=4, 54 at U=8 ~ "20-50 virtual variables", L2298)
    assert O.nsites(O.CP, 4) == 38 and O.nsites(O.CP, 8) == 54
    assert O.nsites(O.MRIQ) == 36 and O.nsites(O.TPACF) == 30  # MRI-Q: 29 Q-kernel + 7 PhiMag sites


# ---------------------------------------------------------------- multi-bit masks (NEXT f1)
@pytest.mark.parametrize("k", [3, 6, 10, 15])
def test_multibit_masks_have_k_distinct_bits_and_extend_the_single_bit_draw(k):
    probs = [W.cp_small(), W.mriq_small(), W.tpacf_small()]
    _, one = O.decode(-1, probs, 31337, 0, 3000)
    _, many = O.decode(-1, probs, 31337, 0, 3000, nbits=k)
    counts = np.zeros(64)
    for (s1, t1, i1, m1), (s, t, i, m) in zip(one, many):
        assert (s1, t1, i1) == (s, t, i)                      # same site / thread / instance
        assert m & m1 == m1                                   # step 0 of the shuffle = the single-bit draw
        assert bin(m).count("1") == k
        for b in range(64):
            counts[b] += (m >> b) & 1
    # 32-bit sites dominate; every bit position of a 32-bit word is used ~uniformly
    c32 = counts[:32]
    assert c32.min() > 0.7 * c32.mean()
