"""Round-2 pins of the oracle (-m "not gpu"): the parts VERDICT r01 listed as "parity unpinned".

Each test fixes a value by hand derivation from the paper's text or by mathematics, never by
re-running the oracle's own formula:
  * R17 hang watchdog: a TPACF `je` flip whose in-bounds run outlives T x the
    golden trips is FAILURE(hang); with a larger T the same flip walks off the buffer (crash).
  * R11 alpha widening (L2073-2077): bounds and verdicts computed by hand at alpha = 10.
  * A6 selection (L1221-1273): Fig. 9's printed counts 12 / 13 and the choice of energyx2
    (L1252-1258), and the selection order it implies for this build's CP / MRI-Q / TPACF loops.
  * R20 FAST transcendentals: closed forms and the MUFU special cases (PTX ISA: .ftz flushes
    denormal inputs; sin/cos of +-inf or NaN are NaN; rsqrt(+-0) = +-inf, rsqrt(<0) = NaN).
  * the double-precision MRI-Q reference's Qr / Qi (one k-sample closed form, k = 0 sum).
  * recovery arithmetic (A11 range extension L1309-1313, alpha controller L2066-2077, Fig. 11
    diagnosis L2021-2058) and the coverage summary (R2, L2372-2375, the paper's bookkeeping).
  * the FI-only binary (row a7, L786-797): its catalogue holds no detector-only site and the data
    path of a fault is the same with or without the detectors.
"""
import math
import os

import numpy as np
import pytest

import oracle as O
import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _f32(x):
    return float(np.float32(x))


# ------------------------------------------------------------------------------ R17 hang model
def _tp64():
    return W.tpacf_small(n=64, n_rand=2)


def test_tpacf_je_flip_is_a_hang_after_ten_times_the_golden_trips():
    """Thread (h = 1 [RR_1], i = 62): jb = 63, golden trips = 1, limit = 10 x max(1, 1) = 10.
    je (@live site 12) 64 -> 64 ^ 2^20 at iteration 0.  Partners sit at pts[3 (boff + j) + a] with
    boff = 64: in bounds while 64 + j < 3 x 64, i.e. j <= 127 -> 65 in-bounds iterations from j = 63,
    more than 10, so the watchdog fires at iteration 10 (R17) before any out-of-bounds load."""
    p = _tp64()
    R = O.profile_ranges(O.TPACF, p)
    g = 1 * p.n + 62
    assert O.trips(O.TPACF, p)[g] == 1
    _, _, info = O.run(O.TPACF, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(12, g, 0, 1 << 20))
    assert info.applied and info.fail == O.FL_HANG
    assert O.lib().ora_classify(0, 0, O.FL_HANG) == O.FAILURE  # R1: failure takes precedence


def test_tpacf_same_flip_crashes_when_the_watchdog_allows_more_than_the_buffer():
    """Same injection with T = 100: limit 100 > 65 in-bounds iterations, so the load of j = 128
    (element 3 x 192 = 576 of a 576-float buffer) is out of bounds first: a modelled crash (R16)."""
    p = _tp64()
    R = O.profile_ranges(O.TPACF, p)
    g = 1 * p.n + 62
    _, _, info = O.run(O.TPACF, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(12, g, 0, 1 << 20, hang=100))
    assert info.fail == O.FL_CRASH


def test_tpacf_dr_row_je_flip_crashes_before_the_watchdog():
    """DR_1 (h = n_rand + 1 = 3), i = 5: jb = 0, golden trips = 64, limit 640; boff = 64 again, so
    only 64 more in-bounds partners (j = 64..127) exist past je: the load of j = 128 crashes."""
    p = _tp64()
    R = O.profile_ranges(O.TPACF, p)
    g = 3 * p.n + 5
    assert O.trips(O.TPACF, p)[g] == 64
    _, _, info = O.run(O.TPACF, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(12, g, 0, 1 << 20))
    assert info.fail == O.FL_CRASH


def test_cp_atomid_rewind_repeats_iterations_without_a_hang_but_a_count_mismatch():
    """atomid 36 -> 4 (bit 5 cleared) at the last iteration of a 37-atom loop: 33 extra iterations,
    70 in all, below the 10 x 37 limit: no failure; it = 70 != 37 -> count alarm (A9)."""
    p = W.cp_small()
    R = O.profile_ranges(O.CP, p)
    assert p.n_atoms == 37 and (36 ^ (1 << 5)) == 4
    _, _, info = O.run(O.CP, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(14, 9, 36, 1 << 5))
    assert info.fail == 0 and info.alarm & O.AL_COUNT
    # with T = 1 the 38th iteration already exceeds the limit of 37 trips: a hang
    _, _, info = O.run(O.CP, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(14, 9, 36, 1 << 5, hang=1))
    assert info.fail == O.FL_HANG


# ------------------------------------------------------------------------------ R11 alpha
def _ranges(pairs, alpha, t=-6):
    R = O.Ranges()
    R.n_det = 1
    R.alpha = alpha
    R.det[0].n = len(pairs)
    R.det[0].t_exp10 = t
    for r, (lo, hi) in enumerate(pairs):
        R.det[0].lo[r] = lo
        R.det[0].hi[r] = hi
    return R


def test_alpha_ten_widens_each_bound_away_from_its_range():
    """R11 (L2073-2077: max x alpha and min / alpha for positive bounds; negative bounds mirrored):
    [-0.5, -2e-6] -> [-5, -2e-7], [3e-6, 2] -> [3e-7, 20] at alpha = 10 (binary32 products)."""
    pairs = [(_f32(-0.5), _f32(-2e-6)), (_f32(3e-6), _f32(2.0))]
    R1, R10 = _ranges(pairs, 1.0), _ranges(pairs, 10.0)
    lo_n, hi_n = _f32(_f32(-0.5) * 10), _f32(np.float32(-2e-6) / np.float32(10))
    lo_p, hi_p = _f32(np.float32(3e-6) / np.float32(10)), _f32(_f32(2.0) * 10)
    assert (lo_n, lo_p, hi_p) == (-5.0, _f32(3e-7), 20.0) and abs(hi_n + 2e-7) < 1e-13
    for v, in1, in10 in [(-4.9, False, True), (-5.01, False, False), (-0.4, True, True), (-1e-6, False, True), (-3e-6, True, True),
                         (-1e-7, False, False), (0.0, False, False), (2.5e-7, False, False), (3.1e-7, False, True),
                         (2.9e-6, False, True), (1.0, True, True), (19.9, False, True), (20.01, False, False),
                         (float("nan"), False, False)]:
        assert O.in_range(R1, 0, v) == in1, v
        assert O.in_range(R10, 0, v) == in10, v
    # exact boundary values are inside (inclusive compares, R10)
    for v in (lo_n, hi_n, lo_p, hi_p):
        assert O.in_range(R10, 0, v)


def test_alpha_keeps_a_zero_bound_and_widens_a_zero_straddling_range():
    R = _ranges([(_f32(-1e-5), 0.0)], 10.0)
    assert O.in_range(R, 0, _f32(-9.9e-5)) and not O.in_range(R, 0, _f32(-1.01e-4))
    assert O.in_range(R, 0, 0.0) and not O.in_range(R, 0, _f32(1e-30))
    R = _ranges([(_f32(-1e-5), _f32(1e-5))], 10.0)
    assert O.in_range(R, 0, _f32(9.9e-5)) and not O.in_range(R, 0, _f32(1.01e-4))


def test_alpha_ten_campaign_detects_no_more_than_alpha_one():
    """Wider ranges can only turn range alarms off (L2078-2081: looser ranges, more false
    negatives): on the same seeded campaign every alpha = 10 alarm set is a subset of alpha = 1's."""
    p = W.cp_small()
    R1 = O.profile_ranges(O.CP, p)
    R10 = O.profile_ranges(O.CP, p, alpha=10.0)
    c1, r1 = O.campaign(O.CP, [p, None, None], [R1, None, None], 77, 0, 300, mode=1)
    c10, r10 = O.campaign(O.CP, [p, None, None], [R10, None, None], 77, 0, 300, mode=1)
    assert np.all((r10["alarm"] & ~r1["alarm"]) == 0)
    assert int(c10[0, O.UNDETECTED]) >= int(c1[0, O.UNDETECTED])


# ------------------------------------------------------------------------------ A6 selection
V, T, LD, K, NLP, ACC = O.A6_VAR, O.A6_TEMP, O.A6_LOAD, O.A6_CONST, O.A6_NLPROT, O.A6_ACCOP  # + O.A6_IND


class G:
    def __init__(self):
        self.names, self.kinds, self.selfacc, self.edges = [], [], [], []

    def node(self, name, kind, selfacc=False, srcs=()):
        self.names.append(name)
        self.kinds.append(kind)
        self.selfacc.append(1 if selfacc else 0)
        i = len(self.names) - 1
        for s in srcs:
            self.edges.append((self.names.index(s), i))
        if selfacc:
            self.edges.append((i, i))
        return i

    def count(self, name):
        return O.a6_count(self.kinds, self.edges, self.names.index(name))

    def select(self, maxvar):
        return [self.names[i] for i in O.a6_select(self.kinds, self.selfacc, self.edges, maxvar)]


def fig9_graph():
    """PAPER Fig. 9 (L1315-1392, text L1242-1258): the CP loop with two unrolled points.  Loads of
    atominfo[atomid].{x,y,z,w} (the address is not data); coorx / coory / gridspacing_u are the
    loop invariants protected by non-loop detectors (black ellipses); T1..T9 temporaries; the
    `x w` product of each `energyx += w * (1/sqrt(...))` is the accumulate statement's own op."""
    g = G()
    g.node("coorx", NLP); g.node("coory", NLP); g.node("gu", NLP); g.node("one", K)
    for a in "xyzw":
        g.node("L" + a, LD)
    g.node("dy", V, srcs=("coory", "Ly"))
    g.node("T1", T, srcs=("dy",))                     # dy * dy
    g.node("dyz2", V, srcs=("T1", "Lz"))
    g.node("dx1", V, srcs=("coorx", "Lx"))
    g.node("dx2", V, srcs=("dx1", "gu"))
    g.node("T2", T, srcs=("dx1",)); g.node("T3", T, srcs=("T2", "dyz2")); g.node("T4", T, srcs=("T3",))
    g.node("T5", T, srcs=("one", "T4"))               # 1.0 / sqrt
    g.node("M1", ACC, srcs=("Lw", "T5"))
    g.node("energyx1", V, selfacc=True, srcs=("M1",))
    g.node("T6", T, srcs=("dx2",)); g.node("T7", T, srcs=("T6", "dyz2")); g.node("T8", T, srcs=("T7",))
    g.node("T9", T, srcs=("one", "T8"))
    g.node("M2", ACC, srcs=("Lw", "T9"))
    g.node("energyx2", V, selfacc=True, srcs=("M2",))
    return g


def test_fig9_cumulative_backward_dependency_is_12_and_13_and_energyx2_is_chosen():
    g = fig9_graph()
    assert g.count("energyx1") == 12 and g.count("energyx2") == 13
    assert g.select(1) == ["energyx2"]                                # "we first select energyx2", L1258


def cp_graph(U):
    """This build's fused CP loop: fmaf for dyz2 / r2 / the accumulate, one rsqrt."""
    g = G()
    g.node("coorx", NLP); g.node("coory", NLP); g.node("gu", NLP)
    g.node("atomid", O.A6_IND)  # induction variable: covered by the iteration counter (A9)
    for a in "xyzw":
        g.node("a" + a, LD)
    g.node("dy", V, srcs=("coory", "ay"))
    g.node("dyz2", V, srcs=("dy", "az"))
    g.node("dx0", V, srcs=("coorx", "ax"))
    for j in range(1, U):
        g.node(f"dx{j}", V, srcs=(f"dx{j - 1}", "gu"))
    for j in range(U):
        g.node(f"r2_{j}", V, srcs=(f"dx{j}", "dyz2"))
        g.node(f"s{j}", V, srcs=(f"r2_{j}",))
        g.node(f"E{j}", V, selfacc=True, srcs=("aw", f"s{j}"))
    return g


@pytest.mark.parametrize("U", [1, 2, 4, 8])
def test_cp_fused_graph_counts_and_selection_order(U):
    """E_j's backward set = 4 loads, dy, dyz2, dx_0..dx_j, r2_j, s_j = 8 + j + 1 (9 and 10 for
    E_0 / E_1).  Once E_{U-1} and its ancestors are removed every other E_j keeps
    {r2_j, s_j}: a tie resolved in program order (R12) -> E_{U-1}, E_0, E_1, ..., E_{U-2}; the
    kernels' detector d checks exactly that accumulator (cp_sel in the oracle, cp.cu)."""
    g = cp_graph(U)
    for j in range(U):
        assert g.count(f"E{j}") == 9 + j
    assert g.select(U) == [f"E{U - 1}"] + [f"E{j}" for j in range(U - 1)]


def test_mriq_graph_selects_qr_then_qi_and_tpacf_selects_bin():
    g = G()
    for nm in ("sX", "sY", "sZ"):
        g.node(nm, NLP)
    g.node("C", K); g.node("twopi", K); g.node("k", O.A6_IND)
    for nm in ("kx", "ky", "kz", "pm"):
        g.node(nm, LD)
    g.node("t1", V, srcs=("kx", "sX")); g.node("t2", V, srcs=("ky", "sY", "t1")); g.node("t", V, srcs=("kz", "sZ", "t2"))
    g.node("u1", T, srcs=("t", "C")); g.node("u2", T, srcs=("u1", "C")); g.node("r", V, srcs=("t", "u2"))
    g.node("ang", T, srcs=("r", "twopi"))
    g.node("c", V, srcs=("ang",)); g.node("s", V, srcs=("ang",))
    g.node("Qr", V, selfacc=True, srcs=("pm", "c")); g.node("Qi", V, selfacc=True, srcs=("pm", "s"))
    assert g.count("Qr") == g.count("Qi") == 12
    assert g.select(2) == ["Qr", "Qi"]  # tie -> program order (R12); then Qi keeps {s}
    h = G()
    for nm in ("x1", "y1", "z1"):
        h.node(nm, NLP)
    h.node("j", O.A6_IND)
    for nm in ("x2", "y2", "z2", "edge"):
        h.node(nm, LD)
    h.node("p1", T, srcs=("x1", "x2")); h.node("p2", T, srcs=("y1", "y2", "p1"))
    h.node("dot", V, srcs=("z1", "z2", "p2"))
    h.node("bin", V, srcs=("dot", "edge"))
    h.node("hidx", T, srcs=("bin",))   # the histogram store's address temporary
    assert h.count("bin") == 7 and h.count("dot") == 5
    assert h.select(1) == ["bin"]      # DESIGN R12: TPACF protects bin (acc += bin)


# ------------------------------------------------------------------------------ R20 FAST specials
def test_fast_transcendentals_closed_forms_and_mufu_special_cases():
    L = O.lib()
    sin, cos, rsq = (lambda x: L.ora_sin(x, 0)), (lambda x: L.ora_cos(x, 0)), (lambda x: L.ora_rsqrt(x, 0))
    bits = lambda x: int(np.array([x], dtype=np.float32).view(np.uint32)[0])
    # closed forms (correctly rounded binary32 of the exact value)
    assert sin(0.0) == 0.0 and bits(sin(-0.0)) == 0x80000000 and cos(0.0) == 1.0 and cos(-0.0) == 1.0
    pi_f = _f32(math.pi)                       # 3.14159274 > pi: sin(pi_f) = sin(pi - pi_f) = -8.742278e-8
    assert sin(pi_f) == _f32(math.sin(float(pi_f))) and abs(sin(pi_f) + 8.742278e-8) < 1e-14
    assert abs(sin(_f32(math.pi / 6)) - 0.5) <= 2 ** -24 and abs(cos(_f32(math.pi / 3)) - 0.5) <= 2 ** -23
    assert rsq(4.0) == 0.5 and rsq(0.25) == 2.0 and rsq(1.0) == 1.0
    # MUFU .ftz: denormal inputs are flushed to a signed zero first
    den = float(np.array([1], dtype=np.uint32).view(np.float32)[0])
    assert bits(sin(den)) == 0 and bits(sin(-den)) == 0x80000000 and cos(den) == 1.0 and cos(-den) == 1.0
    assert rsq(den) == math.inf and rsq(-den) == -math.inf
    # rsqrt(+-0) = +-inf, rsqrt(< 0) = NaN, rsqrt(+inf) = +0; sin / cos of +-inf and NaN are NaN
    assert rsq(0.0) == math.inf and rsq(-0.0) == -math.inf and math.isnan(rsq(-1.0)) and rsq(math.inf) == 0.0
    for x in (math.inf, -math.inf, math.nan):
        assert math.isnan(sin(x)) and math.isnan(cos(x))


def test_mriq_double_reference_qr_qi_closed_forms():
    """One k-sample: Q = |phi|^2 e^{i 2 pi k.x}; k = 0: Qr = sum |phi|^2, Qi = 0 (the plain MRI-Q
    definition) — the f64 reference's own outputs, not only its mass."""
    p = W.mriq_problem(4, 1, n_vox=64, seed=3)
    (qr, qi), mass = O.reference_f64(O.MRIQ, p)
    pm = float(p.phi_r[0]) ** 2 + float(p.phi_i[0]) ** 2
    arg = 2 * math.pi * (float(p.kx[0]) * p.x.astype(np.float64) + float(p.ky[0]) * p.y + float(p.kz[0]) * p.z)
    assert np.allclose(qr, pm * np.cos(arg), rtol=0, atol=1e-12) and np.allclose(qi, pm * np.sin(arg), rtol=0, atol=1e-12)
    assert np.allclose(mass, pm)
    q = W.mriq_problem(4, 9, n_vox=20, seed=4)
    for a in (q.kx, q.ky, q.kz):
        a[:] = 0
    (qr, qi), _ = O.reference_f64(O.MRIQ, q)
    tot = float((q.phi_r.astype(np.float64) ** 2 + q.phi_i.astype(np.float64) ** 2).sum())
    assert np.allclose(qr, tot, rtol=1e-15) and np.all(qi == 0)


# ------------------------------------------------------------------------------ recovery twins
def test_extend_ranges_joins_each_value_to_its_correlation_class():
    """A11 / R24 at T = 1e-6: -3 widens the negative range, 5e-7 lands in the (missing) zero class
    and creates it, 4 widens the positive range; NaN is ignored.  Classes stay ordered."""
    rs = O.RSet()
    rs.n, rs.t_exp10 = 2, -6
    rs.lo[0], rs.hi[0], rs.lo[1], rs.hi[1] = _f32(-0.5), _f32(-2e-6), _f32(3e-6), _f32(2.0)
    added = O.extend_ranges(rs, [-3.0, 5e-7, 4.0, float("nan")])
    assert added == 1 and rs.n == 3
    got = [(rs.lo[r], rs.hi[r]) for r in range(3)]
    assert got == [(-3.0, _f32(-2e-6)), (_f32(5e-7), _f32(5e-7)), (_f32(3e-6), 4.0)]
    rs2 = O.RSet()
    rs2.n, rs2.t_exp10 = 0, -5
    assert O.extend_ranges(rs2, [_f32(1e-6), -7.0]) == 2
    assert [(rs2.lo[r], rs2.hi[r]) for r in range(rs2.n)] == [(-7.0, -7.0), (_f32(1e-6), _f32(1e-6))]


def test_alpha_controller_sequence():
    """L2066-2077: > 10 % false positives -> x 10; < 5 % -> / 10 as long as alpha stays >= 1."""
    a, seq = 1.0, []
    for fp in (0.2, 0.5, 0.07, 0.01, 0.01, 0.01, 0.10, 0.05):
        a = O.alpha_step(a, fp)
        seq.append(a)
    assert seq == [10.0, 100.0, 100.0, 10.0, 1.0, 1.0, 1.0, 1.0]


def test_reexecution_diagnosis_truth_table():
    """Fig. 11 (L2021-2058)."""
    assert O.diagnose(0, 0, 0, 0, True) == "ok"
    assert O.diagnose(4, 0, 4, 0, True) == "false_alarm"
    assert O.diagnose(4, 0, 8, 0, True) == "false_alarm"        # "also raises an SDC alarm"
    assert O.diagnose(4, 0, 0, 0, False) == "transient"         # re-run ends normally, no alarm
    assert O.diagnose(4, 0, 4, 0, False) == "persistent"        # alarm again, different output
    assert O.diagnose(0, 1, 0, 0, True) == "failed" and O.diagnose(4, 0, 0, 2, True) == "failed"


def test_coverage_summary_reproduces_the_paper_bookkeeping():
    """L2567-2573 single-bit breakdown (x 10 injections): coverage = 1 - undetected = 90.2 %."""
    rows = [l.split() for l in open(os.path.join(GOLDEN, "paper_outcomes.txt")) if l.strip() and not l.startswith("#")]
    masked, failure, detected, det_masked, undetected = [round(float(v) * 10) for v in rows[0]]
    counts = np.array([masked, det_masked, detected, undetected, failure], dtype=np.int64)
    s = O.coverage(counts)
    assert abs(s["coverage"] - 0.902) < 1e-12 and abs(s["sdc"] - 0.098) < 1e-12
    assert abs(s["detected"] - 0.436) < 1e-12 and abs(s["failure"] - 0.110) < 1e-12
    assert math.isnan(O.coverage(np.zeros(5, np.int64))["coverage"])


# ------------------------------------------------------------------------------ FI-only binary (a7)
def test_detector_only_sites():
    assert [s for s in range(O.nsites(O.CP, 4)) if O.detector_site(O.CP, s, 4)] == [37]
    assert [s for s in range(O.nsites(O.MRIQ)) if O.detector_site(O.MRIQ, s)] == [28]
    assert [s for s in range(O.nsites(O.TPACF)) if O.detector_site(O.TPACF, s)] == [6, 13, 28, 29]


@pytest.mark.parametrize("bench", [O.CP, O.MRIQ, O.TPACF])
def test_fi_only_campaign_uses_original_sites_and_never_alarms(bench):
    probs = [W.cp_small(), W.mriq_problem(4, 23, n_vox=60), W.tpacf_small(n=60, n_rand=1)]
    pr = [probs[b] if b == bench else None for b in range(3)]
    R = [O.profile_ranges(b, probs[b]) if b == bench else None for b in range(3)]
    c, rec = O.campaign(bench, pr, R, 5150, 0, 400, mode=1, variant=1)
    U = getattr(probs[bench], "unroll", 4)
    assert not any(O.detector_site(bench, int(s), U) for s in rec["site"])
    assert (rec["alarm"] == 0).all() and c[bench, O.DET_MASKED] == 0 and c[bench, O.DETECTED] == 0
    c0, rec0 = O.campaign(bench, pr, R, 5150, 0, 400, mode=0, variant=1)
    assert np.array_equal(c, c0) and np.array_equal(rec["cls"], rec0["cls"])


@pytest.mark.parametrize("bench", [O.CP, O.MRIQ, O.TPACF])
def test_detectors_never_change_the_data_path_of_a_fault(bench):
    """HAUBERK only sets alarm bits: for the same fault on an original-program site,
    the FI-only run and the FI&FT run produce bitwise-identical outputs and the same failure."""
    p = [W.cp_small(), W.mriq_problem(4, 23, n_vox=60), W.tpacf_small(n=60, n_rand=1)][bench]
    R = O.profile_ranges(bench, p)
    _, faults = O.decode(bench, [p if b == bench else None for b in range(3)], 808, 0, 60, variant=1)
    for (site, thread, inst, mask) in faults:
        f = O.fault(site, thread, inst, mask)
        a, _, ia = O.run(bench, p, flags=0, ranges=R, ndet=R.n_det, f=f)
        b, _, ib = O.run(bench, p, flags=O.FT, ranges=R, ndet=R.n_det, f=f)
        assert ia.fail == ib.fail and ia.alarm == 0
        if not ia.fail:
            for x, y in zip(a if bench == O.MRIQ else (a,), b if bench == O.MRIQ else (b,)):
                assert np.array_equal(np.asarray(x).view(np.uint8), np.asarray(y).view(np.uint8)), (site, thread)
