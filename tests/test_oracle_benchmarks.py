"""Pins of the oracle's benchmark arithmetic and detector semantics (-m "not gpu").

Benchmarks are checked against closed forms (single charge, one k-sample, k = 0), superposition,
numpy brute force in double (an independent program), and pair-count totals.  Detectors are
checked against the invariants the paper states (chk == 0 and no alarm fault-free, PAPER L993-995,
L2402-2403) and directed injections whose outcome follows from the method by reasoning (T4)."""
import math

import numpy as np
import pytest

import oracle as O
import workloads as W


def _cp(atoms, nx=32, ny=16, h=0.25, bx=8, by=4, unroll=2, z0=0.0):
    a = np.asarray(atoms, dtype=np.float32).reshape(-1, 4)
    return W.CPProblem(atoms=a, nx=nx, ny=ny, h=float(np.float32(h)), z0=z0, bx=bx, by=by, unroll=unroll)


def _grid_xy(p):
    h = np.float32(p.h)
    xs = (h * np.arange(p.nx, dtype=np.float32)).astype(np.float64)
    ys = (h * np.arange(p.ny, dtype=np.float32)).astype(np.float64)
    return np.meshgrid(xs, ys)


# ---------------------------------------------------------------- CP (K1)
@pytest.mark.parametrize("unroll", [1, 2, 4, 8])
def test_cp_single_charge_closed_form(unroll):
    p = _cp([[1.3, 2.2, 0.75, -0.8]], nx=64, ny=8, bx=8, unroll=unroll)
    out, _, info = O.run(O.CP, p)
    X, Y = _grid_xy(p)
    dz = np.float64(np.float32(0.75))
    exact = -0.8 / np.sqrt((X - np.float32(1.3)) ** 2 + (Y - np.float32(2.2)) ** 2 + dz * dz)
    exact *= float(np.float32(-0.8)) / -0.8
    assert np.max(np.abs(out - exact) / np.abs(exact)) < 4e-7
    assert info.alarm == 0


def test_cp_superposition_and_antisymmetry():
    a1 = [2.0, 1.0, 0.5, 0.7]
    a2 = [5.5, 3.0, 1.25, -0.3]
    p1, p2, p12 = _cp([a1]), _cp([a2]), _cp([a1, a2])
    o1, o2, o12 = (O.run(O.CP, p)[0] for p in (p1, p2, p12))
    assert np.max(np.abs(o12 - (o1 + o2)) / (np.abs(o1) + np.abs(o2))) < 3e-7
    # +q and -q mirrored across the line x = 4: E = 0 on the grid column at x = 4 (h = 0.25, column 16)
    pa = _cp([[3.0, 2.0, 1.0, 1.0], [5.0, 2.0, 1.0, -1.0]])
    oa = O.run(O.CP, pa)[0]
    assert np.max(np.abs(oa[:, 16])) < 1e-6
    assert np.max(np.abs(oa)) > 0.1


def test_cp_bruteforce_double_numpy():
    p = W.cp_small()
    out, _, _ = O.run(O.CP, p)
    # the definition: grid point (h*x, h*y) exactly (the fp32 program rounds h*x; its error budget)
    X, Y = np.meshgrid(p.h * np.arange(p.nx, dtype=np.float64), p.h * np.arange(p.ny, dtype=np.float64))
    a = p.atoms.astype(np.float64)
    terms = a[:, 3, None, None] / np.sqrt((X[None] - a[:, 0, None, None]) ** 2 + (Y[None] - a[:, 1, None, None]) ** 2 + (a[:, 2, None, None] - p.z0) ** 2)
    ref = terms.sum(0)
    mass = np.abs(terms).sum(0)
    # R21: relative 1e-5, or 4 * 2^-23 * mass where the sum cancels
    bad = np.abs(out - ref) > np.maximum(1e-5 * np.abs(ref), 4 * 2.0**-23 * mass)
    assert not bad.any()
    # and the oracle's own double definition is the same program
    ref2, _ = O.reference_f64(O.CP, p)
    assert np.allclose(ref, ref2, rtol=1e-12, atol=0)


def test_cp_exact_mode_rsqrt_spec_accuracy():
    L = O.lib()
    xs = np.float32(10.0) ** np.linspace(-6, 6, 301).astype(np.float32)
    for x in xs:
        e = L.ora_rsqrt(float(x), 1)
        assert abs(e - 1 / math.sqrt(float(x))) <= 2.5e-7 / math.sqrt(float(x))
        f = L.ora_rsqrt(float(x), 0)
        assert f == float(np.float32(1 / math.sqrt(float(x))))
    assert L.ora_rsqrt(0.0, 0) == math.inf and L.ora_rsqrt(-0.0, 0) == -math.inf
    assert math.isnan(L.ora_rsqrt(-1.0, 0)) and L.ora_rsqrt(math.inf, 0) == 0.0


def test_cp_ft_output_bit_equal_to_base_and_no_alarm():
    p = W.cp_small()
    base = O.run(O.CP, p, flags=0)[0]
    R = O.profile_ranges(O.CP, p, maxvar=p.unroll)
    ft, _, info = O.run(O.CP, p, flags=O.FT, ranges=R, ndet=p.unroll)
    assert np.array_equal(base.view(np.uint32), ft.view(np.uint32))
    assert info.alarm == 0 and info.n_alarm_threads == 0


# ---------------------------------------------------------------- MRI-Q (K2)
def _mriq_one(kx, ky, kz, pr, pi, side=4):
    p = W.mriq_problem(side, 1)
    p.kx[:] = kx; p.ky[:] = ky; p.kz[:] = kz; p.phi_r[:] = pr; p.phi_i[:] = pi
    return p


@pytest.mark.parametrize("exact", [0, 1])
def test_mriq_single_k_closed_form(exact):
    p = _mriq_one(3.25, -1.5, 0.75, 0.6, -0.8)
    (qr, qi), _, info = O.run(O.MRIQ, p, exact=exact)
    pm = 0.6**2 + 0.8**2
    arg = 2 * math.pi * (3.25 * p.x.astype(np.float64) - 1.5 * p.y + 0.75 * p.z)
    tol = 2e-6 if not exact else 3e-6
    assert np.max(np.abs(qr - pm * np.cos(arg))) < tol
    assert np.max(np.abs(qi - pm * np.sin(arg))) < tol


def test_mriq_k_zero_sums_phimag():
    p = W.mriq_problem(4, 5)
    p.kx[:] = 0; p.ky[:] = 0; p.kz[:] = 0
    (qr, qi), _, _ = O.run(O.MRIQ, p)
    pm = (p.phi_r.astype(np.float64) ** 2 + p.phi_i.astype(np.float64) ** 2).sum()
    assert np.allclose(qr, pm, rtol=1e-6) and np.all(qi == 0)


def test_mriq_bruteforce_double_numpy():
    p = W.mriq_small()
    (qr, qi), _, _ = O.run(O.MRIQ, p)
    pm = p.phi_r.astype(np.float64) ** 2 + p.phi_i.astype(np.float64) ** 2
    arg = 2 * np.pi * (np.outer(p.x, p.kx) + np.outer(p.y, p.ky) + np.outer(p.z, p.kz))
    rr, ri = (np.cos(arg) * pm).sum(1), (np.sin(arg) * pm).sum(1)
    mass = pm.sum()
    for got, ref in ((qr, rr), (qi, ri)):
        assert not (np.abs(got - ref) > np.maximum(1e-5 * np.abs(ref), 8 * 2.0**-23 * mass)).any()


def test_mriq_exact_transcendentals_accuracy():
    L = O.lib()
    for a in np.linspace(-math.pi, math.pi, 257):
        a = float(np.float32(a))
        assert abs(L.ora_sin(a, 1) - math.sin(a)) < 6e-7
        assert abs(L.ora_cos(a, 1) - math.cos(a)) < 6e-7


# ---------------------------------------------------------------- TPACF (K3)
def _tpacf_bruteforce(p):
    """Independent definition: double angle via acos, log10(arcmin) binning, 5 bins per decade."""
    pts = p.pts.astype(np.float64)
    nr = p.n_rand
    nb = p.n_bins
    hist = np.zeros((1 + 2 * nr, nb + 2), dtype=np.int64)
    near_edge = 0

    def add(h, A, B, self_pairs):
        nonlocal near_edge
        dot = np.clip(A @ B.T, -1, 1)
        if self_pairs:
            iu = np.triu_indices(A.shape[0], 1)
            dot = dot[iu]
        else:
            dot = dot.ravel()
        ang = np.degrees(np.arccos(dot)) * 60.0
        with np.errstate(divide="ignore"):
            lg = np.log10(ang) * nb / 4.0  # edges at 10^(k/5) arcmin, k = 0..nb (1..1e4 arcmin)
        b = np.where(ang < 1.0, 0, np.where(ang >= 1e4, nb + 1, np.floor(lg).astype(np.int64) + 1))
        # fp32 dot error ~2.4e-7 absolute -> angle error 2.4e-7/sin(theta); in bin units (5 per decade):
        th = np.radians(ang / 60.0)
        with np.errstate(divide="ignore"):
            unc = 10 * (nb / 4.0) / math.log(10) * 2.4e-7 / (np.sin(th) * th)
        frac = np.abs(lg - np.round(lg))
        near_edge += int(np.sum((frac < unc) & (ang > 0.5) & (ang < 2e4)))
        hist[h] += np.bincount(b, minlength=nb + 2)

    add(0, pts[0], pts[0], True)
    for s in range(1, nr + 1):
        add(s, pts[s], pts[s], True)
        add(nr + s, pts[0], pts[s], False)
    return hist, near_edge


@pytest.mark.parametrize("seed", [8, 1, 5, 13])
def test_tpacf_bruteforce_acos_binning_and_totals(seed):
    p = W.tpacf_problem(64, 2, seed=seed, clumps=4, sigma_deg=3.0)
    h, _, info = O.run(O.TPACF, p)
    ref, near = _tpacf_bruteforce(p)
    # bin 0 (< 1 arcmin) is rounding-dominated in fp32 (edge[0] = 1 - 2^-24); compare bins >= 1.
    # Pairs within fp32 rounding of an edge may legitimately land in either neighbour.
    assert np.abs(h[:, 1:] - ref[:, 1:]).sum() <= 2 * near
    if near == 0:
        assert np.array_equal(h[:, 1:], ref[:, 1:])
    n = p.n
    assert all(h[k].sum() == n * (n - 1) // 2 for k in range(1 + p.n_rand))
    assert all(h[k].sum() == n * n for k in range(1 + p.n_rand, 1 + 2 * p.n_rand))
    assert info.alarm == 0


def test_tpacf_abstract_threads_and_trip_counts_follow_the_program():
    """one abstract thread per (histogram h, point i) over partners j in [jb, N):
    nh * N threads; trips N - i - 1 on the self-correlation rows (DD, RR_s), N on the DR rows."""
    p = W.tpacf_small(n=37, n_rand=2)
    n, nr = p.n, p.n_rand
    assert O.n_threads(O.TPACF, p) == (1 + 2 * nr) * n
    tr = O.trips(O.TPACF, p).reshape(1 + 2 * nr, n)
    for h in range(1 + 2 * nr):
        want = [n - i - 1 for i in range(n)] if h <= nr else [n] * n
        assert tr[h].tolist() == want


def test_tpacf_trip_counts_sum_to_pairs():
    p = W.tpacf_small(n=100, n_rand=2)
    tr = O.trips(O.TPACF, p)
    n = p.n
    assert tr.sum() == 3 * n * (n - 1) // 2 + 2 * n * n


def test_tpacf_edges_are_strictly_decreasing_fp32():
    e = W.tpacf_edges()
    assert np.all(np.diff(e) < 0)
    # fp32 quantisation of the first edges: 1, 2 and 4 ulps below 1.0
    below = (1.0 - e[:3].astype(np.float64)) / 2.0**-24
    assert list(np.round(below)) == [1, 2, 4]


# ---------------------------------------------------------------- detector invariants & directed faults
BENCH_PROBS = {O.CP: W.cp_small, O.MRIQ: W.mriq_small, O.TPACF: lambda: W.tpacf_small(n=120, n_rand=2)}


@pytest.mark.parametrize("bench", [O.CP, O.MRIQ, O.TPACF])
@pytest.mark.parametrize("exact", [0, 1])
def test_fault_free_runs_raise_no_alarm(bench, exact):
    if bench == O.TPACF and exact:
        pytest.skip("TPACF has no transcendentals")
    p = BENCH_PROBS[bench]()
    maxvar = {O.CP: p.unroll if bench == O.CP else 1, O.MRIQ: 2, O.TPACF: 1}[bench]
    R = O.profile_ranges(bench, p, maxvar=maxvar, exact=exact)
    _, _, info = O.run(bench, p, flags=O.FT, exact=exact, ranges=R, ndet=maxvar)
    assert info.alarm == 0


def _one(bench, p, R, site, thread, inst, mask, exact=0):
    f = O.fault(site, thread, inst, mask)
    out, _, info = O.run(bench, p, flags=O.FT, exact=exact, ranges=R, ndet=R.n_det, f=f)
    assert info.applied == 1
    return out, info


@pytest.mark.parametrize("bench", [O.CP, O.MRIQ, O.TPACF])
def test_every_nl_def_flip_is_detected_by_the_duplicate(bench):
    p = BENCH_PROBS[bench]()
    R = O.profile_ranges(bench, p)
    rng = np.random.default_rng(bench)
    nthr = O.n_threads(bench, p)
    nl = [s for s in range(O.nsites(bench, getattr(p, "unroll", 1))) if O.site_info(bench, getattr(p, "unroll", 1), s)[0] == 0]
    for s in nl:
        for _ in range(3):
            t = int(rng.integers(p.n_k if (bench == O.MRIQ and s >= 29) else nthr)); b = int(rng.integers(32))
            _, info = _one(bench, p, R, s, t, 0, 1 << b)
            assert info.fail or (info.alarm & O.AL_DUP), (s, t, b)


def test_cp_bit30_of_selected_accumulator_at_last_iteration_is_a_range_miss():
    p = W.cp_small()
    R = O.profile_ranges(O.CP, p)  # maxvar = 1 -> E_{U-1}
    U = p.unroll
    s_E = 22 + (U - 1) + 2 * U + (U - 1)  # E_{U-1}
    for t in (0, 17, 200):
        _, info = _one(O.CP, p, R, s_E, t, p.n_atoms - 1, 1 << 30)
        assert info.alarm & O.AL_RANGE and not info.fail


def test_cp_low_mantissa_flip_of_accumulator_is_masked():
    p = W.cp_small()
    R = O.profile_ranges(O.CP, p)
    U = p.unroll
    s_E0 = 22 + (U - 1) + 2 * U  # E_0: not range checked at maxvar = 1
    golden = O.run(O.CP, p, flags=O.FT, ranges=R, ndet=1)[0]
    out, info = _one(O.CP, p, R, s_E0, 5, p.n_atoms - 1, 1 << 1)
    assert info.alarm == 0 and info.fail == 0
    M = np.abs(golden).max()
    assert np.all(np.abs(out - golden) <= np.maximum(1e-4 * M, 0.002 * np.abs(golden)))


def test_cp_counter_flip_is_a_count_mismatch():
    p = W.cp_small()
    R = O.profile_ranges(O.CP, p)
    s_it = 22 + 4 * p.unroll - 1
    _, info = _one(O.CP, p, R, s_it, 3, 4, 1 << 3)
    assert info.alarm & O.AL_COUNT


def test_cp_induction_variable_sign_flip_crashes_and_pointer_misalign_crashes():
    p = W.cp_small()
    R = O.profile_ranges(O.CP, p)
    _, info = _one(O.CP, p, R, 14, 9, 3, 1 << 31)   # atomid -> negative -> OOB load (R16)
    assert info.fail & O.FL_CRASH
    _, info = _one(O.CP, p, R, 13, 9, 3, 1 << 2)    # atoms* + 4 B -> misaligned float4 (R16)
    assert info.fail & O.FL_CRASH
    _, info = _one(O.CP, p, R, 14, 9, 3, 1 << 4)    # atomid 3 -> 19: loop repeats -> count mismatch
    assert (info.alarm & O.AL_COUNT) and not info.fail


def test_cp_numatoms_flip_to_small_value_ends_loop_early_and_is_caught_by_checksum():
    p = W.cp_small()
    R = O.profile_ranges(O.CP, p)
    # numatoms (param @live) 37 -> 5 at iteration 2: loop stops at 5 iterations; it == numatoms' holds,
    # but the parameter's exit XOR differs from its entry XOR
    _, info = _one(O.CP, p, R, 10, 0, 2, 1 << 5)
    assert info.alarm & O.AL_CHK and not (info.alarm & O.AL_COUNT)


def test_live_flip_of_loop_invariant_is_caught_by_checksum():
    p = W.cp_small()
    R = O.profile_ranges(O.CP, p)
    _, info = _one(O.CP, p, R, 9, 11, 20, 1 << 12)   # gu @live
    assert info.alarm & O.AL_CHK


def test_hang_model_watchdog():
    p = W.mriq_small()
    R = O.profile_ranges(O.MRIQ, p)
    # k (loop @def) bit 30 set at the last iteration -> k huge -> loop exits (count mismatch)
    _, info = _one(O.MRIQ, p, R, 15, 4, p.n_k - 1, 1 << 30)
    assert info.alarm & O.AL_COUNT and not info.fail
    # numK param bit 30 -> loop runs past numK -> kv OOB -> crash (crash precedes the hang watchdog)
    _, info = _one(O.MRIQ, p, R, 8, 4, 0, 1 << 30)
    assert info.fail & O.FL_CRASH


def test_tpacf_bin_flip_out_of_histogram_crashes():
    p = BENCH_PROBS[O.TPACF]()
    R = O.profile_ranges(O.TPACF, p)
    tr = O.trips(O.TPACF, p)
    g = int(np.nonzero(tr > 3)[0][0])
    _, info = _one(O.TPACF, p, R, 26, g, 1, 1 << 20)  # bin -> huge -> hidx OOB (R16)
    assert info.fail & O.FL_CRASH


# ---------------------------------------------------------------- campaign modes (R22)
@pytest.mark.parametrize("exact", [0, 1])
def test_replay_equals_replica_small_campaign(exact):
    probs = [W.cp_small(), W.mriq_problem(4, 23, n_vox=60), W.tpacf_small(n=60, n_rand=1)]
    R = [O.profile_ranges(b, probs[b], exact=exact) for b in range(3)]
    c1, r1 = O.campaign(-1, probs, R, seed=321, first=0, count=240, exact=exact, mode=1)
    c0, r0 = O.campaign(-1, probs, R, seed=321, first=0, count=240, exact=exact, mode=0)
    assert np.array_equal(c0, c1)
    for k in ("cls", "alarm", "fail", "site", "thread", "inst", "mask"):
        assert np.array_equal(r0[k], r1[k]), k
    assert c1.sum() == 240


def test_phimag_fault_reaches_every_voxel_and_nl_detects_it():
    p = W.mriq_problem(4, 19, n_vox=40, seed=8)
    R = O.profile_ranges(O.MRIQ, p)
    golden = O.run(O.MRIQ, p, flags=O.FT, ranges=R, ndet=1)[0]
    # pm of PhiMag thread 5 (site 32): detected by its duplicate; every voxel's output changes
    (qr, qi), _, info = O.run(O.MRIQ, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(32, 5, 0, 1 << 28))
    assert info.applied and info.alarm & O.AL_DUP
    assert np.count_nonzero(qr != golden[0]) > 0.9 * p.n_vox
    # kidx flipped out of range: modelled crash (R16)
    _, _, info = O.run(O.MRIQ, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(29, 3, 0, 1 << 20))
    assert info.fail & O.FL_CRASH
    # kidx flipped onto another slot: additive kv (R18) -> two k-samples in one slot, one slot empty
    (qr2, _), _, info = O.run(O.MRIQ, p, flags=O.FT, ranges=R, ndet=1, f=O.fault(29, 2, 0, 1 << 0))
    assert not info.fail and info.alarm & O.AL_DUP and not np.array_equal(qr2, golden[0])


def test_phimag_sites_are_replica_only_in_the_oracle_campaign():
    p = W.mriq_problem(4, 19, n_vox=40, seed=8)
    R = [None, O.profile_ranges(O.MRIQ, p), None]
    masks = (O.ALL_SITES, O.MRIQ_PHIMAG_SITES, O.ALL_SITES)
    c1, r1 = O.campaign(O.MRIQ, [None, p, None], R, 99, 0, 60, mode=1, site_masks=masks)
    c0, r0 = O.campaign(O.MRIQ, [None, p, None], R, 99, 0, 60, mode=0, site_masks=masks)
    assert np.array_equal(c0, c1) and set(r1["site"]) <= set(range(29, 36))
    assert (r1["thread"] < p.n_k).all()
