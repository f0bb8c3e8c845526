"""ctypes front-end of the HAUBERK CPU oracle (oracle/hk_oracle.c).

TEST INFRASTRUCTURE — only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` legs may import this module.  It shares no code with the CUDA path
(paper_conf_ipps_yimpski11_b200/); the only common dependency is `workloads` (seeded inputs).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

CP, MRIQ, TPACF = 0, 1, 2
MASKED, DET_MASKED, DETECTED, UNDETECTED, FAILURE = range(5)
CLASS_NAMES = ["masked", "detected_masked", "detected", "undetected", "failure"]
F_NL, F_L, F_PROFILE, F_FI = 1, 2, 4, 8
FT = F_NL | F_L
AL_DUP, AL_CHK, AL_RANGE, AL_COUNT = 1, 2, 4, 8
FL_CRASH, FL_HANG = 1, 2
ALL_SITES = (1 << 64) - 1
MRIQ_PHIMAG_SITES = ((1 << 36) - 1) ^ ((1 << 29) - 1)
DEFAULT_SITE_MASKS = (ALL_SITES, (1 << 29) - 1, ALL_SITES)  # PhiMag sites excluded by default (R22)


class RSet(C.Structure):
    _fields_ = [("n", C.c_int32), ("lo", C.c_float * 3), ("hi", C.c_float * 3), ("t_exp10", C.c_int32)]


class Ranges(C.Structure):
    _fields_ = [("n_det", C.c_int32), ("alpha", C.c_float), ("det", RSet * 8)]


class CPArgs(C.Structure):
    _fields_ = [("atoms", C.c_void_p), ("n_atoms", C.c_int32), ("z0", C.c_float), ("h", C.c_float),
                ("nx", C.c_int32), ("ny", C.c_int32), ("bx", C.c_int32), ("by", C.c_int32), ("unroll", C.c_int32)]


class MRIQArgs(C.Structure):
    _fields_ = [("x", C.c_void_p), ("y", C.c_void_p), ("z", C.c_void_p), ("n_vox", C.c_int32), ("n_k", C.c_int32),
                ("kx", C.c_void_p), ("ky", C.c_void_p), ("kz", C.c_void_p), ("phi_r", C.c_void_p), ("phi_i", C.c_void_p)]


class TPACFArgs(C.Structure):
    _fields_ = [("pts", C.c_void_p), ("edges", C.c_void_p), ("n", C.c_int32), ("n_rand", C.c_int32),
                ("n_bins", C.c_int32)]


class Fault(C.Structure):
    # hang: R17 watchdog factor T of this injection (0 = the paper's 10)
    _fields_ = [("site", C.c_int32), ("hang", C.c_int32), ("thread", C.c_int64), ("inst", C.c_int64), ("mask", C.c_uint64)]


class RunInfo(C.Structure):
    _fields_ = [("alarm", C.c_uint32), ("fail", C.c_uint32), ("domain", C.c_uint32), ("margin", C.c_uint32),
                ("n_alarm_threads", C.c_uint32), ("first_thread", C.c_uint32), ("applied", C.c_int32), ("gap", C.c_float)]


class Record(C.Structure):
    _fields_ = [("index", C.c_int64), ("bench", C.c_int32), ("site", C.c_int32), ("thread", C.c_int64),
                ("inst", C.c_int64), ("mask", C.c_uint64), ("cls", C.c_int32), ("alarm", C.c_uint32),
                ("fail", C.c_uint32), ("domain", C.c_uint32), ("margin", C.c_uint32), ("worst", C.c_float),
                ("gap", C.c_float), ("pad", C.c_int32)]


RECORD_DTYPE = np.dtype([("index", "<i8"), ("bench", "<i4"), ("site", "<i4"), ("thread", "<i8"), ("inst", "<i8"),
                         ("mask", "<u8"), ("cls", "<i4"), ("alarm", "<u4"), ("fail", "<u4"), ("domain", "<u4"),
                         ("margin", "<u4"), ("worst", "<f4"), ("gap", "<f4"), ("pad", "<i4")], align=True)
assert RECORD_DTYPE.itemsize == C.sizeof(Record)


def build(force: bool = False) -> str:
    """Compile liboracle.so with the oracle Makefile (plain gcc)."""
    with _lock:
        src = os.path.join(_HERE, "hk_oracle.c")
        if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            subprocess.check_call(["make", "-s", "-B", "-C", _HERE, "liboracle.so"])
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB_PATH)
        P = C.c_void_p
        L.ora_ord.restype = C.c_int64; L.ora_ord.argtypes = [C.c_float]
        L.ora_splitmix.restype = C.c_uint64; L.ora_splitmix.argtypes = [C.c_uint64, C.c_uint64]
        L.ora_bounded.restype = C.c_uint64; L.ora_bounded.argtypes = [C.c_uint64, C.c_uint64]
        for f in ("ora_rsqrt", "ora_sin", "ora_cos"):
            getattr(L, f).restype = C.c_float; getattr(L, f).argtypes = [C.c_float, C.c_int32]
        L.ora_cp_run.restype = C.c_int
        L.ora_cp_run.argtypes = [P, C.c_int32, C.c_int32, P, C.c_int32, P, P, P, P]
        L.ora_mriq_run.restype = C.c_int
        L.ora_mriq_run.argtypes = [P, C.c_int32, C.c_int32, P, C.c_int32, P, P, P, P, P]
        L.ora_tpacf_run.restype = C.c_int
        L.ora_tpacf_run.argtypes = [P, C.c_int32, P, C.c_int32, P, P, P, P]
        L.ora_tpacf_trips.restype = C.c_int64; L.ora_tpacf_trips.argtypes = [P, C.c_int64]
        L.ora_tpacf_threads.restype = C.c_int64; L.ora_tpacf_threads.argtypes = [P]
        L.ora_cp_threads.restype = C.c_int64; L.ora_cp_threads.argtypes = [P]
        L.ora_cp_threads_out.restype = C.c_int; L.ora_cp_threads_out.argtypes = [P, C.c_int32, P, C.c_int64, P, P]
        L.ora_mriq_threads_out.restype = C.c_int; L.ora_mriq_threads_out.argtypes = [P, C.c_int32, P, C.c_int64, P, P]
        L.ora_cp_reference_f64.restype = None; L.ora_cp_reference_f64.argtypes = [P, P, P]
        L.ora_mriq_reference_f64.restype = None; L.ora_mriq_reference_f64.argtypes = [P, P, P, P]
        L.ora_threshold.restype = C.c_float; L.ora_threshold.argtypes = [C.c_int32]
        L.ora_profile_cost.restype = C.c_int64; L.ora_profile_cost.argtypes = [P, P, C.c_int64, C.c_int32]
        L.ora_profile.restype = C.c_int; L.ora_profile.argtypes = [P, P, C.c_int64, C.c_int32, P]
        L.ora_fp_wrong.restype = C.c_int; L.ora_fp_wrong.argtypes = [P, P, C.c_int64, C.c_float, P]
        L.ora_max_abs.restype = C.c_float; L.ora_max_abs.argtypes = [P, C.c_int64]
        L.ora_tpacf_outputs.restype = None; L.ora_tpacf_outputs.argtypes = [P, C.c_int32, C.c_int32, P]
        L.ora_tpacf_wrong.restype = C.c_int; L.ora_tpacf_wrong.argtypes = [P, P, C.c_int32, C.c_int32, P]
        L.ora_classify.restype = C.c_int32; L.ora_classify.argtypes = [C.c_int32, C.c_uint32, C.c_uint32]
        L.ora_nsites.restype = C.c_int32; L.ora_nsites.argtypes = [C.c_int32, C.c_int32]
        L.ora_site_info.restype = None; L.ora_site_info.argtypes = [C.c_int32, C.c_int32, C.c_int32, P, P]
        L.ora_decode.restype = C.c_int
        L.ora_decode.argtypes = [C.c_int32, P, P, C.c_uint64, C.c_int32, C.c_int32, C.c_int64, C.c_int64, P, P]
        L.ora_campaign.restype = C.c_int
        L.ora_campaign.argtypes = [C.c_int32, P, P, P, C.c_uint64, C.c_int32, C.c_int64, C.c_int64, C.c_int32, C.c_int32,
                                   C.c_int32, C.c_int32, P, P]
        L.ora_detector_site.restype = C.c_int32; L.ora_detector_site.argtypes = [C.c_int32, C.c_int32, C.c_int32]
        L.ora_a6_count.restype = C.c_int32; L.ora_a6_count.argtypes = [C.c_int32, P, C.c_int32, P, P, P, C.c_int32]
        L.ora_a6_select.restype = C.c_int32; L.ora_a6_select.argtypes = [C.c_int32, P, P, C.c_int32, P, P, C.c_int32, P]
        L.ora_in_range.restype = C.c_int32; L.ora_in_range.argtypes = [P, C.c_int32, C.c_float]
        L.ora_extend_ranges.restype = C.c_int32; L.ora_extend_ranges.argtypes = [P, P, C.c_int32]
        L.ora_alpha_step.restype = C.c_float; L.ora_alpha_step.argtypes = [C.c_float, C.c_double, C.c_double, C.c_double]
        L.ora_diagnose.restype = C.c_int32; L.ora_diagnose.argtypes = [C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, C.c_int32]
        L.ora_coverage.restype = C.c_int32; L.ora_coverage.argtypes = [P, P]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


# ------------------------------------------------------------------------------------------------
# argument marshalling (keeps numpy arrays alive by attaching them to the struct)
# ------------------------------------------------------------------------------------------------
def cp_args(p) -> CPArgs:
    atoms = np.ascontiguousarray(p.atoms, dtype=np.float32)
    a = CPArgs(_p(atoms), p.n_atoms, p.z0, p.h, p.nx, p.ny, p.bx, p.by, p.unroll)
    a._keep = atoms
    return a


def mriq_args(p) -> MRIQArgs:
    arrs = [np.ascontiguousarray(v, dtype=np.float32) for v in (p.x, p.y, p.z, p.kx, p.ky, p.kz, p.phi_r, p.phi_i)]
    a = MRIQArgs(_p(arrs[0]), _p(arrs[1]), _p(arrs[2]), p.n_vox, p.n_k, *[_p(v) for v in arrs[3:]])
    a._keep = arrs
    return a


def tpacf_args(p) -> TPACFArgs:
    pts = np.ascontiguousarray(p.pts, dtype=np.float32)
    edges = np.ascontiguousarray(p.edges, dtype=np.float32)
    a = TPACFArgs(_p(pts), _p(edges), p.n, p.n_rand, p.n_bins)
    a._keep = (pts, edges)
    return a


def make_args(bench: int, p):
    return (cp_args, mriq_args, tpacf_args)[bench](p)


def fault(site: int, thread: int, inst: int, mask: int, hang: int = 0) -> Fault:
    return Fault(site, hang, thread, inst, mask)


# ------------------------------------------------------------------------------------------------
# runs
# ------------------------------------------------------------------------------------------------
def n_threads(bench: int, p) -> int:
    if bench == CP:
        return (p.nx // p.unroll) * p.ny
    if bench == MRIQ:
        return p.n_vox
    return int(lib().ora_tpacf_threads(C.byref(tpacf_args(p))))


def run(bench: int, p, flags: int = FT, exact: int = 0, ranges: Ranges | None = None, ndet: int = 0,
        f: Fault | None = None):
    """One full program run (all abstract threads).  Returns (output, samples, RunInfo).

    output: CP float32 [ny, nx]; MRI-Q (qr, qi); TPACF int64 [nh, n_bins + 2]."""
    L = lib()
    R = ranges if ranges is not None else Ranges()
    info = RunInfo()
    nthr = n_threads(bench, p)
    samples = np.full(max(ndet, 1) * max(nthr, 1), np.nan, dtype=np.float32)
    fp = C.byref(f) if f is not None else None
    if bench == CP:
        a = cp_args(p)
        out = np.zeros((p.ny, p.nx), dtype=np.float32)
        rc = L.ora_cp_run(C.byref(a), flags, exact, C.byref(R), ndet, fp, _p(out), _p(samples), C.byref(info))
    elif bench == MRIQ:
        a = mriq_args(p)
        qr = np.zeros(p.n_vox, dtype=np.float32); qi = np.zeros(p.n_vox, dtype=np.float32)
        rc = L.ora_mriq_run(C.byref(a), flags, exact, C.byref(R), ndet, fp, _p(qr), _p(qi), _p(samples), C.byref(info))
        out = (qr, qi)
    else:
        a = tpacf_args(p)
        out = np.zeros((1 + 2 * p.n_rand, p.n_bins + 2), dtype=np.int64)
        rc = L.ora_tpacf_run(C.byref(a), flags, C.byref(R), ndet, fp, _p(out), _p(samples), C.byref(info))
    if rc != 0:
        raise ValueError(f"oracle run rejected the arguments (rc={rc})")
    return out, samples[: ndet * nthr].reshape(ndet, nthr) if ndet else samples[:0], info


def trips(bench: int, p) -> np.ndarray:
    """Golden trip count per abstract thread."""
    if bench == CP:
        return np.full(n_threads(CP, p), p.n_atoms, dtype=np.int64)
    if bench == MRIQ:
        return np.full(p.n_vox, p.n_k, dtype=np.int64)
    a = tpacf_args(p)
    L = lib()
    return np.array([L.ora_tpacf_trips(C.byref(a), g) for g in range(n_threads(TPACF, p))], dtype=np.int64)


def profile_samples(samples: np.ndarray, valid: np.ndarray | None = None, t0_exp10: int = -5) -> RSet:
    s = np.ascontiguousarray(samples, dtype=np.float32)
    v = None if valid is None else np.ascontiguousarray(valid, dtype=np.uint8)
    out = RSet()
    rc = lib().ora_profile(_p(s), None if v is None else _p(v), s.size, t0_exp10, C.byref(out))
    if rc != 0:
        raise FloatingPointError("profile samples contain NaN/Inf (HK_ERR_PROFILE_NAN)")
    return out


def profile_cost(samples: np.ndarray, k: int, valid: np.ndarray | None = None) -> int:
    s = np.ascontiguousarray(samples, dtype=np.float32)
    v = None if valid is None else np.ascontiguousarray(valid, dtype=np.uint8)
    return int(lib().ora_profile_cost(_p(s), None if v is None else _p(v), s.size, k))


def profile_ranges(bench: int, p, maxvar: int = 1, t0_exp10: int = -5, alpha: float = 1.0, exact: int = 0) -> Ranges:
    """PROFILE run + threshold search per detector (hauberk_profile_ranges' oracle twin)."""
    out, samples, _ = run(bench, p, flags=F_PROFILE, exact=exact, ndet=maxvar)
    valid = (trips(bench, p) > 0).astype(np.uint8)
    R = Ranges()
    R.n_det = maxvar
    R.alpha = alpha
    for d in range(maxvar):
        R.det[d] = profile_samples(samples[d], valid, t0_exp10)
    return R


def ranges_to_list(R: Ranges):
    return [(R.det[d].t_exp10, [(R.det[d].lo[r], R.det[d].hi[r]) for r in range(R.det[d].n)]) for d in range(R.n_det)]


def campaign(bench_mode: int, problems, ranges, seed: int, first: int, count: int, exact: int = 0,
             mode: int = 1, site_masks=DEFAULT_SITE_MASKS, records: bool = True, nbits: int = 1,
             variant: int = 0, hang_factor: int = 0):
    """Seeded campaign.  problems/ranges: 3-lists indexed by bench (None where unused).
    mode 1 = replay, 0 = replica; variant 0 = FI&FT binary, 1 = FI-only binary (original program's
    sites, no detectors); hang_factor = R17's T (0 = 10).
    Returns (counts int64[3,5], records structured array)."""
    L = lib()
    argv = [make_args(b, problems[b]) if problems[b] is not None else None for b in range(3)]
    aptr = (C.c_void_p * 3)(*[C.cast(C.byref(a), C.c_void_p) if a is not None else None for a in argv])
    rng = [ranges[b] if ranges[b] is not None else Ranges() for b in range(3)]
    rptr = (C.c_void_p * 3)(*[C.cast(C.byref(r), C.c_void_p) for r in rng])
    masks = (C.c_uint64 * 3)(*site_masks)
    counts = np.zeros((3, 5), dtype=np.int64)
    recs = np.zeros(count, dtype=RECORD_DTYPE) if records else None
    rc = L.ora_campaign(bench_mode, aptr, rptr, masks, seed, nbits, first, count, exact, mode, variant, hang_factor,
                        _p(recs) if records else None, _p(counts))
    if rc != 0:
        raise RuntimeError(f"oracle campaign failed rc={rc} (1 = bad args/empty catalogue, 2 = fault-free alarm)")
    return counts, recs


def decode(bench_mode: int, problems, seed: int, first: int, count: int, site_masks=DEFAULT_SITE_MASKS, nbits: int = 1,
           variant: int = 0):
    L = lib()
    argv = [make_args(b, problems[b]) if problems[b] is not None else None for b in range(3)]
    aptr = (C.c_void_p * 3)(*[C.cast(C.byref(a), C.c_void_p) if a is not None else None for a in argv])
    masks = (C.c_uint64 * 3)(*site_masks)
    benches = np.zeros(count, dtype=np.int32)
    faults = (Fault * count)()
    rc = L.ora_decode(bench_mode, aptr, masks, seed, nbits, variant, first, count, _p(benches), C.cast(faults, C.c_void_p))
    if rc != 0:
        raise RuntimeError("decode failed")
    return benches, [(f.site, f.thread, f.inst, f.mask) for f in faults]


def site_info(bench: int, unroll: int, site: int):
    c, w = C.c_int32(), C.c_int32()
    lib().ora_site_info(bench, unroll, site, C.byref(c), C.byref(w))
    return c.value, w.value


def nsites(bench: int, unroll: int = 4) -> int:
    return int(lib().ora_nsites(bench, unroll))


def reference_f64(bench: int, p):
    """Plain double-precision definitions: CP E(p) = sum q/|p-a|; MRI-Q Q(x) = sum |phi|^2 e^{i 2pi k.x}.
    Returns (value(s), mass) where mass = sum |term| (R21 cancellation scale)."""
    L = lib()
    if bench == CP:
        a = cp_args(p)
        out = np.zeros((p.ny, p.nx)); mass = np.zeros((p.ny, p.nx))
        L.ora_cp_reference_f64(C.byref(a), _p(out), _p(mass))
        return out, mass
    a = mriq_args(p)
    qr = np.zeros(p.n_vox); qi = np.zeros(p.n_vox); mass = np.zeros(p.n_vox)
    L.ora_mriq_reference_f64(C.byref(a), _p(qr), _p(qi), _p(mass))
    return (qr, qi), mass


def threads_out(bench: int, p, tids, exact: int = 0):
    """Outputs of selected abstract threads only (sampled parity at full sizes).
    CP: (flat grid indices [n, U], values [n, U]); MRI-Q: (qr [n], qi [n])."""
    t = np.ascontiguousarray(np.asarray(tids, dtype=np.int64))
    L = lib()
    if bench == CP:
        a = cp_args(p)
        idx = np.zeros((t.size, p.unroll), dtype=np.int64); val = np.zeros((t.size, p.unroll), dtype=np.float32)
        assert L.ora_cp_threads_out(C.byref(a), exact, _p(t), t.size, _p(idx), _p(val)) == 0
        return idx, val
    a = mriq_args(p)
    qr = np.zeros(t.size, dtype=np.float32); qi = np.zeros(t.size, dtype=np.float32)
    assert L.ora_mriq_threads_out(C.byref(a), exact, _p(t), t.size, _p(qr), _p(qi)) == 0
    return qr, qi


def detector_site(bench: int, site: int, unroll: int = 4) -> bool:
    """True for sites that exist only because of HAUBERK (absent from the FI-only binary)."""
    return bool(lib().ora_detector_site(bench, unroll, site))


# ------------------------------------------------------------------------------------------------
# A6 selection, recovery and evaluation arithmetic
# ------------------------------------------------------------------------------------------------
A6_VAR, A6_TEMP, A6_LOAD, A6_CONST, A6_NLPROT, A6_ACCOP, A6_IND = range(7)


def _graph(kinds, edges):
    k = np.ascontiguousarray(np.asarray(kinds, dtype=np.int32))
    e = np.asarray(edges, dtype=np.int32).reshape(-1, 2)
    return k, np.ascontiguousarray(e[:, 0]), np.ascontiguousarray(e[:, 1])


def a6_count(kinds, edges, v: int, removed=None) -> int:
    k, s, d = _graph(kinds, edges)
    rm = None if removed is None else np.ascontiguousarray(np.asarray(removed, dtype=np.uint8))
    return int(lib().ora_a6_count(k.size, _p(k), s.size, _p(s), _p(d), None if rm is None else _p(rm), v))


def a6_select(kinds, selfacc, edges, maxvar: int):
    k, s, d = _graph(kinds, edges)
    sa = np.ascontiguousarray(np.asarray(selfacc, dtype=np.uint8))
    out = np.zeros(max(maxvar, 1), dtype=np.int32)
    got = lib().ora_a6_select(k.size, _p(k), _p(sa), s.size, _p(s), _p(d), maxvar, _p(out))
    return out[:got].tolist()


def in_range(R: Ranges, d: int, v: float) -> bool:
    return bool(lib().ora_in_range(C.byref(R), d, v))


def extend_ranges(rs: RSet, values) -> int:
    v = np.ascontiguousarray(np.asarray(values, dtype=np.float32))
    return int(lib().ora_extend_ranges(C.byref(rs), _p(v), v.size))


def alpha_step(alpha: float, fp_ratio: float, hi: float = 0.10, lo: float = 0.05) -> float:
    return float(lib().ora_alpha_step(alpha, fp_ratio, hi, lo))


DIAG_NAMES = ["ok", "false_alarm", "transient", "persistent", "failed"]


def diagnose(alarm1: int, fail1: int, alarm2: int, fail2: int, identical: bool) -> str:
    return DIAG_NAMES[lib().ora_diagnose(alarm1, fail1, alarm2, fail2, 1 if identical else 0)]


def coverage(counts) -> dict:
    """{coverage, sdc, detected, failure} of int64 counts [.., 5] summed over benchmarks."""
    c = np.ascontiguousarray(np.asarray(counts, dtype=np.int64).reshape(-1, 5).sum(0))
    out = np.zeros(4)
    lib().ora_coverage(_p(c), _p(out))
    return dict(zip(("coverage", "sdc", "detected", "failure"), out.tolist()))
