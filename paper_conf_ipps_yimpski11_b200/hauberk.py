"""Thin ctypes binding of libhauberk.so (include/hauberk.h) — argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels; PyTorch only owns device memory,
the stream and (in parallel.py) the process group.  There is no CPU fallback: if the library or a
CUDA device is missing, the calls raise.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
# HAUBERK_LIB: another build of the same library (A/B timing of two builds on one box)
LIB_PATH = os.environ.get("HAUBERK_LIB") or os.path.join(_HERE, "libhauberk.so")

HK_CP, HK_MRIQ, HK_TPACF, HK_MIXED = 0, 1, 2, -1
HK_BASE, HK_FT, HK_FT_NL, HK_FT_L, HK_PROFILE = 0, 1, 2, 3, 4
HK_ALARM_DUP, HK_ALARM_CHECKSUM, HK_ALARM_RANGE, HK_ALARM_COUNT = 1, 2, 4, 8  # hk_control.alarm bits
CLASS_NAMES = ["masked", "detected_masked", "detected", "undetected", "failure"]
BENCH_NAMES = ["cp", "mriq", "tpacf"]
ALL_SITES = (1 << 64) - 1
MRIQ_PHIMAG_SITES = ((1 << 36) - 1) ^ ((1 << 29) - 1)  # sites 29-35: PhiMag (replica mode only, R22)
# default campaign masks: every site except MRI-Q's PhiMag sites
DEFAULT_SITE_MASKS = (ALL_SITES, (1 << 29) - 1, ALL_SITES)


class HauberkError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        super().__init__(f"{where}: status {status} ({detail})")
        self.status = status


class RangeSet(C.Structure):
    _fields_ = [("n", C.c_int32), ("lo", C.c_float * 3), ("hi", C.c_float * 3), ("t_exp10", C.c_int32)]


class Ranges(C.Structure):
    _fields_ = [("n_det", C.c_int32), ("alpha", C.c_float), ("det", RangeSet * 8)]

    def as_list(self):
        return [(self.det[d].t_exp10, [(self.det[d].lo[r], self.det[d].hi[r]) for r in range(self.det[d].n)])
                for d in range(self.n_det)]


class Control(C.Structure):
    _fields_ = [("alarm", C.c_uint32), ("fail", C.c_uint32), ("n_alarm_warps", C.c_uint32), ("first_thread", C.c_uint32),
                ("outlier_min_ord", C.c_int32 * 8), ("outlier_max_ord", C.c_int32 * 8), ("fault_applied", C.c_uint32),
                ("check_margin", C.c_uint32), ("domain", C.c_uint32), ("check_gap", C.c_float)]


CONTROL_BYTES = C.sizeof(Control)  # 96


class CPArgs(C.Structure):
    _fields_ = [("atoms", C.c_void_p), ("atoms_ws", C.c_void_p), ("n_atoms", C.c_int32), ("z0", C.c_float),
                ("h", C.c_float), ("nx", C.c_int32), ("ny", C.c_int32), ("bx", C.c_int32), ("by", C.c_int32),
                ("unroll", C.c_int32), ("grid", C.c_void_p), ("exact", C.c_int32)]


class MRIQArgs(C.Structure):
    _fields_ = [("x", C.c_void_p), ("y", C.c_void_p), ("z", C.c_void_p), ("n_vox", C.c_int32), ("n_k", C.c_int32),
                ("kx", C.c_void_p), ("ky", C.c_void_p), ("kz", C.c_void_p), ("phi_r", C.c_void_p), ("phi_i", C.c_void_p),
                ("kv_ws", C.c_void_p), ("qr", C.c_void_p), ("qi", C.c_void_p), ("exact", C.c_int32)]


class TPACFArgs(C.Structure):
    _fields_ = [("pts", C.c_void_p), ("edges", C.c_void_p), ("n", C.c_int32), ("n_rand", C.c_int32),
                ("n_bins", C.c_int32), ("hist", C.c_void_p)]


class ProfileOpts(C.Structure):
    _fields_ = [("maxvar", C.c_int32), ("t0_exp10", C.c_int32), ("alpha", C.c_float)]


class Campaign(C.Structure):
    _fields_ = [("seed", C.c_uint64), ("first", C.c_int64), ("count", C.c_int64), ("nbits", C.c_int32),
                ("mode", C.c_int32), ("batch", C.c_int32), ("exact", C.c_int32), ("site_mask", C.c_uint64 * 3),
                ("variant", C.c_int32), ("hang_factor", C.c_int32)]


HK_FIFT, HK_FI_ONLY = 0, 1  # hk_campaign.variant: FI&FT binary / FI-only binary (row a7)


class Fault(C.Structure):
    _fields_ = [("site", C.c_int32), ("hang", C.c_int32), ("thread", C.c_int64), ("inst", C.c_int64), ("mask", C.c_uint64)]


class Summary(C.Structure):
    _fields_ = [("coverage", C.c_double), ("sdc", C.c_double), ("detected", C.c_double), ("failure", C.c_double),
                ("total", C.c_int64)]


OUTCOME_DTYPE = np.dtype([("index", "<i8"), ("bench", "<i4"), ("site", "<i4"), ("thread", "<i8"), ("inst", "<i8"),
                          ("mask", "<u8"), ("cls", "<i4"), ("alarm", "<u4"), ("fail", "<u4"), ("domain", "<u4"),
                          ("margin", "<u4"), ("worst", "<f4"), ("gap", "<f4"), ("pad2", "<i4")], align=True)

_lib = None


def lib():
    """Load libhauberk.so (built by `python -c "import __graft_entry__ as g; g.build()"`)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build the CUDA extension first (__graft_entry__.build())")
        L = C.CDLL(LIB_PATH)
        P, I32, I64, U64 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64
        for name in ("hauberk_run_cp", "hauberk_run_mriq", "hauberk_run_tpacf"):
            f = getattr(L, name)
            f.restype = I32
            f.argtypes = [P, I32, P, P, P, P]
        L.hauberk_profile_ranges.restype = I32
        L.hauberk_profile_ranges.argtypes = [I32, P, P, P, P]
        L.hauberk_inject_campaign.restype = I32
        L.hauberk_inject_campaign.argtypes = [I32, P, P, P, P, P, P, P]
        L.hauberk_decode.restype = I32
        L.hauberk_decode.argtypes = [I32, P, P, U64, I32, I32, I64, I64, P, P]
        L.hauberk_num_sites.restype = I32
        L.hauberk_num_sites.argtypes = [I32, I32]
        L.hauberk_strerror.restype = C.c_char_p
        L.hauberk_strerror.argtypes = [I32]
        L.hauberk_last_error.restype = C.c_char_p
        L.hauberk_last_error.argtypes = []
        L.hauberk_version.restype = I32
        L.hauberk_launch_count.restype = U64
        L.hauberk_campaign_create.restype = I32
        L.hauberk_campaign_create.argtypes = [I32, P, P, P, P, P]
        L.hauberk_campaign_run.restype = I32
        L.hauberk_campaign_run.argtypes = [P, I64, I64, P, P, P]
        L.hauberk_campaign_destroy.restype = None
        L.hauberk_campaign_destroy.argtypes = [P]
        L.hauberk_profile_search.restype = I32
        L.hauberk_profile_search.argtypes = [P, I64, I32, P]
        L.hauberk_timing_enable.restype = None
        L.hauberk_timing_enable.argtypes = [I32]
        L.hauberk_timing_read.restype = I32
        L.hauberk_timing_read.argtypes = [I32, I32, P, P, P]
        L.hauberk_part_units.restype = I32
        L.hauberk_part_units.argtypes = [I32, P, P, P]
        L.hauberk_compare.restype = I32
        L.hauberk_compare.argtypes = [P, P, I64, P, P]
        L.hauberk_run_part.restype = I32
        L.hauberk_run_part.argtypes = [I32, P, I32, P, P, I64, I64, P]
        L.hauberk_detector_site.restype = I32
        L.hauberk_detector_site.argtypes = [I32, I32, I32]
        L.hauberk_campaign_workspace_bytes.restype = C.c_size_t
        L.hauberk_campaign_workspace_bytes.argtypes = [I32, P, P]
        L.hauberk_summarize.restype = I32
        L.hauberk_summarize.argtypes = [P, P]
        L.hauberk_extend_ranges.restype = I32
        L.hauberk_extend_ranges.argtypes = [P, P, I32, P]
        L.hauberk_outliers.restype = I32
        L.hauberk_outliers.argtypes = [P, I32, P, P]
        L.hauberk_alpha_update.restype = C.c_float
        L.hauberk_alpha_update.argtypes = [C.c_float, C.c_double, C.c_double, C.c_double]
        L.hauberk_diagnose.restype = I32
        L.hauberk_diagnose.argtypes = [C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, I32]
        L.hauberk_release_caches.restype = None
        L.hauberk_release_caches.argtypes = []
        _lib = L
    return _lib


EXPORTED = ["hauberk_run_cp", "hauberk_run_mriq", "hauberk_run_tpacf", "hauberk_profile_ranges",
            "hauberk_inject_campaign", "hauberk_decode", "hauberk_num_sites", "hauberk_strerror",
            "hauberk_last_error", "hauberk_version", "hauberk_launch_count", "hauberk_timing_enable",
            "hauberk_timing_read", "hauberk_campaign_create", "hauberk_campaign_run", "hauberk_campaign_destroy",
            "hauberk_profile_search", "hauberk_part_units", "hauberk_run_part", "hauberk_compare",
            "hauberk_detector_site", "hauberk_campaign_workspace_bytes", "hauberk_summarize", "hauberk_extend_ranges",
            "hauberk_outliers", "hauberk_alpha_update", "hauberk_diagnose", "hauberk_release_caches"]


def _check(status: int, where: str):
    if status != 0:
        L = lib()
        raise HauberkError(status, where, f"{L.hauberk_strerror(status).decode()}; {L.hauberk_last_error().decode()}")


def _stream(stream=None) -> C.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def _ptr(t: torch.Tensor | None):
    if t is None:
        return None
    if not t.is_cuda:
        raise ValueError("device tensor expected")
    if not t.is_contiguous():
        raise ValueError("contiguous tensor expected")
    return C.c_void_p(t.data_ptr())


def launch_count() -> int:
    return int(lib().hauberk_launch_count())


def timing_enable(on: bool = True):
    lib().hauberk_timing_enable(1 if on else 0)


def timing_read(bench: int, cls: int):
    """(device ms, launches, pairs) of the main (cls 0) or FI replica (cls 1) kernels since the last read."""
    ms, n, w = C.c_double(), C.c_int64(), C.c_double()
    _check(lib().hauberk_timing_read(bench, cls, C.byref(ms), C.byref(n), C.byref(w)), "hauberk_timing_read")
    return ms.value, n.value, w.value


def version() -> int:
    return int(lib().hauberk_version())


def num_sites(bench: int, unroll: int = 4) -> int:
    return int(lib().hauberk_num_sites(bench, unroll))


# ------------------------------------------------------------------------------------------------
# Device-resident benchmark inputs/outputs (torch tensors) and their ABI argument structs
# ------------------------------------------------------------------------------------------------
def _dev(a: np.ndarray, device) -> torch.Tensor:
    return torch.from_numpy(np.ascontiguousarray(a)).to(device)


@dataclass
class CPDevice:
    atoms: torch.Tensor
    atoms_ws: torch.Tensor
    grid: torch.Tensor
    n_atoms: int
    z0: float
    h: float
    nx: int
    ny: int
    bx: int
    by: int
    unroll: int
    exact: int = 0
    bench = HK_CP

    @classmethod
    def from_problem(cls, p, device="cuda", exact: int = 0):
        n = max(p.n_atoms, 1)
        atoms = torch.zeros((n, 4), dtype=torch.float32, device=device)
        if p.n_atoms:
            atoms[: p.n_atoms] = _dev(p.atoms.astype(np.float32), device)
        return cls(atoms=atoms, atoms_ws=torch.empty((n, 4), dtype=torch.float32, device=device),
                   grid=torch.empty((p.ny, p.nx), dtype=torch.float32, device=device), n_atoms=p.n_atoms, z0=p.z0,
                   h=p.h, nx=p.nx, ny=p.ny, bx=p.bx, by=p.by, unroll=p.unroll, exact=exact)

    def args(self) -> CPArgs:
        return CPArgs(_ptr(self.atoms), _ptr(self.atoms_ws), self.n_atoms, self.z0, self.h, self.nx, self.ny, self.bx,
                      self.by, self.unroll, _ptr(self.grid), self.exact)

    @property
    def n_threads(self) -> int:
        return (self.nx // self.unroll) * self.ny

    def output(self):
        return self.grid


@dataclass
class MRIQDevice:
    x: torch.Tensor
    y: torch.Tensor
    z: torch.Tensor
    kx: torch.Tensor
    ky: torch.Tensor
    kz: torch.Tensor
    phi_r: torch.Tensor
    phi_i: torch.Tensor
    kv_ws: torch.Tensor
    qr: torch.Tensor
    qi: torch.Tensor
    exact: int = 0
    bench = HK_MRIQ

    @classmethod
    def from_problem(cls, p, device="cuda", exact: int = 0):
        d = lambda a: _dev(a.astype(np.float32), device)
        nk = max(p.n_k, 1)
        return cls(x=d(p.x), y=d(p.y), z=d(p.z), kx=d(p.kx), ky=d(p.ky), kz=d(p.kz), phi_r=d(p.phi_r),
                   phi_i=d(p.phi_i), kv_ws=torch.empty((nk, 4), dtype=torch.float32, device=device),
                   qr=torch.empty(p.n_vox, dtype=torch.float32, device=device),
                   qi=torch.empty(p.n_vox, dtype=torch.float32, device=device), exact=exact)

    @property
    def n_vox(self) -> int:
        return int(self.x.numel())

    @property
    def n_k(self) -> int:
        return int(self.kx.numel())

    def args(self) -> MRIQArgs:
        return MRIQArgs(_ptr(self.x), _ptr(self.y), _ptr(self.z), self.n_vox, self.n_k, _ptr(self.kx), _ptr(self.ky),
                        _ptr(self.kz), _ptr(self.phi_r), _ptr(self.phi_i), _ptr(self.kv_ws), _ptr(self.qr),
                        _ptr(self.qi), self.exact)

    @property
    def n_threads(self) -> int:
        return self.n_vox

    def output(self):
        return (self.qr, self.qi)


@dataclass
class TPACFDevice:
    pts: torch.Tensor
    edges: torch.Tensor
    hist: torch.Tensor
    n: int
    n_rand: int
    n_bins: int
    bench = HK_TPACF

    @classmethod
    def from_problem(cls, p, device="cuda", exact: int = 0):
        return cls(pts=_dev(p.pts.astype(np.float32), device), edges=_dev(p.edges.astype(np.float32), device),
                   hist=torch.empty((1 + 2 * p.n_rand, p.n_bins + 2), dtype=torch.int64, device=device),
                   n=p.n, n_rand=p.n_rand, n_bins=p.n_bins)

    def args(self) -> TPACFArgs:
        return TPACFArgs(_ptr(self.pts), _ptr(self.edges), self.n, self.n_rand, self.n_bins, _ptr(self.hist))

    @property
    def n_threads(self) -> int:
        return (1 + 2 * self.n_rand) * self.n  # abstract thread g = h * n + i

    def output(self):
        return self.hist


_RUN = {HK_CP: "hauberk_run_cp", HK_MRIQ: "hauberk_run_mriq", HK_TPACF: "hauberk_run_tpacf"}


def new_control(device="cuda") -> torch.Tensor:
    return torch.zeros(CONTROL_BYTES // 4, dtype=torch.int32, device=device)


def read_control(cb: torch.Tensor) -> Control:
    raw = cb.cpu().numpy().tobytes()
    return Control.from_buffer_copy(raw)


def run(dev, variant: int = HK_FT, ranges: Ranges | None = None, cb: torch.Tensor | None = None,
        samples: torch.Tensor | None = None, stream=None):
    """hauberk_run_{cp,mriq,tpacf}: stream-asynchronous; outputs land in dev.output()."""
    a = dev.args()
    f = getattr(lib(), _RUN[dev.bench])
    st = f(C.byref(a), variant, C.byref(ranges) if ranges is not None else None, _ptr(cb), _ptr(samples), _stream(stream))
    _check(st, _RUN[dev.bench])


def compare(a: torch.Tensor, b: torch.Tensor, cb: torch.Tensor, stream=None):
    """hauberk_compare (R-Naive's compare step): bitwise compare of two equally sized buffers."""
    assert a.numel() * a.element_size() == b.numel() * b.element_size() and (a.numel() * a.element_size()) % 4 == 0
    _check(lib().hauberk_compare(_ptr(a), _ptr(b), a.numel() * a.element_size() // 4, _ptr(cb), _stream(stream)),
           "hauberk_compare")


def part_units(dev) -> tuple[int, int]:
    """hauberk_part_units: (number of partition units, alignment granule) of a single run."""
    a = dev.args()
    u, g = C.c_int64(0), C.c_int64(0)
    _check(lib().hauberk_part_units(dev.bench, C.byref(a), C.byref(u), C.byref(g)), "hauberk_part_units")
    return int(u.value), int(g.value)


def run_part(dev, begin: int, end: int, variant: int = HK_FT, ranges: Ranges | None = None,
             cb: torch.Tensor | None = None, stream=None):
    """hauberk_run_part: partition units [begin, end) of one single run (stream-asynchronous)."""
    a = dev.args()
    st = lib().hauberk_run_part(dev.bench, C.byref(a), variant, C.byref(ranges) if ranges is not None else None,
                                _ptr(cb), begin, end, _stream(stream))
    _check(st, "hauberk_run_part")


def profile_ranges(dev, maxvar: int = 1, t0_exp10: int = -5, alpha: float = 1.0, stream=None) -> Ranges:
    """hauberk_profile_ranges: PROFILE run + threshold search (synchronises the stream)."""
    a = dev.args()
    out = Ranges()
    opts = ProfileOpts(maxvar, t0_exp10, alpha)
    st = lib().hauberk_profile_ranges(dev.bench, C.byref(a), C.byref(opts), C.byref(out), _stream(stream))
    _check(st, "hauberk_profile_ranges")
    return out


def profile_search(samples: np.ndarray, t0_exp10: int = -5) -> RangeSet:
    """hauberk_profile_search on host samples (float32)."""
    s = np.ascontiguousarray(samples, dtype=np.float32)
    out = RangeSet()
    st = lib().hauberk_profile_search(s.ctypes.data_as(C.c_void_p), s.size, t0_exp10, C.byref(out))
    _check(st, "hauberk_profile_search")
    return out


def profile_samples(dev, maxvar: int = 1, stream=None) -> torch.Tensor:
    """PROFILE run (hauberk_run_* with HK_PROFILE): per-thread acc/it samples [maxvar, threads] on
    the device (threads with zero trips keep NaN)."""
    samples = torch.full((maxvar, dev.n_threads), float("nan"), dtype=torch.float32, device=dev.output()[0].device
                         if isinstance(dev.output(), tuple) else dev.output().device)
    R = Ranges()
    R.n_det = maxvar
    R.alpha = 1.0
    cb = new_control(samples.device)
    run(dev, HK_PROFILE, R, cb, samples, stream)
    return samples


def _arg_array(devs):
    structs = [d.args() if d is not None else None for d in devs]
    arr = (C.c_void_p * 3)(*[C.cast(C.byref(s), C.c_void_p) if s is not None else None for s in structs])
    return arr, structs


def _check_campaign_buffers(count: int, counts: torch.Tensor, records, site_counts):
    """The library writes counts[bench*5 + cls], site_counts[(bench*64 + site)*5 + cls] (u64 atomics)
    and records[n - first]: reject buffers that would be written out of bounds."""
    if not (isinstance(counts, torch.Tensor) and counts.is_cuda and counts.dtype == torch.int64
            and counts.is_contiguous() and counts.numel() == 15):
        raise ValueError("counts must be a contiguous int64 CUDA tensor of 15 elements ([3, 5])")
    if site_counts is not None and not (site_counts.is_cuda and site_counts.dtype == torch.int64
                                        and site_counts.is_contiguous() and site_counts.numel() == 3 * 64 * 5):
        raise ValueError("site_counts must be a contiguous int64 CUDA tensor of 3*64*5 elements")
    if records is not None and not (records.is_cuda and records.is_contiguous()
                                    and records.numel() * records.element_size() >= count * OUTCOME_DTYPE.itemsize):
        raise ValueError(f"records must be a contiguous CUDA tensor of >= {count} x {OUTCOME_DTYPE.itemsize} bytes")


def inject_campaign(bench_mode: int, devs, ranges, seed: int, first: int, count: int, counts: torch.Tensor,
                    records: torch.Tensor | None = None, site_counts: torch.Tensor | None = None, exact: int = 0,
                    batch: int = 0, site_masks=DEFAULT_SITE_MASKS, stream=None, nbits: int = 1, mode: int = 0,
                    variant: int = HK_FIFT, hang_factor: int = 0):
    """hauberk_inject_campaign.  devs/ranges: 3-lists by bench (None where unused; ranges may be None
    for variant HK_FI_ONLY).  counts: int64 cuda tensor [3, 5] (accumulated); records: optional uint8
    tensor of count * OUTCOME_DTYPE.itemsize bytes; site_counts: optional int64 [3, 64, 5]."""
    _check_campaign_buffers(count, counts, records, site_counts)
    arr, keep = _arg_array(devs)
    rng = [r if r is not None else Ranges() for r in ranges]
    rarr = (C.c_void_p * 3)(*[C.cast(C.byref(r), C.c_void_p) for r in rng])
    camp = Campaign(seed, first, count, nbits, mode, batch, exact, (C.c_uint64 * 3)(*site_masks), variant, hang_factor)
    st = lib().hauberk_inject_campaign(bench_mode, arr, rarr, C.byref(camp), _ptr(records), _ptr(counts),
                                       _ptr(site_counts), _stream(stream))
    _check(st, "hauberk_inject_campaign")


class CampaignSession:
    """hauberk_campaign_create / _run / _destroy: golden runs and workspaces prepared once, then
    asynchronous slices of the same seeded campaign.  Keep `devs` alive while the session lives."""

    def __init__(self, bench_mode: int, devs, ranges, seed: int, exact: int = 0, batch: int = 0,
                 site_masks=DEFAULT_SITE_MASKS, stream=None, nbits: int = 1, mode: int = 0,
                 variant: int = HK_FIFT, hang_factor: int = 0):
        self._arr, self._keep = _arg_array(devs)
        self._devs = devs
        self._rng = [r if r is not None else Ranges() for r in ranges]
        self._rarr = (C.c_void_p * 3)(*[C.cast(C.byref(r), C.c_void_p) for r in self._rng])
        self._camp = Campaign(seed, 0, 0, nbits, mode, batch, exact, (C.c_uint64 * 3)(*site_masks), variant, hang_factor)
        self._h = C.c_void_p()
        st = lib().hauberk_campaign_create(bench_mode, self._arr, self._rarr, C.byref(self._camp), C.byref(self._h),
                                           _stream(stream))
        _check(st, "hauberk_campaign_create")

    def run(self, first: int, count: int, counts: torch.Tensor, records: torch.Tensor | None = None,
            site_counts: torch.Tensor | None = None):
        _check_campaign_buffers(count, counts, records, site_counts)
        st = lib().hauberk_campaign_run(self._h, first, count, _ptr(records), _ptr(counts), _ptr(site_counts))
        _check(st, "hauberk_campaign_run")

    def close(self):
        if self._h:
            lib().hauberk_campaign_destroy(self._h)
            self._h = C.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def records_tensor(count: int, device="cuda") -> torch.Tensor:
    return torch.zeros(count * OUTCOME_DTYPE.itemsize, dtype=torch.uint8, device=device)


def records_numpy(rec: torch.Tensor) -> np.ndarray:
    return np.frombuffer(rec.cpu().numpy().tobytes(), dtype=OUTCOME_DTYPE)


def decode(bench_mode: int, devs, seed: int, first: int, count: int, site_masks=DEFAULT_SITE_MASKS, nbits: int = 1,
           variant: int = HK_FIFT):
    """hauberk_decode (host): the campaign's (bench, site, thread, instance, mask) tuples."""
    arr, keep = _arg_array(devs)
    masks = (C.c_uint64 * 3)(*site_masks)
    benches = np.zeros(count, dtype=np.int32)
    faults = (Fault * count)()
    st = lib().hauberk_decode(bench_mode, arr, masks, seed, nbits, variant, first, count,
                              benches.ctypes.data_as(C.c_void_p), C.cast(faults, C.c_void_p))
    _check(st, "hauberk_decode")
    return benches, [(f.site, f.thread, f.inst, f.mask) for f in faults]


def detector_site(bench: int, site: int, unroll: int = 4) -> bool:
    """hauberk_detector_site: the site exists only because of HAUBERK (absent from the FI-only binary)."""
    return lib().hauberk_detector_site(bench, unroll, site) == 1


def campaign_workspace_bytes(bench: int, dev, batch: int = 0, mode: int = 0, site_masks=DEFAULT_SITE_MASKS) -> int:
    a = dev.args()
    camp = Campaign(0, 0, 0, 1, mode, batch, 0, (C.c_uint64 * 3)(*site_masks), HK_FIFT, 0)
    return int(lib().hauberk_campaign_workspace_bytes(bench, C.byref(a), C.byref(camp)))


def summarize(counts) -> dict:
    """hauberk_summarize over the [.., 5] counters summed across benchmarks: coverage = P(detected or
    masked or failure) = 1 - undetected/total, sdc = undetected/total
    (an FI-only campaign's unprotected SDC rate, L211-213), detected, failure."""
    c = np.ascontiguousarray(np.asarray(counts, dtype=np.int64).reshape(-1, 5).sum(0))
    out = Summary()
    st = lib().hauberk_summarize(c.ctypes.data_as(C.c_void_p), C.byref(out))
    if st != 0:
        return {"coverage": float("nan"), "sdc": float("nan"), "detected": float("nan"), "failure": float("nan"), "total": 0}
    return {"coverage": out.coverage, "sdc": out.sdc, "detected": out.detected, "failure": out.failure, "total": out.total}


def coverage(counts) -> float:
    """Coverage of a campaign (hauberk_summarize)."""
    return summarize(counts)["coverage"]


def unprotected_sdc(counts) -> float:
    """SDC ratio of an FI-only campaign's counters (hauberk_summarize: undetected / total)."""
    return summarize(counts)["sdc"]


def extend_ranges(rs: RangeSet, values) -> int:
    """hauberk_extend_ranges (A11): add the values to their correlation classes; returns ranges added."""
    v = np.ascontiguousarray(np.asarray(values, dtype=np.float32))
    added = C.c_int32(0)
    _check(lib().hauberk_extend_ranges(C.byref(rs), v.ctypes.data_as(C.c_void_p), v.size, C.byref(added)),
           "hauberk_extend_ranges")
    return int(added.value)


def outliers(cb: Control, d: int) -> list:
    """hauberk_outliers: the out-of-range interval the run recorded for detector d (0-2 floats)."""
    out = (C.c_float * 2)()
    n = C.c_int32(0)
    _check(lib().hauberk_outliers(C.byref(cb), d, out, C.byref(n)), "hauberk_outliers")
    return [float(out[k]) for k in range(n.value)]


def alpha_update(alpha: float, fp_ratio: float, hi: float = 0.10, lo: float = 0.05) -> float:
    return float(lib().hauberk_alpha_update(alpha, fp_ratio, hi, lo))


DIAG_NAMES = ["ok", "false_alarm", "transient", "persistent", "failed"]


def diagnose(alarm1: int, fail1: int, alarm2: int, fail2: int, identical: bool) -> str:
    return DIAG_NAMES[lib().hauberk_diagnose(alarm1, fail1, alarm2, fail2, 1 if identical else 0)]


def release_caches():
    lib().hauberk_release_caches()
