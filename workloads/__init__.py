"""Seeded synthetic input generators shared by the CPU oracle and the CUDA path.

This module holds NO arithmetic of the HAUBERK method (no detector, profiler,
injector or benchmark kernel math).  It only draws the inputs of the three
benchmarks with the shapes and value distributions stated in DESIGN.md §4
("input recipe"), from the counter-based SplitMix64 stream of DESIGN.md R15.
Both `oracle/` and `paper_conf_ipps_yimpski11_b200/` consume the arrays it returns.

Configs (BASELINE.json `configs`, restated in SURVEY.md §8(d)):
  1  CP-s   100 atoms, 64x64 grid, h = 0.1 A          seed 54321
  2  MRI-Q  32^3 voxels, 3,072 k-space samples         seed 0x4D5249
  3  TPACF  4,096 points x (1 data + 4 random sets)    seed 0x545041
  4  CP-L   40,000 atoms, 512x512 grid                 seed 54321
  5  mixed campaign over the cfg 1/2/3 shapes          seed 0x4841554245524B05
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

CAMPAIGN_SEED_CFG1 = 0x4841554245524B01
CAMPAIGN_SEED_CFG5 = 0x4841554245524B05


def splitmix64(seed: int, count: int, start: int = 0) -> np.ndarray:
    """Outputs number start..start+count-1 (0-based) of SplitMix64 seeded with `seed`.

    Output m = mix(seed + (m+1)*gamma) (R15).  Pure integer stream; wraps mod 2^64.
    """
    with np.errstate(over="ignore"):
        idx = np.arange(start + 1, start + count + 1, dtype=np.uint64)
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + idx * GAMMA
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def uniform(seed: int, count: int, lo: float, hi: float, start: int = 0) -> np.ndarray:
    """Doubles uniform in [lo, hi) from the top 53 bits of the stream."""
    u = (splitmix64(seed, count, start) >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)
    return lo + (hi - lo) * u


def gaussian(seed: int, count: int, start: int = 0) -> np.ndarray:
    """Standard normals by Box-Muller from 2*count stream outputs."""
    u = uniform(seed, 2 * count, 0.0, 1.0, start)
    u1 = 1.0 - u[0::2]  # (0, 1]
    u2 = u[1::2]
    return np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * math.pi * u2)


# ----------------------------------------------------------------------------------------------
# CP (Coulombic potential) — Fig. 9 dataflow; Parboil-style planar slice.
# ----------------------------------------------------------------------------------------------
@dataclass
class CPProblem:
    atoms: np.ndarray  # float32 [n_atoms, 4] = (x, y, z, q)
    nx: int
    ny: int
    h: float  # grid spacing (A), float32-representable
    z0: float  # z of the potential slice
    bx: int = 16
    by: int = 16
    unroll: int = 4

    @property
    def n_atoms(self) -> int:
        return int(self.atoms.shape[0])


def cp_problem(n_atoms: int, nx: int, ny: int, seed: int = 54321, h: float = 0.1,
               bx: int = 16, by: int = 16, unroll: int = 4) -> CPProblem:
    """Atoms uniform over the slice's x/y extent, z in [0.5, 2.0) A above the slice z0 = 0, q ~ U(-1, 1).

    The minimum atom-to-grid distance is therefore >= 0.5 A (no near-singular r^2).
    Stream layout: outputs [0, n) x, [n, 2n) y, [2n, 3n) z, [3n, 4n) q.
    """
    hf = float(np.float32(h))
    n = n_atoms
    a = np.empty((n, 4), dtype=np.float32)
    a[:, 0] = uniform(seed, n, 0.0, nx * hf, 0).astype(np.float32)
    a[:, 1] = uniform(seed, n, 0.0, ny * hf, n).astype(np.float32)
    a[:, 2] = uniform(seed, n, 0.5, 2.0, 2 * n).astype(np.float32)
    a[:, 3] = uniform(seed, n, -1.0, 1.0, 3 * n).astype(np.float32)
    return CPProblem(atoms=a, nx=nx, ny=ny, h=hf, z0=0.0, bx=bx, by=by, unroll=unroll)


def cp_config1() -> CPProblem:
    return cp_problem(100, 64, 64, seed=54321, h=0.1, bx=16, by=16, unroll=4)


def cp_config4(bx: int = 16, by: int = 16, unroll: int = 8) -> CPProblem:
    return cp_problem(40000, 512, 512, seed=54321, h=0.1, bx=bx, by=by, unroll=unroll)


# ----------------------------------------------------------------------------------------------
# MRI-Q — Parboil-small shape (outside PAPER.md; PAPER.md names it at L503, L1440-1487).
# ----------------------------------------------------------------------------------------------
@dataclass
class MRIQProblem:
    x: np.ndarray
    y: np.ndarray
    z: np.ndarray
    kx: np.ndarray
    ky: np.ndarray
    kz: np.ndarray
    phi_r: np.ndarray
    phi_i: np.ndarray

    @property
    def n_vox(self) -> int:
        return int(self.x.shape[0])

    @property
    def n_k(self) -> int:
        return int(self.kx.shape[0])


def mriq_problem(side: int, n_k: int, seed: int = 0x4D5249, kmax: float = 16.0,
                 n_vox: int | None = None) -> MRIQProblem:
    """Voxels on a side^3 grid at (i - side/2)/side per axis (normalised FOV, exact in fp32),
    optionally truncated to the first n_vox voxels (ragged parity shapes);
    k-samples kx, ky, kz ~ U(-kmax, kmax) cycles/FOV; phiR, phiI ~ U(-1, 1)."""
    n = side ** 3 if n_vox is None else n_vox
    i = np.arange(n)
    ix, iy, iz = i % side, (i // side) % side, i // (side * side)
    f = lambda v: ((v - side // 2) / side).astype(np.float32)
    k = n_k
    return MRIQProblem(
        x=f(ix), y=f(iy), z=f(iz),
        kx=uniform(seed, k, -kmax, kmax, 0).astype(np.float32),
        ky=uniform(seed, k, -kmax, kmax, k).astype(np.float32),
        kz=uniform(seed, k, -kmax, kmax, 2 * k).astype(np.float32),
        phi_r=uniform(seed, k, -1.0, 1.0, 3 * k).astype(np.float32),
        phi_i=uniform(seed, k, -1.0, 1.0, 4 * k).astype(np.float32),
    )


def mriq_config2() -> MRIQProblem:
    return mriq_problem(32, 3072)


# ----------------------------------------------------------------------------------------------
# TPACF — two-point angular correlation (PAPER.md L80-84 names its 1 % rule; Parboil shape).
# ----------------------------------------------------------------------------------------------
@dataclass
class TPACFProblem:
    pts: np.ndarray  # float32 [(1 + n_rand), n, 3] unit vectors; set 0 = data
    edges: np.ndarray  # float32 [n_bins + 1], strictly decreasing cos(angle edges)

    @property
    def n(self) -> int:
        return int(self.pts.shape[1])

    @property
    def n_rand(self) -> int:
        return int(self.pts.shape[0]) - 1

    @property
    def n_bins(self) -> int:
        return int(self.edges.shape[0]) - 1


def tpacf_edges(n_bins: int = 20, lo_arcmin: float = 1.0, hi_arcmin: float = 10000.0) -> np.ndarray:
    """edge[k] = (float) cos(10^(log10(lo) + k*(log10(hi)-log10(lo))/n_bins) arcmin), k = 0..n_bins.
    Computed in double on the host and shared as data."""
    l0, l1 = math.log10(lo_arcmin), math.log10(hi_arcmin)
    ang = [10.0 ** (l0 + k * (l1 - l0) / n_bins) / 60.0 * math.pi / 180.0 for k in range(n_bins + 1)]
    return np.array([math.cos(a) for a in ang], dtype=np.float32)


def _sphere_uniform(seed: int, n: int, start: int) -> np.ndarray:
    z = uniform(seed, n, -1.0, 1.0, start)
    ph = uniform(seed, n, 0.0, 2.0 * math.pi, start + n)
    s = np.sqrt(np.maximum(0.0, 1.0 - z * z))
    return np.stack([s * np.cos(ph), s * np.sin(ph), z], axis=1)


def tpacf_problem(n: int, n_rand: int, seed: int = 0x545041, n_bins: int = 20,
                  clumps: int = 64, sigma_deg: float = 0.5) -> TPACFProblem:
    """Random sets uniform on the sphere; the data set is 50 % uniform + 50 % in `clumps`
    Gaussian clumps of width sigma_deg (so DD differs from RR)."""
    pts = np.empty((1 + n_rand, n, 3), dtype=np.float32)
    off = 0
    nu = n // 2
    nc = n - nu
    d_uni = _sphere_uniform(seed, nu, off); off += 2 * nu
    centers = _sphere_uniform(seed, clumps, off); off += 2 * clumps
    which = (uniform(seed, nc, 0.0, clumps, off)).astype(np.int64); off += nc
    g = gaussian(seed, 3 * nc, off).reshape(nc, 3); off += 6 * nc
    sig = sigma_deg * math.pi / 180.0
    v = centers[which] + sig * g
    v /= np.linalg.norm(v, axis=1, keepdims=True)
    pts[0] = np.concatenate([d_uni, v], axis=0).astype(np.float32)
    for s in range(n_rand):
        pts[1 + s] = _sphere_uniform(seed ^ (0x1000 * (s + 1)), n, 0).astype(np.float32)
    return TPACFProblem(pts=pts, edges=tpacf_edges(n_bins))


def tpacf_config3() -> TPACFProblem:
    return tpacf_problem(4096, 4)


# ----------------------------------------------------------------------------------------------
# Small "parity" shapes: several tiles plus a ragged tail, oracle finishes in well under a second.
# ----------------------------------------------------------------------------------------------
def cp_small(seed: int = 7, unroll: int = 4) -> CPProblem:
    return cp_problem(37, 64, 32, seed=seed, h=0.1, bx=16, by=8, unroll=unroll)


def mriq_small(seed: int = 11) -> MRIQProblem:
    return mriq_problem(8, 197, seed=seed, n_vox=500)


def tpacf_small(seed: int = 13, n: int = 300, n_rand: int = 2) -> TPACFProblem:
    return tpacf_problem(n, n_rand, seed=seed, clumps=8, sigma_deg=2.0)
