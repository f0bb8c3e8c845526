"""Host-side pin of the TPACF bucket-table rule the CUDA kernels use (tpacf.cu: tpacf_lut_kernel,
DESIGN §6.3), checked against the binning definition by brute force — no GPU.

Binning definition (PAPER L80-84 names the histogram): bin(dot) = #{e : dot < edge[e]}.
The kernels look up bmin = table[bits(u) >> 21] with u = fl(1 - dot) and return
bin = bmin + (dot < edge[bmin]).  The table rule restated here: bucket ordinal ord(q) = 1024 + q for
q < 1024 (u >= +0) and 2047 - q otherwise (u <= -0); bmin(q) = #{k : ord(bucket(fl(1 - edge[k]))) <
ord(q)}; NaN-u buckets and the -inf / negative-NaN buckets give 0; the table is valid iff no two
edges share a bucket.  This file re-derives nothing from the CUDA source: it evaluates the rule
with numpy binary32 arithmetic and compares it with the definition on every bucket boundary of the
configuration-3 edges and on random and special dots.
"""
import numpy as np

import workloads as W

F32 = np.float32


def bits(x):
    return np.asarray(x, dtype=np.float32).view(np.uint32)


def from_bits(b):
    return np.asarray(b, dtype=np.uint32).view(np.float32)


def ordq(q):
    q = np.asarray(q, dtype=np.int64)
    return np.where(q < 1024, 1024 + q, 2047 - q)


def table(edges):
    u = (F32(1.0) - edges.astype(np.float32)).astype(np.float32)
    eo = ordq(bits(u) >> 21)
    valid = bool(np.all(eo[:-1] < eo[1:]) and not np.isnan(u).any())
    q = np.arange(2048)
    ex = (q >> 2) & 0xFF
    t = (ordq(q)[:, None] > eo[None, :]).sum(axis=1)
    t[(ex == 0xFF) & ((q & 0x400) == 0) & ((q & 3) != 0)] = 0  # positive NaN buckets
    t[(ex == 0xFF) & ((q & 0x400) != 0)] = 0  # -inf and negative NaN buckets
    return t, valid


def bin_def(edges, dot):
    return (dot[:, None] < edges[None, :].astype(np.float32)).sum(axis=1)


def bin_table(edges, t, dot):
    u = (F32(1.0) - dot).astype(np.float32)
    bm = t[bits(u) >> 21]
    e = np.concatenate([edges.astype(np.float32), np.full(32, -np.inf, dtype=np.float32)])
    return bm + (dot < e[bm])


def boundary_dots(edges):
    """Dots at and around every bucket boundary of u and around every edge (binary32 neighbours)."""
    qs = np.arange(2048, dtype=np.uint64)
    lo = (qs << 21).astype(np.uint32)
    hi = lo | np.uint32(0x1FFFFF)
    us = np.concatenate([from_bits(lo), from_bits(hi)])
    us = us[np.isfinite(us)]
    d = (F32(1.0) - us).astype(np.float32)
    e32 = edges.astype(np.float32)
    base = np.concatenate([d, e32[np.isfinite(e32)]])
    near = [base]
    up, dn = base.copy(), base.copy()
    with np.errstate(over="ignore"):
        for _ in range(6):
            up, dn = np.nextafter(up, F32(np.inf)), np.nextafter(dn, F32(-np.inf))
            near += [up, dn]
    return np.concatenate(near).astype(np.float32)


def test_table_rule_equals_the_binning_definition_config3():
    edges = W.tpacf_edges(20)
    t, valid = table(edges)
    assert valid
    dots = boundary_dots(edges)
    rng = np.random.default_rng(5)
    dots = np.concatenate([dots, rng.uniform(-1, 1, 200000).astype(np.float32),
                           (1 - rng.exponential(1e-5, 200000)).astype(np.float32),
                           np.array([1.0, -1.0, 0.0, -0.0, 1.0000001, np.inf, -np.inf, np.nan], dtype=np.float32)])
    with np.errstate(invalid="ignore"):
        np.testing.assert_array_equal(bin_table(edges, t, dots), bin_def(edges, dots))


def test_table_rule_with_edges_at_one_zero_and_infinities():
    # an edge at 1.0 (u = +0), one at 0.0, a -inf pad: the definition still holds wherever valid
    edges = np.array([1.0, 0.999, 0.5, 0.0, -0.5, -np.inf], dtype=np.float32)
    t, valid = table(edges)
    assert valid
    dots = boundary_dots(edges)
    with np.errstate(invalid="ignore"):
        np.testing.assert_array_equal(bin_table(edges, t, dots), bin_def(edges, dots))


def test_table_invalid_when_two_edges_share_a_bucket():
    # two edges whose u = 1 - e fall in the same (exponent, top-2-mantissa-bits) bucket
    edges = np.array([0.5, 0.49, 0.0], dtype=np.float32)
    _, valid = table(edges)
    assert not valid
