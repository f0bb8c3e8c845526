"""C ABI checks that need no GPU: libhauberk.so loads, exports every symbol include/hauberk.h
declares, and its host-side decode (R14/R15) matches the oracle's bit for bit."""
import ctypes as C
import os
import re
import subprocess

import numpy as np
import pytest

import oracle as O
import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "hauberk.h")
LIB = os.path.join(ROOT, "paper_conf_ipps_yimpski11_b200", "libhauberk.so")


@pytest.fixture(scope="module")
def hk():
    if not os.path.exists(LIB):
        import __graft_entry__ as g
        g.build()
    from paper_conf_ipps_yimpski11_b200 import hauberk
    return hauberk


def declared_symbols():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"HK_API\s+[\w\s\*]+?\b(hauberk_\w+)\s*\(", txt)))


def test_header_declares_the_north_star_entry_points():
    syms = declared_symbols()
    for s in ["hauberk_profile_ranges", "hauberk_run_cp", "hauberk_run_mriq", "hauberk_run_tpacf",
              "hauberk_inject_campaign"]:
        assert s in syms


def test_library_exports_every_declared_symbol(hk):
    out = subprocess.check_output(["nm", "-D", "--defined-only", LIB], text=True)
    exported = set(re.findall(r"\sT\s(hauberk_\w+)", out))
    missing = set(declared_symbols()) - exported
    assert not missing, missing
    L = hk.lib()
    for s in declared_symbols():
        assert hasattr(L, s)
    assert sorted(hk.EXPORTED) == declared_symbols()


def test_version_and_strerror(hk):
    L = hk.lib()
    assert L.hauberk_version() == 2
    assert L.hauberk_strerror(0) == b"ok"
    assert b"ranges" in L.hauberk_strerror(3)


def test_site_counts_match_oracle(hk):
    for b in range(3):
        for u in (1, 2, 4, 8):
            assert hk.num_sites(b, u) == O.nsites(b, u)


class _FakeDev:
    """ABI structs with non-null dummy device pointers: decode only reads shapes."""

    def __init__(self, hk, bench, p):
        self.bench = bench
        self.p = p
        self.hk = hk

    def args(self):
        hk, p, fake = self.hk, self.p, C.c_void_p(0x10000)
        if self.bench == 0:
            return hk.CPArgs(fake, fake, p.n_atoms, p.z0, p.h, p.nx, p.ny, p.bx, p.by, p.unroll, fake, 0)
        if self.bench == 1:
            return hk.MRIQArgs(fake, fake, fake, p.n_vox, p.n_k, fake, fake, fake, fake, fake, fake, fake, fake, 0)
        return hk.TPACFArgs(fake, fake, p.n, p.n_rand, p.n_bins, fake)


@pytest.mark.parametrize("mode", [-1, 0, 1, 2])
def test_decode_parity_with_oracle(hk, mode):
    probs = [W.cp_config1(), W.mriq_config2(), W.tpacf_config3()]
    devs = [_FakeDev(hk, b, probs[b]) for b in range(3)]
    seed = W.CAMPAIGN_SEED_CFG5
    first, count = 123456, 3000
    gb, gf = hk.decode(mode, devs, seed, first, count)
    ob, of = O.decode(mode, probs, seed, first, count)
    assert np.array_equal(gb, ob)
    assert gf == of


def test_decode_parity_with_site_masks(hk):
    probs = [W.cp_small(), W.mriq_small(), W.tpacf_small()]
    devs = [_FakeDev(hk, b, probs[b]) for b in range(3)]
    masks = (0b1010101010101010101010101, (1 << 15) - 1, ((1 << 31) - 1) ^ 0b111)
    gb, gf = hk.decode(-1, devs, 77, 0, 900, site_masks=masks)
    ob, of = O.decode(-1, probs, 77, 0, 900, site_masks=masks)
    assert gf == of
    for b, (s, *_rest) in zip(gb, gf):
        assert (masks[b] >> s) & 1


def test_invalid_arguments_fail_before_launch(hk):
    p = W.cp_small()
    d = _FakeDev(hk, 0, p)
    a = d.args()
    a.unroll = 3
    st = hk.lib().hauberk_run_cp(C.byref(a), 1, None, None, None, None)
    assert st == 1  # HK_ERR_INVALID
    a = d.args()
    st = hk.lib().hauberk_run_cp(C.byref(a), 1, None, C.c_void_p(0x10000), None, None)
    assert st == 3  # FT without ranges -> HK_ERR_NO_RANGES


@pytest.mark.parametrize("k", [3, 6, 10, 15])
def test_multibit_decode_parity_with_oracle(hk, k):
    probs = [W.cp_config1(), W.mriq_config2(), W.tpacf_config3()]
    devs = [_FakeDev(hk, b, probs[b]) for b in range(3)]
    gb, gf = hk.decode(-1, devs, 99, 5000, 1500, nbits=k)
    ob, of = O.decode(-1, probs, 99, 5000, 1500, nbits=k)
    assert gf == of


@pytest.mark.parametrize("mode", [-1, 0, 2])
def test_fi_only_decode_parity_with_oracle(hk, mode):
    """Row a7: the FI-only catalogue (original program's sites only) decodes identically on both sides."""
    probs = [W.cp_config1(), W.mriq_config2(), W.tpacf_config3()]
    devs = [_FakeDev(hk, b, probs[b]) for b in range(3)]
    gb, gf = hk.decode(mode, devs, 4242, 77, 2000, variant=hk.HK_FI_ONLY)
    ob, of = O.decode(mode, probs, 4242, 77, 2000, variant=1)
    assert np.array_equal(gb, ob) and gf == of
    for b, (s, *_r) in zip(gb, gf):
        assert not hk.detector_site(int(b), s, 4)


def test_detector_sites_match_oracle(hk):
    for b in range(3):
        for u in (4, 8):
            for s in range(hk.num_sites(b, u)):
                assert hk.detector_site(b, s, u) == O.detector_site(b, s, u), (b, u, s)
    assert hk.lib().hauberk_detector_site(2, 4, 30) == -1 and hk.lib().hauberk_detector_site(5, 4, 0) == -1


def test_summary_extension_alpha_and_diagnosis_match_the_oracle_twins(hk):
    """The evaluation / recovery arithmetic of the C ABI (hauberk_summarize, _extend_ranges,
    _alpha_update, _diagnose) against the oracle's independent implementations, whose values are
    pinned by hand in tests/test_oracle_pins.py."""
    rng = np.random.default_rng(5)
    for _ in range(50):
        c = rng.integers(0, 1000, size=(3, 5))
        g, o = hk.summarize(c), O.coverage(c)
        for k in ("coverage", "sdc", "detected", "failure"):
            assert g[k] == o[k]
    for _ in range(200):
        a = float(10.0 ** rng.integers(0, 4))
        fp = float(rng.choice([0.0, 0.01, 0.05, 0.07, 0.10, 0.11, 0.5]))
        assert hk.alpha_update(a, fp) == O.alpha_step(a, fp)
    for a1 in (0, 4, 9):
        for f1 in (0, 1):
            for a2 in (0, 4, 8):
                for f2 in (0, 2):
                    for ident in (False, True):
                        assert hk.diagnose(a1, f1, a2, f2, ident) == O.diagnose(a1, f1, a2, f2, ident)
    for t in (-6, -3, 0):
        for _ in range(40):
            vals = (rng.standard_normal(rng.integers(0, 6)) * 10.0 ** rng.integers(-8, 3)).astype(np.float32)
            base = np.sort(rng.standard_normal(2).astype(np.float32))
            g, o = hk.RangeSet(), O.RSet()
            for rs in (g, o):
                rs.t_exp10 = t
                rs.n = 1
                rs.lo[0], rs.hi[0] = float(base[0]), float(base[1])
            ga, oa = hk.extend_ranges(g, vals), O.extend_ranges(o, vals)
            assert ga == oa and g.n == o.n
            assert [(g.lo[r], g.hi[r]) for r in range(g.n)] == [(o.lo[r], o.hi[r]) for r in range(o.n)]


def test_outliers_decodes_the_control_block_ordinals(hk):
    cb = hk.Control()
    for d in range(8):
        cb.outlier_min_ord[d], cb.outlier_max_ord[d] = 0x7FFFFFFF, -0x80000000
    assert hk.outliers(cb, 0) == []
    L = O.lib()
    cb.outlier_min_ord[1], cb.outlier_max_ord[1] = L.ora_ord(-2.5), L.ora_ord(1e-3)
    assert hk.outliers(cb, 1) == [-2.5, float(np.float32(1e-3))]
    cb.outlier_min_ord[2] = cb.outlier_max_ord[2] = L.ora_ord(7.0)
    assert hk.outliers(cb, 2) == [7.0]


def test_campaign_buffers_are_validated_before_the_call(hk):
    import torch
    with pytest.raises(ValueError):
        hk._check_campaign_buffers(10, torch.zeros(15, dtype=torch.int32), None, None)


def test_workspace_bytes(hk):
    p = W.tpacf_config3()
    d = _FakeDev(hk, 2, p)
    n = hk.campaign_workspace_bytes(2, d, batch=64)
    # golden + 64 replica histograms (9 x 22 u64, padded to 200) + 65 control blocks + the TPACF tables
    assert n >= 65 * 200 * 8 + 65 * hk.CONTROL_BYTES
    assert hk.campaign_workspace_bytes(2, d, batch=64, mode=1) < n
