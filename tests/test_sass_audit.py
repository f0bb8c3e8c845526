"""T5 SASS audit: nvcc/ptxas must not have folded HAUBERK's detectors away.

cuobjdump -sass of libhauberk.so (sm_100a): the FT kernels keep the duplicated definitions
(extra ISETP compares), the XOR checksum pairs (LOP3), and a per-atom counter add inside the main
loop; BASE has none of them; both issue the same MUFU work.  The campaign path must also carry
the TMA bulk copy (UBLKCP) that stages atoms / k-space."""
import os
import re
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_yimpski11_b200", "libhauberk.so")


@pytest.fixture(scope="module")
def sass():
    if not shutil.which("cuobjdump"):
        pytest.skip("cuobjdump not available")
    if not os.path.exists(LIB):
        import __graft_entry__ as g
        g.build()
    txt = subprocess.check_output(["cuobjdump", "-sass", LIB], text=True)
    out = {}
    for sec in re.split(r"\n\s*Function : ", txt)[1:]:
        name = sec.split("\n", 1)[0].strip()
        ops = [m[1] for m in re.findall(r"/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*(?:\.[A-Z0-9_]+)*)", sec)]
        out[name] = ops
    return out


def _find(sass, pattern):
    names = [n for n in sass if re.search(pattern, n)]
    assert names, pattern
    return sass[names[0]]


def _count(ops, prefix):
    return sum(1 for o in ops if o.startswith(prefix))


def _loop_region(ops, anchor):
    idx = [i for i, o in enumerate(ops) if o.startswith(anchor)]
    return ops[idx[0]: idx[-1] + 1]


@pytest.mark.parametrize("u", [4, 8])
def test_cp_ft_keeps_detectors(sass, u):
    ft = _find(sass, rf"cp_kernelILi3ELi{u}ELb0E")
    base = _find(sass, rf"cp_kernelILi0ELi{u}ELb0E")
    assert _count(ft, "MUFU.RSQ") >= _count(base, "MUFU.RSQ") > 0
    assert _count(ft, "LOP3") >= _count(base, "LOP3") + 20       # chk ^= v twice per virtual variable
    assert _count(ft, "ISETP") >= _count(base, "ISETP") + 6      # duplicate compares, CheckEqual
    loop_ft = _loop_region(ft, "MUFU.RSQ")
    loop_base = _loop_region(base, "MUFU.RSQ")
    adds = lambda ops: sum(1 for o in ops if o.startswith(("IADD3", "VIADD", "IADD ")))
    assert adds(loop_ft) >= 4 > adds(loop_base)                   # it++ per atom survives unrolling
    assert "UBLKCP.S.G" in ft                                      # TMA bulk copy of atom tiles


def test_mriq_ft_keeps_detectors(sass):
    ft = _find(sass, r"mriq_kernelILi3ELb0E")
    base = _find(sass, r"mriq_kernelILi0ELb0E")
    assert _count(ft, "MUFU.SIN") == _count(base, "MUFU.SIN") > 0
    assert _count(ft, "MUFU.COS") == _count(base, "MUFU.COS") > 0
    assert _count(ft, "LOP3") >= _count(base, "LOP3") + 10
    # duplicated loads of sX, sY, sZ (A3) through an opaque index
    assert _count(ft, "LDG") >= _count(base, "LDG") + 3
    # the counter advances once per unrolled group of samples (it += UNR through an opaque 1, the
    # strength reduction of an unrolled it++): the FT loop keeps an add the BASE loop does not have
    adds = lambda ops: sum(1 for o in ops if o.startswith(("IADD3", "VIADD", "IADD ", "IMAD")))
    assert adds(_loop_region(ft, "MUFU.SIN")) > adds(_loop_region(base, "MUFU.SIN"))
    assert "UBLKCP.S.G" in ft


def test_tpacf_ft_keeps_detectors(sass):
    ft = _find(sass, r"tpacf_kernelILi3EE")
    base = _find(sass, r"tpacf_kernelILi0EE")
    assert _count(ft, "LOP3") >= _count(base, "LOP3") + 10
    assert _count(ft, "ISETP") >= _count(base, "ISETP") + 8
    assert len(ft) > len(base)


def test_fi_kernels_compiled_for_every_site_kind(sass):
    # kinds x {FAST, EXACT} x U {4, 8} x {FI&FT, FI-only}
    assert len([n for n in sass if "cp_fi_kernel" in n]) == 15 * 2 * 2 * 2
    assert len([n for n in sass if "mriq_fi_kernel" in n]) == 17 * 2 * 2  # 16 Q-kernel kinds + PhiMag
    assert len([n for n in sass if "tpacf_fi_kernel" in n]) == 11 * 2


@pytest.mark.parametrize("pat", [r"tpacf_fi_kernelILi2ELb{}EE", r"mriq_fi_kernelILi2ELb0ELb{}EE", r"cp_fi_kernelILi2ELi4ELb0ELb{}EE"])
def test_fi_only_binary_has_no_detector_code(sass, pat):
    """Row a7: the FI-only replicas are the original program plus the hook — fewer instructions
    than the FI&FT replicas of the same site kind (no duplicates, checksums, counters, checks)."""
    fift, fionly = _find(sass, pat.format(1)), _find(sass, pat.format(0))
    assert len(fionly) < len(fift)
    assert _count(fionly, "LOP3") < _count(fift, "LOP3")


def test_tpacf_replica_loop_uses_byte_table_edge_load_and_one_shared_atomic_per_pair(sass):
    """per pair one LDS.U8 (4 * bmin), one 32-bit edge load, one compare, one ATOMS; the
    partner quads come in as broadcast LDS.128 shared by the 4 points of a thread (no LDS.64: a
    64-bit shared load costs 2-3 wavefronts)."""
    ops = _find(sass, r"tpacf_fi_kernelILi2ELb1EE")
    assert _count(ops, "LDS.U8") >= 16 and _count(ops, "ATOMS") >= 16 and _count(ops, "LDS.128") >= 3
    assert _count(ops, "LDS.64") == 0
