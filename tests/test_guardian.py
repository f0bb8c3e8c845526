"""Guardian host logic (DESIGN R25) without a GPU: supervision of a fake child that
answers, crashes (CRASH line + status 3), dies on a signal, or hangs; the blob format read by the
native child; the modelled-vs-real comparison.  The real unguarded runs are -m gpu
(test_gpu_parity.py::test_guardian_real_crash_validation)."""
import os
import struct
import subprocess
import sys
import textwrap
import time

import numpy as np
import pytest

import workloads as W
from paper_conf_ipps_yimpski11_b200 import guardian as G

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

FAKE_CHILD = textwrap.dedent("""
    import os, signal, sys, time
    blob, idx_file, start = sys.argv[1], sys.argv[2], int(sys.argv[3])
    idx = [int(x) for x in open(idx_file).read().split()]
    print("READY 50.0", flush=True)
    for n in idx[start:]:
        print(f"BEGIN {n}", flush=True)
        k = n % 4
        if k == 0:
            print(f"DONE {n} {n % 3} 4 0", flush=True)
        elif k == 1:
            print(f"CRASH {n} cudaErrorIllegalAddress", flush=True)
            sys.exit(3)
        elif k == 2:
            time.sleep(60)
        else:
            os.kill(os.getpid(), signal.SIGSEGV)
""")


def test_guardian_supervises_done_crash_hang_and_signal(tmp_path):
    child = tmp_path / "child.py"
    child.write_text(FAKE_CHILD)
    g = G.Guardian(str(tmp_path / "unused.blob"), child_cmd=[sys.executable, str(child)], floor_s=0.5)
    idx = [0, 1, 2, 3, 4, 8, 5, 6, 7]
    t0 = time.monotonic()
    out = g.run(idx)
    wall = time.monotonic() - t0
    assert sorted(out) == sorted(idx)
    assert [out[n].kind for n in idx] == ["done", "crash", "hang", "crash", "done", "done", "crash", "hang", "crash"]
    assert out[0].cls == 0 and out[4].cls == 1 and out[8].cls == 2 and out[0].alarm == 4
    assert out[1].detail == "cudaErrorIllegalAddress"
    assert "status" in out[3].detail  # died on a signal without a CRASH line
    assert out[2].label == "hang" and out[2].seconds >= 0.5
    assert g.restarts == 6  # one new child after every crash / hang / death
    assert wall < 30  # hangs were cut at the 0.5 s floor, not the child's 60 s sleep


def test_guardian_timeout_rule():
    g = G.Guardian("x", floor_s=2.0, factor=10.0)
    assert g._limit(None) == 2.0
    assert g._limit(1e-3) == 2.0
    assert g._limit(0.5) == 5.0


def test_guardian_child_error_is_raised(tmp_path):
    child = tmp_path / "child.py"
    child.write_text("print('ERROR blob bad', flush=True)\nimport sys; sys.exit(2)\n")
    g = G.Guardian("x", child_cmd=[sys.executable, str(child)])
    with pytest.raises(RuntimeError, match="blob bad"):
        g.run([1, 2])


def _ranges():
    from paper_conf_ipps_yimpski11_b200 import hauberk as hk
    R = hk.Ranges()
    R.n_det = 1
    R.alpha = 1.0
    R.det[0].n = 1
    R.det[0].lo[0], R.det[0].hi[0] = -1.0, 2.0
    return R


@pytest.mark.parametrize("bench", [0, 1, 2])
def test_blob_layout(tmp_path, bench):
    p = [W.cp_small(), W.mriq_small(), W.tpacf_small()][bench]
    path = tmp_path / "p.blob"
    G.write_blob(str(path), bench, p, _ranges(), seed=77, site_mask=(1 << 64) - 1, nbits=3)
    b = path.read_bytes()
    assert b[:8] == b"HKGRD01\0"
    bench_, exact, nbits, narr = struct.unpack_from("<4i", b, 8)
    assert (bench_, exact, nbits) == (bench, 0, 3)
    seed, mask = struct.unpack_from("<2Q", b, 24)
    assert seed == 77 and mask == (1 << 64) - 1
    off = 40 + 264 + 32 + 16  # hk_ranges is 264 bytes (include/hauberk.h)
    sizes = []
    for _ in range(narr):
        (n,) = struct.unpack_from("<Q", b, off)
        sizes.append(n)
        off += 8 + 4 * n
    assert off == len(b)
    if bench == 0:
        want = [p.n_atoms * 4]
    elif bench == 1:
        want = [p.n_vox] * 3 + [p.n_k] * 5
    else:
        want = [p.pts.size, p.edges.size]
    assert sizes == want


def test_native_child_parses_blob_before_touching_cuda(tmp_path):
    """hk_guardian_child exits 2 with ERROR blob on a bad file, and gets past the blob (failing at
    its first CUDA call on this GPU-less host) on a good one."""
    if not os.path.exists(G.CHILD_PATH):
        import __graft_entry__ as g
        g.build()
    bad = tmp_path / "bad.blob"
    bad.write_bytes(b"nope")
    idx = tmp_path / "i.txt"
    idx.write_text("0\n")
    r = subprocess.run([G.CHILD_PATH, str(bad), str(idx), "0"], capture_output=True, text=True, timeout=60)
    assert r.returncode == 2 and r.stdout.startswith("ERROR blob")
    good = tmp_path / "good.blob"
    G.write_blob(str(good), 0, W.cp_small(), _ranges(), seed=1, site_mask=(1 << 64) - 1)
    r = subprocess.run([G.CHILD_PATH, str(good), str(idx), "0"], capture_output=True, text=True, timeout=120)
    assert "ERROR blob" not in r.stdout
    try:
        import torch
        has_gpu = torch.cuda.is_available()
    except Exception:
        has_gpu = False
    if not has_gpu:
        assert r.returncode == 2 and r.stdout.startswith("ERROR cuda")


def test_compare_counts_agreement():
    real = {1: G.RealOutcome(1, "crash"), 2: G.RealOutcome(2, "done", cls=0), 3: G.RealOutcome(3, "hang"),
            4: G.RealOutcome(4, "done", cls=3), 5: G.RealOutcome(5, "done", cls=2)}
    modelled = {1: "crash", 2: "crash", 3: "hang", 4: "undetected", 5: "detected"}
    r = G.compare(modelled, real)
    assert r["n"] == 5
    assert r["confusion"]["crash"] == {"crash": 1, "masked": 1}
    assert r["exact_agreement"] == pytest.approx(4 / 5)
    assert r["failure_agreement"] == pytest.approx(4 / 5)
    assert r["non_failure_identical"] == 1.0
    assert G.modelled_label(4, 1) == "crash" and G.modelled_label(4, 2) == "hang" and G.modelled_label(3, 0) == "undetected"
