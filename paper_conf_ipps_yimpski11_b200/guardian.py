"""Guardian: real-crash / real-hang validation of the crash and hang models (SURVEY §8 row f4,
DESIGN R25).

The paper's FI controller runs each faulty program under supervision and "detects a crash or
hang of the GPU program" through its return status and a timeout (PAPER L1520-1528,
L1996-2007, L2636-2650).  The campaign kernels model both instead (R16: a corrupted address
outside its buffer is a crash; R17: a loop past 10x its golden trips is a hang), because a real
crash kills the CUDA context of the whole process.  This module measures how well the models
agree with the hardware:

* the injections run UNGUARDED (hauberk_inject_campaign mode 2) one at a time in a native child
  process (csrc/guardian_child.cpp -> hk_guardian_child), which reports each outcome on stdout;
* a lost CUDA context is a real crash (the child prints CRASH and exits 3; any other death of the
  child counts as a crash too); no answer within max(floor, 10 x golden kernel time) after BEGIN
  is a real hang — the child's process group is killed and a new child resumes after that
  injection;
* the modelled outcome of the same index comes from the ordinary guarded campaign.

Host orchestration only: every FI run is the library's kernels, in the child.
"""
from __future__ import annotations

import os
import selectors
import signal
import struct
import subprocess
import tempfile
import time
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
CHILD_PATH = os.path.join(_HERE, "hk_guardian_child")

CP, MRIQ, TPACF = 0, 1, 2
LABELS = ["masked", "detected_masked", "detected", "undetected", "crash", "hang"]


# ------------------------------------------------------------------------------------------------
# problem blob (format: csrc/guardian_child.cpp header)
# ------------------------------------------------------------------------------------------------
def _f32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.float32)).ravel()


def write_blob(path: str, bench: int, problem, ranges, seed: int, site_mask: int, nbits: int = 1, exact: int = 0):
    """Serialise one benchmark input + its profiled ranges (hauberk.Ranges) for the child."""
    iargs = [0] * 8
    fargs = [0.0] * 4
    if bench == CP:
        p = problem
        atoms = _f32(p.atoms) if p.n_atoms else np.zeros(4, np.float32)
        arrays = [atoms]
        iargs[:6] = [p.n_atoms, p.nx, p.ny, p.bx, p.by, p.unroll]
        fargs[:2] = [p.z0, p.h]
    elif bench == MRIQ:
        p = problem
        arrays = [_f32(a) for a in (p.x, p.y, p.z, p.kx, p.ky, p.kz, p.phi_r, p.phi_i)]
        iargs[:2] = [p.n_vox, p.n_k]
    elif bench == TPACF:
        p = problem
        arrays = [_f32(p.pts), _f32(p.edges)]
        iargs[:3] = [p.n, p.n_rand, p.edges.size - 1]
    else:
        raise ValueError(f"bad bench {bench}")
    with open(path, "wb") as f:
        f.write(b"HKGRD01\0")
        f.write(struct.pack("<4i", bench, exact, nbits, len(arrays)))
        f.write(struct.pack("<2Q", seed & (2**64 - 1), site_mask & (2**64 - 1)))
        f.write(bytes(ranges))
        f.write(struct.pack("<8i", *iargs))
        f.write(struct.pack("<4f", *fargs))
        for a in arrays:
            f.write(struct.pack("<Q", a.size))
            f.write(a.tobytes())


# ------------------------------------------------------------------------------------------------
# supervision
# ------------------------------------------------------------------------------------------------
@dataclass
class RealOutcome:
    index: int
    kind: str            # "done" | "crash" | "hang"
    cls: int = -1        # outcome class of a completed run (hk_outcome.cls)
    alarm: int = 0
    fail: int = 0
    detail: str = ""
    seconds: float = 0.0

    @property
    def label(self) -> str:
        if self.kind != "done":
            return self.kind
        return LABELS[self.cls] if 0 <= self.cls < 4 else "failure"


@dataclass
class Guardian:
    """Runs `indices` through child processes: [*child_cmd, blob, index_file, start_position]."""
    blob: str
    child_cmd: list = field(default_factory=lambda: [CHILD_PATH])
    floor_s: float = 2.0          # the timeout floor (L2636-2650: a hang is "no answer in time")
    factor: float = 10.0          # x the golden kernel time (R17's 10x)
    startup_s: float = 120.0      # child start-up (CUDA context creation, first call)
    restarts: int = 0
    log: list = field(default_factory=list)

    def _spawn(self, index_file: str, start: int):
        if not os.path.exists(self.child_cmd[0]) and self.child_cmd[0] == CHILD_PATH:
            raise FileNotFoundError(f"{CHILD_PATH} missing: run `make -C paper_conf_ipps_yimpski11_b200/csrc`")
        return subprocess.Popen([*self.child_cmd, self.blob, index_file, str(start)], stdout=subprocess.PIPE,
                                stderr=subprocess.DEVNULL, start_new_session=True)

    @staticmethod
    def _kill(proc):
        try:
            os.killpg(proc.pid, signal.SIGKILL)
        except (ProcessLookupError, PermissionError):
            pass
        try:
            proc.wait(timeout=30)
        except subprocess.TimeoutExpired:
            pass

    def run(self, indices) -> dict:
        indices = [int(n) for n in indices]
        out: dict[int, RealOutcome] = {}
        with tempfile.NamedTemporaryFile("w", suffix=".idx", delete=False) as f:
            f.write("\n".join(str(n) for n in indices) + "\n")
            index_file = f.name
        try:
            pos = 0
            while pos < len(indices):
                pos = self._one_child(index_file, indices, pos, out)
        finally:
            os.unlink(index_file)
        return out

    def _one_child(self, index_file, indices, pos, out) -> int:
        """One child from position `pos`; returns the position to resume from."""
        proc = self._spawn(index_file, pos)
        sel = selectors.DefaultSelector()
        sel.register(proc.stdout, selectors.EVENT_READ)
        buf = b""
        golden_s = None
        current, t_begin = None, None
        deadline = time.monotonic() + self.startup_s
        try:
            while True:
                timeout = deadline - time.monotonic()
                events = sel.select(timeout=max(timeout, 0.0)) if timeout > 0 else []
                if not events:
                    if current is None:
                        raise RuntimeError(f"guardian child did not start within {self.startup_s} s")
                    out[current] = RealOutcome(current, "hang", detail=f"no answer in {self._limit(golden_s):.2f} s",
                                               seconds=time.monotonic() - t_begin)
                    self.log.append(("hang", current))
                    self._kill(proc)
                    self.restarts += 1
                    return indices.index(current, pos) + 1
                chunk = os.read(proc.stdout.fileno(), 65536)
                if not chunk:  # EOF: the child exited
                    rc = proc.wait()
                    if current is None:  # between injections: finished, or died in set-up
                        if rc != 0:
                            raise RuntimeError(f"guardian child exited with status {rc} outside an injection")
                        return len(indices)
                    if current not in out:  # died without a CRASH line (e.g. a host-side signal)
                        out[current] = RealOutcome(current, "crash", detail=f"child exited with status {rc}",
                                                   seconds=time.monotonic() - t_begin)
                        self.log.append(("crash", current))
                    self.restarts += 1
                    return indices.index(current, pos) + 1
                buf += chunk
                while b"\n" in buf:
                    line, buf = buf.split(b"\n", 1)
                    w = line.decode(errors="replace").split()
                    if not w:
                        continue
                    if w[0] == "READY":
                        golden_s = float(w[1]) * 1e-6
                        deadline = time.monotonic() + self.startup_s
                    elif w[0] == "BEGIN":
                        current, t_begin = int(w[1]), time.monotonic()
                        deadline = t_begin + self._limit(golden_s)
                    elif w[0] == "DONE":
                        n = int(w[1])
                        out[n] = RealOutcome(n, "done", cls=int(w[2]), alarm=int(w[3]), fail=int(w[4]),
                                             seconds=time.monotonic() - t_begin)
                        current = None
                        deadline = time.monotonic() + self.startup_s
                    elif w[0] == "CRASH":
                        n = int(w[1])
                        out[n] = RealOutcome(n, "crash", detail=" ".join(w[2:]), seconds=time.monotonic() - t_begin)
                        self.log.append(("crash", n))
                    elif w[0] == "ERROR":
                        raise RuntimeError("guardian child: " + " ".join(w[1:]))
        finally:
            sel.close()
            if proc.poll() is None:
                self._kill(proc)

    def _limit(self, golden_s) -> float:
        return max(self.floor_s, self.factor * (golden_s or 0.0))


# ------------------------------------------------------------------------------------------------
# modelled vs real
# ------------------------------------------------------------------------------------------------
def modelled_label(cls: int, fail: int) -> str:
    """Label of a guarded campaign record: R16 crash / R17 hang, else the outcome class."""
    if fail & 1:
        return "crash"
    if fail & 2:
        return "hang"
    return LABELS[cls] if 0 <= cls < 4 else "failure"


def compare(modelled: dict, real: dict) -> dict:
    """modelled: {index: label}; real: {index: RealOutcome}.  Confusion matrix and agreement."""
    labels = LABELS + ["failure"]
    conf = {m: {r: 0 for r in labels} for m in labels}
    for n, m in modelled.items():
        if n in real:
            conf[m][real[n].label] += 1
    tot = sum(sum(r.values()) for r in conf.values())
    same = sum(conf[lab][lab] for lab in labels)
    fail_m = {"crash", "hang"}
    fail_agree = sum(conf[m][r] for m in labels for r in labels if (m in fail_m) == (r in fail_m))
    non_fail = sum(conf[m][r] for m in labels if m not in fail_m for r in labels)
    non_fail_same = sum(conf[lab][lab] for lab in labels if lab not in fail_m)
    return {
        "n": tot,
        "confusion": {m: {r: v for r, v in row.items() if v} for m, row in conf.items() if sum(row.values())},
        "exact_agreement": same / tot if tot else None,
        "failure_agreement": fail_agree / tot if tot else None,
        "non_failure_identical": (non_fail_same / non_fail) if non_fail else None,
    }


def validate(bench: int, problem, n_fail: int = 40, n_other: int = 20, scan: int = 3000, seed: int = 2011,
             floor_s: float = 2.0, exact: int = 0, device: str = "cuda", site_mask: int | None = None):
    """Sample injections of one benchmark (modelled failures and others, from a guarded campaign
    over [0, scan)), run them unguarded under the guardian and compare.  Returns a report dict."""
    import torch
    from . import hauberk as hk

    mk = [hk.CPDevice, hk.MRIQDevice, hk.TPACFDevice][bench]
    dev = mk.from_problem(problem, device, exact=exact)
    maxvar = 1
    R = hk.profile_ranges(dev, maxvar=maxvar)
    masks = list(hk.DEFAULT_SITE_MASKS)
    if site_mask is not None:
        masks[bench] = site_mask
    devs = [None, None, None]
    devs[bench] = dev
    rng = [None, None, None]
    rng[bench] = R
    counts = torch.zeros((3, 5), dtype=torch.int64, device=device)
    rec = hk.records_tensor(scan, device)
    hk.inject_campaign(bench, devs, rng, seed, 0, scan, counts, records=rec, exact=exact, site_masks=masks)
    torch.cuda.synchronize()
    recs = hk.records_numpy(rec)
    lab = {int(r["index"]): modelled_label(int(r["cls"]), int(r["fail"])) for r in recs}
    where = {int(r["index"]): (int(r["site"]), int(r["mask"])) for r in recs}
    fail_idx = [n for n, v in lab.items() if v in ("crash", "hang")][:n_fail]
    pick = np.random.default_rng(seed).permutation([n for n, v in lab.items() if v not in ("crash", "hang")])
    other_idx = [int(n) for n in pick[:n_other]]
    indices = sorted(fail_idx + other_idx)
    with tempfile.TemporaryDirectory() as td:
        blob = os.path.join(td, "problem.blob")
        write_blob(blob, bench, problem, R, seed, masks[bench], exact=exact)
        g = Guardian(blob, floor_s=floor_s)
        t0 = time.monotonic()
        real = g.run(indices)
        wall = time.monotonic() - t0
    rep = compare({n: lab[n] for n in indices}, real)
    by_bit: dict[int, list] = {}
    for n in indices:
        if lab[n] in ("crash", "hang") and n in real:
            bit = int(where[n][1]).bit_length() - 1
            e = by_bit.setdefault(bit, [0, 0])
            e[0] += 1
            e[1] += real[n].label in ("crash", "hang")
    rep["modelled_failures_by_bit"] = {str(k): {"n": v[0], "real_failure": v[1]} for k, v in sorted(by_bit.items())}
    rep.update({
        "bench": hk.BENCH_NAMES[bench], "seed": seed, "scan": scan, "sampled_failures": len(fail_idx),
        "sampled_others": len(other_idx), "child_restarts": g.restarts, "wall_s": round(wall, 2),
        "done_with_model_fail_bits": sum(1 for o in real.values() if o.kind == "done" and o.fail),
        "timeout_rule": f"max({floor_s} s, 10 x golden kernel time)",
        "records": [{"index": n, "site": where[n][0], "mask": hex(where[n][1]), "modelled": lab[n],
                     "real": real[n].label, "detail": real[n].detail, "seconds": round(real[n].seconds, 3)}
                    for n in indices if n in real],
    })
    return rep


def main(argv=None):
    import argparse
    import json

    import workloads as W

    ap = argparse.ArgumentParser(description="real-crash validation of the R16/R17 models (SURVEY f4)")
    ap.add_argument("--bench", choices=["cp", "mriq", "tpacf", "all"], default="all")
    ap.add_argument("--fail", type=int, default=40)
    ap.add_argument("--other", type=int, default=20)
    ap.add_argument("--scan", type=int, default=3000)
    ap.add_argument("--floor", type=float, default=2.0)
    ap.add_argument("--out", default=None)
    a = ap.parse_args(argv)
    probs = {"cp": (CP, W.cp_config1()), "mriq": (MRIQ, W.mriq_config2()), "tpacf": (TPACF, W.tpacf_config3())}
    names = list(probs) if a.bench == "all" else [a.bench]
    reports = {}
    for nm in names:
        b, p = probs[nm]
        reports[nm] = validate(b, p, a.fail, a.other, a.scan, floor_s=a.floor)
        r = reports[nm]
        print(nm, json.dumps({k: r[k] for k in ("n", "exact_agreement", "failure_agreement", "non_failure_identical",
                                                "confusion", "child_restarts", "wall_s")}), flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(reports, f, indent=1)


if __name__ == "__main__":
    main()
