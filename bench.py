#!/usr/bin/env python
"""bench.py — HAUBERK hot path on B200 (BASELINE.json metric:
"protected-kernel overhead % & SDC coverage %; injections/sec at 1/2/4/8 B200").

Step = one chunk of the config-5 campaign (mixed CP-s / MRI-Q / TPACF shapes of configs 1-3,
bench = n mod 3, seeded single-bit injections, replica mode: every injection is one full
FI&FT program run plus the classify epilogue — PAPER L2370-2371).  `value` = injections/s of the
whole job (all ranks; weak scaling: each rank takes its own `--per-rank` slice each step).
Alongside: the FT-vs-BASE overhead of configs 4 (CP-L), 2 (MRI-Q) and 3 (TPACF) (K back-to-back
launches per event pair), coverage of the FI&FT binary and the unprotected SDC rate of the FI-only
binary (row a7) over the same injection indices, roofline fractions, e2e (pinned-host inputs
copied in every step), and the CPU oracle: golden runs of configs 1-4, replay- and replica-mode
campaigns on 1 core and on every host core.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
  torchrun --nproc-per-node N bench.py --gpus N ...   (NCCL; max-over-ranks timing)
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "protected-kernel overhead % & SDC coverage %; injections/sec at 1/2/4/8 B200"
MUFU_PER_SM_CLK = 16     # B200: 16 MUFU lanes / clk / SM (4 per SMSP); measured: profiles/pipes_r01.json
LANES_PER_SM_CLK = 128   # FP32/INT32 lanes / clk / SM
N_SM = 148
TPACF_OPS_PER_PAIR = 11  # 3 FP (dot) + 5 compares (binary search over 22 bins) + 1 histogram add + 2 detector adds
OVH_K = 20               # launches per event pair in the overhead timing


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--per-rank", type=int, default=3000, help="injections per rank per step")
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--no-overhead", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-procs", type=int, default=0, help="oracle processes for the all-cores CPU line (0: all, <= 64)")
    ap.add_argument("--no-multibit", action="store_true")
    ap.add_argument("--replay-count", type=int, default=1000000, help="injections per rank for the replay-mode line")
    ap.add_argument("--no-fp-study", action="store_true")
    return ap.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            m = json.load(f)
        return float(m.get("sm_max_mhz", 1965.0)), "MEASURED_PEAKS.json sm_max_mhz"
    except Exception:
        return 1965.0, "fallback clocks.max.sm 1965 MHz (B200_PROFILING.md)"


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index: int):
        self.path = os.path.join(tempfile.gettempdir(), f"hk_clocks_{os.getpid()}_{index}.csv")
        self.index = index
        self.proc = None

    def start(self):
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                          "-lms", "200"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        self.proc.wait()
        rows = []
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) >= 9:
                try:
                    rows.append((float(f[1]), float(f[2]), f[5:9]))
                except ValueError:
                    pass
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        mx = max(r[1] for r in rows)
        load = [r for r in rows if r[0] > 0.5 * mx] or rows
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in load for i, v in enumerate(r[2]) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(r[0] for r in load), "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(rows), "samples_under_load": len(load)}


# ------------------------------------------------------------------------------------------------------
# reference arm: the CPU oracle, as it stands, on the same metric (replica-mode injections/s)
# ------------------------------------------------------------------------------------------------------
_ORACLE_SETUP = {}


def oracle_replica_sample(seed: int, first: int, count: int):
    """Time `count` consecutive config-5 injections in the oracle's replica mode (full program per injection).
    Inputs and the oracle's own profiled ranges are prepared once, outside the timing."""
    import oracle as O
    import workloads as W

    if not _ORACLE_SETUP:
        probs = [W.cp_config1(), W.mriq_config2(), W.tpacf_config3()]
        _ORACLE_SETUP["probs"] = probs
        _ORACLE_SETUP["R"] = [O.profile_ranges(b, probs[b]) for b in range(3)]
    probs, R = _ORACLE_SETUP["probs"], _ORACLE_SETUP["R"]
    per = {0: [], 1: [], 2: []}
    for n in range(first, first + count):
        b = n % 3
        t0 = time.perf_counter()
        O.campaign(-1, probs, R, seed, n, 1, exact=0, mode=0, records=False)
        per[b].append(time.perf_counter() - t0)
    return per


def _oracle_worker(job):
    seed, first, count = job
    return oracle_replica_sample(seed, first, count)


def oracle_all_cores(seed: int, first: int, procs: int):
    """The same oracle, unchanged, on `procs` forked worker processes (one per host core, no CUDA in
    the children), each timing one (CP-s, MRI-Q, TPACF) injection triple; throughput = injections / wall."""
    import multiprocessing as mp

    oracle_replica_sample(seed, 0, 0)  # inputs and ranges prepared in the parent, inherited by fork
    ctx = mp.get_context("fork")
    with ctx.Pool(procs) as pool:
        pool.map(_oracle_worker, [(seed, 0, 0)] * procs)  # workers started outside the timing
        t0 = time.perf_counter()
        res = pool.map(_oracle_worker, [(seed, first + 3 * w, 3) for w in range(procs)], chunksize=1)
        wall = time.perf_counter() - t0
    n = sum(len(p[b]) for p in res for b in range(3))
    return n / wall, n, wall


def cpu_model():
    try:
        for line in subprocess.check_output(["lscpu"], text=True).splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def oracle_golden_times():
    """The oracle's fault-free FI&FT-binary run (FT flags, own profiled ranges) of configs 1-3 in full
    and of config 4 on a row sample (1/64 of the CP-L grid threads, scaled), 1 core."""
    import numpy as np

    import oracle as O
    import workloads as W
    out = {}
    for name, b, p in (("cfg1_cp_s", 0, W.cp_config1()), ("cfg2_mriq", 1, W.mriq_config2()), ("cfg3_tpacf", 2, W.tpacf_config3())):
        R = O.profile_ranges(b, p)
        t0 = time.perf_counter()
        O.run(b, p, flags=O.FT, ranges=R, ndet=R.n_det)
        out[name] = {"s": round(time.perf_counter() - t0, 4), "sample": "whole run"}
    p4 = W.cp_config4(bx=16, by=16, unroll=8)
    nthr = (p4.nx // p4.unroll) * p4.ny
    tids = np.arange(0, nthr, 64)
    t0 = time.perf_counter()
    O.threads_out(O.CP, p4, tids)
    dt = time.perf_counter() - t0
    out["cfg4_cp_l"] = {"s": round(dt * nthr / tids.size, 2), "sample": f"{tids.size} of {nthr} abstract threads "
                        f"(every 64th; {dt:.2f} s measured, scaled x{nthr / tids.size:.0f})"}
    return out


def _oracle_replay_worker(job):
    """(seconds of a 3-injection call, seconds of a `count`-injection call): both rebuild the oracle's
    golden runs and catalogues, so their difference is the replay work of count - 3 injections."""
    seed, first, count = job
    import oracle as O
    probs, R = _ORACLE_SETUP["probs"], _ORACLE_SETUP["R"]
    t0 = time.perf_counter()
    O.campaign(-1, probs, R, seed, first, 3, mode=1, records=False)
    t1 = time.perf_counter()
    O.campaign(-1, probs, R, seed, first + 3, count, mode=1, records=False)
    return t1 - t0, time.perf_counter() - t1


def oracle_replay(seed: int, count: int, procs: int):
    """The oracle's replay-mode campaign (config-5 indices, bench = n mod 3) on 1 core and on `procs`
    forked processes; injections/s from the replay work alone (golden-run setup subtracted)."""
    import multiprocessing as mp
    oracle_replica_sample(seed, 0, 0)
    ts, tb = _oracle_replay_worker((seed, 0, count))
    one = (count - 3) / max(tb - ts, 1e-9)
    allc = None
    if procs > 1:
        ctx = mp.get_context("fork")
        with ctx.Pool(procs) as pool:
            res = pool.map(_oracle_replay_worker, [(seed, w * count, count) for w in range(procs)], chunksize=1)
        # the workers ran concurrently: total replay injections over the slowest worker's replay time
        allc = procs * (count - 3) / max(max(b - a for a, b in res), 1e-9)
    return one, allc, tb - ts


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    seed = 0x4841554245524B05
    import oracle as O
    O.build()
    step_t = []
    oracle_replica_sample(seed, 0, 0)  # setup (inputs, profiled ranges) outside the timing
    for s in range(args.warmup + args.steps):
        # one config-5 injection per step: index s, benchmark s mod 3 (the campaign's own mix)
        per = oracle_replica_sample(seed, s, 1)
        if s >= args.warmup:
            step_t.append(sum(sum(v) for v in per.values()))
    tot = sum(step_t)
    v = args.steps / tot
    line = {"metric": METRIC, "value": v, "unit": "injections/s", "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": "cfg5 mixed campaign (cfg1 CP-s / cfg2 MRI-Q / cfg3 TPACF), replica mode, 1-bit",
                       "injections_per_step": 1},
            "cpu_baseline": {"value": v, "unit": "injections/s", "cores": 1, "kind": "oracle",
                             "sample": f"config-5 injections {args.warmup}..{args.warmup + args.steps - 1} (bench = n mod 3), "
                                       "replica mode (one full program run each)"},
            "e2e": {"value": v, "unit": "injections/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------------------------------
# our arm
# ------------------------------------------------------------------------------------------------------
def _trimmed_mean(xs, frac=0.1):
    xs = sorted(xs)
    k = int(len(xs) * frac)
    core = xs[k:len(xs) - k] if len(xs) > 2 * k else xs
    return sum(core) / len(core)


def _nccl_version():
    try:
        v = torch.cuda.nccl.version()
        return ".".join(str(x) for x in v) if isinstance(v, (tuple, list)) else str(v)
    except Exception:  # noqa: BLE001 - diagnostics only
        return None


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import numpy as np
    import torch
    import torch.distributed as dist

    import workloads as W
    from paper_conf_ipps_yimpski11_b200 import hauberk as hk
    from paper_conf_ipps_yimpski11_b200 import parallel as par

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # one process per GPU; HK_DIST_BACKEND=gloo (test only) lets a multi-rank run share one GPU
    backend = os.environ.get("HK_DIST_BACKEND", "nccl")
    gpu = local % torch.cuda.device_count() if backend != "nccl" else local
    torch.cuda.set_device(gpu)
    dev = torch.device("cuda", gpu)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    hk.lib()
    sm_mhz_peak, clk_src = peaks()
    mufu_peak = N_SM * MUFU_PER_SM_CLK * sm_mhz_peak * 1e6
    lane_peak = N_SM * LANES_PER_SM_CLK * sm_mhz_peak * 1e6

    probs = [W.cp_config1(), W.mriq_config2(), W.tpacf_config3()]
    devs = [hk.CPDevice.from_problem(probs[0], dev), hk.MRIQDevice.from_problem(probs[1], dev),
            hk.TPACFDevice.from_problem(probs[2], dev)]
    ranges = [hk.profile_ranges(d) for d in devs]
    # C4: every rank profiled identical ranges (same seeded inputs, deterministic kernels)
    rv = torch.tensor([x for R in ranges for (_, rr) in R.as_list() for lohi in rr for x in lohi], dtype=torch.float64,
                      device=dev)
    ranges_identical = par.check_identical(rv)

    # ---- protected vs unprotected overhead (configs 4, 2, 3) and FT-kernel roofline
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    overhead, kernels = {}, {}
    if not args.no_overhead and rank == 0:
        # Fig. 13 columns: HAUBERK-NL, HAUBERK-L and HAUBERK vs the unprotected kernel
        cases = [("cp_cfg4", hk.CPDevice.from_problem(W.cp_config4(bx=16, by=16, unroll=8), dev), "xu", 1.0),
                 ("mriq_cfg2", devs[1], "xu", 2.0), ("tpacf_cfg3", devs[2], "alu", float(TPACF_OPS_PER_PAIR))]
        # R-Naive: the unprotected kernel run twice on two copies of
        # the data, then the outputs compared (hauberk_compare, on the device)
        twins = {"cp_cfg4": hk.CPDevice.from_problem(W.cp_config4(bx=16, by=16, unroll=8), dev),
                 "mriq_cfg2": hk.MRIQDevice.from_problem(W.mriq_config2(), dev),
                 "tpacf_cfg3": hk.TPACFDevice.from_problem(W.tpacf_config3(), dev)}
        variants = (hk.HK_BASE, hk.HK_FT_NL, hk.HK_FT_L, hk.HK_FT)
        for name, d, pipe, ops in cases:
            R = hk.profile_ranges(d)
            cb = hk.new_control(dev)
            # kernel-only device time per launch (library CUDA events around the main kernel)
            hk.timing_enable(True)
            t = {v: [] for v in variants}
            work = 0.0
            for rep in range(22):
                for v in variants:
                    flush.zero_()
                    hk.run(d, v, R, cb)
                    torch.cuda.synchronize()
                    ms, n, w = hk.timing_read(d.bench, 0)
                    if rep >= 2:
                        t[v].append(ms)
                        work = w
            hk.timing_enable(False)
            assert hk.read_control(cb).alarm == 0
            # overhead: K back-to-back hauberk_run_* calls per CUDA-event pair (event resolution ~1 us
            # per pair, so sub-us per-launch differences resolve), variants interleaved, median of rounds
            kt = {v: [] for v in variants}
            for rep in range(8):
                for v in variants:
                    flush.zero_()
                    k0, k1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    k0.record()
                    for _ in range(OVH_K):
                        hk.run(d, v, R, cb)
                    k1.record()
                    torch.cuda.synchronize()
                    if rep >= 1:
                        kt[v].append(k0.elapsed_time(k1) / OVH_K)
            # R-Naive: second BASE run on the twin copy, then the compare kernel (CUDA events)
            tw = twins[name]
            outs = lambda dd: [dd.output()] if not isinstance(dd.output(), tuple) else list(dd.output())
            ccb = hk.new_control(dev)
            tcmp = []
            hk.run(d, hk.HK_BASE, R, cb)
            for rep in range(12):
                hk.run(tw, hk.HK_BASE, R, ccb)
                flush.zero_()
                c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                c0.record()
                for oa, ob in zip(outs(d), outs(tw)):
                    hk.compare(oa, ob, ccb)
                c1.record()
                torch.cuda.synchronize()
                if rep >= 2:
                    tcmp.append(c0.elapsed_time(c1))
            naive_alarm = hk.read_control(ccb).alarm
            med = {v: statistics.median(t[v]) for v in variants}
            kmed = {v: statistics.median(kt[v]) for v in variants}
            tb, tf = med[hk.HK_BASE], med[hk.HK_FT]
            kb, kf = kmed[hk.HK_BASE], kmed[hk.HK_FT]
            peak = mufu_peak if pipe == "xu" else lane_peak
            ach = work * ops / (tf * 1e-3)
            overhead[name] = round(100.0 * (kf / kb - 1.0), 2)
            kernels[name] = {"base_ms": round(kb, 5), "ft_ms": round(kf, 5), "overhead_pct": overhead[name],
                             "overhead_nl_pct": round(100.0 * (kmed[hk.HK_FT_NL] / kb - 1.0), 2),
                             "overhead_l_pct": round(100.0 * (kmed[hk.HK_FT_L] / kb - 1.0), 2),
                             "timing": f"per-call device time of {OVH_K} back-to-back hauberk_run_* calls per CUDA-event pair "
                                       "(pre-pass / PhiMag / table kernels included, identical in every variant), median "
                                       "of 7 interleaved rounds, L2 flushed before each round",
                             "kernel_only_ms": {"base": round(tb, 5), "ft": round(tf, 5),
                                                "overhead_pct": round(100.0 * (tf / tb - 1.0), 2),
                                                "timing": "library CUDA events around the main kernel, median of 20 "
                                                          "launches, L2 flushed before each"},
                             "overhead_rnaive_pct": round(100.0 * ((2 * tb + statistics.median(tcmp)) / tb - 1.0), 2),
                             "rnaive_compare_ms": round(statistics.median(tcmp), 4), "rnaive_alarm": naive_alarm,
                             "pairs": work, "bound": "alu", "pipe": "xu (MUFU)" if pipe == "xu" else "fp32/int lanes",
                             "achieved_gops": round(ach / 1e9, 1), "peak_gops": round(peak / 1e9, 1),
                             "frac": round(ach / peak, 4), "base_frac": round(work * ops / (tb * 1e-3) / peak, 4)}
        del cases, twins

    # ---- campaign steps
    seed = 0x4841554245524B05
    counts = torch.zeros((3, 5), dtype=torch.int64, device=dev)
    scratch = torch.zeros((3, 5), dtype=torch.int64, device=dev)

    session = hk.CampaignSession(-1, devs, ranges, seed, batch=args.batch)

    def step(s, into):
        first, cnt = par.step_slice(s, rank, world, args.per_rank)
        session.run(first, cnt, into)

    for s in range(args.warmup):
        flush.zero_()
        step(args.steps + 1000 + s, scratch)  # warm-up slices outside the timed index range
    torch.cuda.synchronize()
    clocks = Clocks(gpu)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    l0 = hk.launch_count()
    hk.timing_enable(True)
    for s in range(args.steps):
        flush.zero_()  # L2 flush between timed steps (outside the events)
        ev[s][0].record()
        step(s, counts)
        ev[s][1].record()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = hk.launch_count() - l0
    fi_conc = {b: hk.timing_read(b, 1) for b in range(3)}
    mix_mq, mix_tp = hk.timing_read(1, 3), hk.timing_read(2, 3)  # the fused launches (same events, each one's work)
    hk.timing_enable(False)
    clk = clocks.stop()
    # Separate-kernel rooflines: the timed steps run MRI-Q and TPACF replicas in fused launches
    # (mix.cu) and CP replicas on a forked stream.  The same steps are replayed once more as a
    # serial session with one kernel per benchmark (HK_CONCURRENT=0, HK_FUSED=0) to time each
    # replica kernel alone; labelled in the JSON.
    os.environ["HK_CONCURRENT"] = "0"
    os.environ["HK_FUSED"] = "0"
    ser = hk.CampaignSession(-1, devs, ranges, seed, batch=args.batch)
    os.environ.pop("HK_CONCURRENT")
    os.environ.pop("HK_FUSED")
    ser.run(*par.step_slice(args.steps + 2000, rank, world, args.per_rank), scratch)  # warm-up
    torch.cuda.synchronize()
    ser_steps = max(1, min(args.steps, 3))
    ser_ms = 0.0
    hk.timing_enable(True)
    for s in range(ser_steps):
        flush.zero_()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record()
        first, cnt = par.step_slice(s, rank, world, args.per_rank)
        ser.run(first, cnt, scratch)
        a1.record()
        torch.cuda.synchronize()
        ser_ms += a0.elapsed_time(a1)
    fi = {b: hk.timing_read(b, 1) for b in range(3)}
    hk.timing_enable(False)
    ser.close()
    my_ms = sum(a.elapsed_time(b) for a, b in ev)
    t = torch.tensor([my_ms], dtype=torch.float64, device=dev)
    par.all_reduce_max(t)
    par.all_reduce_counts(counts)
    tot_ms = float(t.item())
    total_inj = args.per_rank * args.steps * world
    value = total_inj / (tot_ms * 1e-3)
    c = counts.cpu().numpy()

    # Separate replica kernels (serial pass): algorithmic ops / device time against their own pipe
    # (CP-s and MRI-Q: MUFU rsqrt / sin+cos per interaction; TPACF: TPACF_OPS_PER_PAIR lane ops per pair)
    def sep_roofline(b):
        ms, nl, work = fi[b]
        ops, peak, pipe = ((TPACF_OPS_PER_PAIR, lane_peak, "fp32/int lanes") if b == 2 else
                           ((1.0 if b == 0 else 2.0), mufu_peak, "xu (MUFU)"))
        ach = work * ops / (ms * 1e-3) if ms > 0 else 0.0
        return {"ms": round(ms, 3), "launches": nl, "work": work, "pipe": pipe, "achieved_gops": round(ach / 1e9, 1),
                "peak_gops": round(peak / 1e9, 1), "frac": round(ach / peak, 4), "serial_steps": ser_steps,
                "share_of_serial_step": round(ms / ser_ms, 3) if ser_ms else None}
    fi_split = {hk.BENCH_NAMES[b]: sep_roofline(b) for b in range(3)}

    # Dominant kernel of the timed step: the fused MRI-Q + TPACF replica launch (mix_fi_kernel).  Its
    # two roles bind different pipes (MRI-Q: MUFU sin/cos; TPACF: the fp32/int lanes), so its
    # roofline is the serial-equivalent fraction: the time both roles' algorithmic ops need, each at
    # its own pipe's peak, one after the other, over the measured time (1.0 = both at peak; above
    # 1.0 only by overlapping them).
    ms_mix, nl_mix, w_mq = mix_mq
    w_tp = mix_tp[2]
    if ms_mix > 0:
        t_mq = w_mq * 2.0 / mufu_peak
        t_tp = w_tp * TPACF_OPS_PER_PAIR / lane_peak
        sec = ms_mix * 1e-3
        roofline = {"bound": "alu", "pipe": "xu (MUFU) for the MRI-Q role + fp32/int lanes for the TPACF role",
                    "kernel": "mix_fi_kernel (fused MRI-Q + TPACF FI&FT replicas)",
                    "achieved": round((t_mq + t_tp) / sec, 4), "peak": 1.0, "unit": "pipe-s/s (serial-equivalent)",
                    "frac": round((t_mq + t_tp) / sec, 4),
                    "parts": {"mriq_xu": {"achieved_gops": round(w_mq * 2.0 / sec / 1e9, 1), "peak_gops": round(mufu_peak / 1e9, 1),
                                          "frac": round(t_mq / sec, 4), "interactions": w_mq},
                              "tpacf_lanes": {"achieved_gops": round(w_tp * TPACF_OPS_PER_PAIR / sec / 1e9, 1),
                                              "peak_gops": round(lane_peak / 1e9, 1), "frac": round(t_tp / sec, 4), "pairs": w_tp}},
                    "traffic": None, "launches": nl_mix, "share_of_step": round(ms_mix / my_ms, 3) if my_ms else None,
                    "measured": f"library CUDA events on the fused launch's stream inside the {args.steps} timed steps",
                    "peak_source": f"{N_SM} SMs x {MUFU_PER_SM_CLK} MUFU / {LANES_PER_SM_CLK} lanes per clk/SM x "
                                   f"{sm_mhz_peak:.0f} MHz ({clk_src})",
                    "limiter_ncu": "instruction issue (profiles/r02_ncu_mix_summary.txt): 85.8M warp instructions per MRI-Q + "
                                   "TPACF replica pair = 73.7 us at one instruction per clock per SM sub-partition; "
                                   "83.6 % of issue slots active"}
        tr_key = "mix_fi_kernel"
        n_rep = [sum(1 for st in range(args.steps)
                     for n in range(*(lambda f, c: (f, f + c))(*par.step_slice(st, rank, world, args.per_rank))) if n % 3 == b)
                 for b in (1, 2)]
        rpl = (n_rep[0] + n_rep[1]) / nl_mix if nl_mix else 0.0
    else:  # HK_FUSED=0: the largest separate replica kernel
        dom = max(range(3), key=lambda b: fi[b][0])
        sr = fi_split[hk.BENCH_NAMES[dom]]
        roofline = {"bound": "alu", "pipe": sr["pipe"], "kernel": f"{hk.BENCH_NAMES[dom]}_fi_kernel (FI&FT replicas)",
                    "achieved": sr["achieved_gops"], "peak": sr["peak_gops"], "unit": "Gop/s", "frac": sr["frac"],
                    "traffic": None, "launches": sr["launches"], "share_of_step": sr["share_of_serial_step"],
                    "measured": f"CUDA events on the launch stream over {ser_steps} serial step(s)"}
        tr_key = f"{hk.BENCH_NAMES[dom]}_fi_kernel"
        n_inj = sum(1 for st in range(ser_steps)
                    for n in range(*(lambda f, c: (f, f + c))(*par.step_slice(st, rank, world, args.per_rank))) if n % 3 == dom)
        rpl = n_inj / sr["launches"] if sr["launches"] else 0.0
    # traffic: DRAM bytes per launch of the same kernel from the committed ncu capture, scaled per
    # replica to this run's mean replicas per launch
    try:
        with open(os.path.join(ROOT, "profiles", "r02_traffic.json")) as f:
            tr = json.load(f).get(tr_key)
        if tr:
            roofline["traffic"] = round(tr["dram_bytes_per_launch"] / tr["replicas_per_launch"] * rpl)
            roofline["traffic_source"] = (f"{tr['source']}; scaled to {rpl:.1f} replicas per launch "
                                          f"({tr['dram_bytes_per_launch'] / tr['replicas_per_launch']:.0f} B per replica)")
    except (OSError, ValueError):
        pass

    # ---- e2e: pinned host inputs copied to the device every step, counts read back every step
    host = {}
    for d in devs:
        for k, v in vars(d).items():
            if isinstance(v, torch.Tensor) and k in ("atoms", "x", "y", "z", "kx", "ky", "kz", "phi_r", "phi_i", "pts", "edges"):
                host[(id(d), k)] = (v, v.cpu().pin_memory())
    h2d = sum(h.numel() * h.element_size() for _, h in host.values())
    e2e_steps = max(1, min(args.steps, 5))
    e2e_counts = torch.zeros((3, 5), dtype=torch.int64, device=dev)
    out_host = torch.zeros((3, 5), dtype=torch.int64).pin_memory()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for s in range(e2e_steps):
        for dt, ht in host.values():
            dt.copy_(ht, non_blocking=True)
        step(args.steps + 100 + s, e2e_counts)
        out_host.copy_(e2e_counts, non_blocking=True)
    e1.record()
    torch.cuda.synchronize()
    t2 = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
    par.all_reduce_max(t2)
    e2e_value = args.per_rank * e2e_steps * world / (float(t2.item()) * 1e-3)

    # ---- FI-only binary (row a7): the same injection indices over the original
    #      program's sites, no detectors -> the unprotected SDC rate (untimed)
    fionly = torch.zeros((3, 5), dtype=torch.int64, device=dev)
    with hk.CampaignSession(-1, devs, [None, None, None], seed, batch=args.batch, variant=hk.HK_FI_ONLY) as sf:
        for st_ in range(args.steps):
            first, cnt = par.step_slice(st_, rank, world, args.per_rank)
            sf.run(first, cnt, fionly)
        torch.cuda.synchronize()
    par.all_reduce_counts(fionly)
    cfo = fionly.cpu().numpy()

    # ---- CPU oracle baseline (rank 0 at N = 1 only; bounded samples)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        procs = args.cpu_procs if args.cpu_procs > 0 else min(64, len(os.sched_getaffinity(0)))
        per = oracle_replica_sample(seed, 0, 6)  # 2 x (CP-s, MRI-Q, TPACF)
        tm = [statistics.mean(per[b]) for b in range(3)]
        cpu = {"value": round(3.0 / sum(tm), 4), "unit": "injections/s", "cores": 1, "kind": "oracle",
               "cpu_model": cpu_model(), "host_cores": len(os.sched_getaffinity(0)),
               "sample": "6 config-5 injections (2 each CP-s / MRI-Q / TPACF), replica mode (full program run each), "
                         f"mean s/injection cp={tm[0]:.4f} mriq={tm[1]:.3f} tpacf={tm[2]:.3f}"}
        if procs > 1:
            v_all, n_all, wall = oracle_all_cores(seed, 300, procs)
            cpu["all_cores"] = {"value": round(v_all, 4), "unit": "injections/s", "cores": procs, "kind": "oracle",
                                "sample": f"{n_all} config-5 injections ({procs} forked processes x one CP-s / MRI-Q / "
                                          f"TPACF triple), replica mode, {wall:.1f} s wall"}
        rp1, rpall, rpt = oracle_replay(seed, 1500, procs)
        cpu["replay"] = {"value_1core": round(rp1, 1), "value_all_cores": round(rpall, 1) if rpall else None,
                         "unit": "injections/s", "cores": procs, "kind": "oracle",
                         "sample": f"1,497 config-5 injections per process (bench = n mod 3), replay mode (the faulted "
                                   f"abstract thread and its golden twin re-run, golden patched); {rpt:.2f} s of replay "
                                   "work on 1 core (a 3-injection call's golden-run setup subtracted)"}
        cpu["golden_runs_s"] = oracle_golden_times()

    session.close()

    # ---- replay accelerator (campaign mode 1): the full config-5 campaign, one CUDA
    #      thread per injection; reported separately from the faithful replica-mode headline
    replay = None
    if args.replay_count > 0:
        cr = torch.zeros((3, 5), dtype=torch.int64, device=dev)
        with hk.CampaignSession(-1, devs, ranges, seed, mode=1) as sr:
            first, cnt = par.shard(args.replay_count * world, rank, world)
            sr.run(first, cnt, torch.zeros((3, 5), dtype=torch.int64, device=dev))  # warm-up at full size (workspaces grow on first use)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            r0, r1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            t_host = time.perf_counter()
            r0.record()
            sr.run(first, cnt, cr)
            r1.record()
            torch.cuda.synchronize()
            t_host = time.perf_counter() - t_host
        tr = torch.tensor([r0.elapsed_time(r1)], dtype=torch.float64, device=dev)
        par.all_reduce_max(tr)
        par.all_reduce_counts(cr)
        crn = cr.cpu().numpy()
        replay = {"injections": args.replay_count * world, "ms": round(float(tr.item()), 2),
                  "injections_per_s": round(args.replay_count * world / (float(tr.item()) * 1e-3), 1),
                  "host_wall_s": round(t_host, 3), "coverage_pct": round(100.0 * hk.coverage(crn), 3),
                  "outcomes": {hk.BENCH_NAMES[b]: dict(zip(hk.CLASS_NAMES, crn[b].tolist())) for b in range(3)},
                  "note": "config-5 campaign indices [0, N) in replay mode; decode + counting sort by site kind on the device, then one launch per benchmark"}

    # ---- coverage vs number of flipped bits (Fig. 14; NEXT f1): the same
    #      injection indices with k-bit masks (untimed)
    multibit = {}
    if not args.no_multibit:
        for k in (3, 6, 10, 15):
            ck = torch.zeros((3, 5), dtype=torch.int64, device=dev)
            with hk.CampaignSession(-1, devs, ranges, seed, batch=args.batch, nbits=k) as sk:
                first, cnt = par.step_slice(0, rank, world, args.per_rank)
                sk.run(first, cnt, ck)
                torch.cuda.synchronize()
            par.all_reduce_counts(ck)
            cc = ck.cpu().numpy()
            multibit[str(k)] = {"coverage_pct": round(100.0 * hk.coverage(cc), 3),
                                "coverage_by_bench_pct": {hk.BENCH_NAMES[b]: round(100.0 * hk.coverage(cc[b]), 3) for b in range(3)},
                                "outcomes_pct": dict(zip(hk.CLASS_NAMES, (100.0 * cc.sum(0) / max(1, cc.sum())).round(2).tolist()))}
    # ---- Fig. 16 analogue (NEXT f2): false-positive ratio of fault-free runs on 2
    #      held-out synthetic datasets vs the number of training datasets (52 per program, 10 repeats)
    fp_study = {}
    if not args.no_fp_study and rank == 0:
        from paper_conf_ipps_yimpski11_b200 import recovery as rc
        makers = {"cp": lambda i: hk.CPDevice.from_problem(W.cp_problem(100, 64, 64, seed=60000 + i), dev),
                  "mriq": lambda i: hk.MRIQDevice.from_problem(W.mriq_problem(32, 3072, seed=70000 + i), dev),
                  "tpacf": lambda i: hk.TPACFDevice.from_problem(W.tpacf_problem(4096, 4, seed=80000 + i), dev)}
        for name, mk in makers.items():
            fp_study[name] = rc.false_positive_study(mk, n_sets=52, n_test=2, train_sizes=(1, 2, 5, 10, 20, 50), repeats=10)
            torch.cuda.empty_cache()

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "injections/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(tot_ms / args.steps, 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": "cfg5 mixed campaign: cfg1 CP-s (100 atoms, 64x64, U=4) / cfg2 MRI-Q (32^3 x 3072) / "
                                   "cfg3 TPACF (4096 x (1+4), 20 bins); replica mode (one full FI&FT program run per "
                                   "injection), single-bit, bench = n mod 3",
                       "per_rank_injections_per_step": args.per_rank, "parallelism": f"campaign-sharded x{world}",
                       "l2": "flushed between steps (512 MiB write, outside the events)"},
            "clocks": clk,
            # the process group the counters were all-reduced over (a multi-GPU run shows its NCCL ranks)
            "dist": {"backend": (backend if world > 1 else "none"),
                     "world_size": (dist.get_world_size() if dist.is_initialized() else 1),
                     "nccl_version": _nccl_version() if (world > 1 and backend == "nccl") else None},
            "e2e": {"value": round(e2e_value, 2), "unit": "injections/s", "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": 3 * 5 * 8, "steps": e2e_steps},
            "gpu_launches": int(launches),
            "roofline": roofline,
            "cpu_baseline": cpu,
            "coverage_pct": round(100.0 * hk.coverage(c), 3),
            "unprotected_sdc_pct": round(100.0 * hk.unprotected_sdc(cfo), 3),
            "protected_sdc_pct": round(100.0 * hk.summarize(c)["sdc"], 3),
            "fi_only_outcomes": {hk.BENCH_NAMES[b]: dict(zip(hk.CLASS_NAMES, cfo[b].tolist())) for b in range(3)},
            "fi_only_sdc_by_bench_pct": {hk.BENCH_NAMES[b]: round(100.0 * hk.unprotected_sdc(cfo[b]), 3) for b in range(3)},
            "outcomes": {hk.BENCH_NAMES[b]: dict(zip(hk.CLASS_NAMES, c[b].tolist())) for b in range(3)},
            "coverage_by_bench_pct": {hk.BENCH_NAMES[b]: round(100.0 * hk.coverage(c[b]), 3) for b in range(3)},
            "overhead_pct": overhead, "kernels": kernels, "fi_kernels": fi_split,
            "coverage_vs_bits": multibit,
            "replay": replay,
            "false_positive_vs_training_sets": fp_study,
            "outcomes_pct_1bit": dict(zip(hk.CLASS_NAMES, (100.0 * c.sum(0) / max(1, c.sum())).round(2).tolist())),
            "ranges_identical_across_ranks": ranges_identical,
            "paper_context": {"overhead_pct_avg7": 15.3, "coverage_pct_avg": 86.8, "hardware": "Tesla S1070 (GT200)",
                              "source": "PAPER.md L186-189, L2401-2404, L2480-2483"},
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
