/*
 * hauberk.h — C ABI of the B200 (sm_100a) HAUBERK hot path.
 *
 * HAUBERK (Yim et al., IPDPS 2011; /root/reference/PAPER.md, "Lnnn" = line) derives lightweight
 * software detectors for silent data corruption in GPU kernels: duplication + an XOR checksum on
 * non-loop code (L986-1053 [§V.A]) and accumulator/counter value-range checks on loops
 * (L1216-1313, L1405-1508 [§V.B]), reported through a control block after the kernel ends
 * (L751-762, L1202-1214), and evaluates them with a software fault injector (L2083-2305 [§VII-VIII]).
 * This library implements that path for three Parboil-class kernels (CP, MRI-Q, TPACF) —
 * DESIGN.md §3 states the exact per-thread programs.
 *
 * Conventions (every entry point):
 *  - Pointers inside *_args structs, d_cb, d_samples, d_records, d_counts, d_site_counts are
 *    DEVICE pointers owned by the caller; the library never frees them.  Host structs
 *    (hk_ranges, hk_*_args, hk_campaign, hk_profile_opts) are read during the call only.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *  - Return value: HK_OK or an hk_status; no exception crosses the ABI.  Invalid arguments return
 *    HK_ERR_INVALID before anything is launched.  CUDA failures return HK_ERR_CUDA; the text is in
 *    hauberk_last_error() (thread-local).
 *  - A detected SDC is DATA, not an error: it is reported in hk_control.alarm (L757-759).
 *  - Device kernels are compiled for sm_100a only; there is no CPU fallback.
 */
#ifndef HAUBERK_H
#define HAUBERK_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define HK_ABI_VERSION 2

#if defined(__GNUC__)
#define HK_API __attribute__((visibility("default")))
#else
#define HK_API
#endif

typedef int32_t hk_status;
enum {
  HK_OK = 0,
  HK_ERR_INVALID = 1,      /* bad argument; nothing launched */
  HK_ERR_CUDA = 2,         /* a CUDA API call failed; see hauberk_last_error() */
  HK_ERR_NO_RANGES = 3,    /* FT variant without profiled ranges */
  HK_ERR_OOM = 4,          /* stream-ordered allocation failed */
  HK_ERR_UNSUPPORTED = 5,  /* shape/variant not compiled in (e.g. FI kernels only for unroll 4) */
  HK_ERR_PROFILE_NAN = 6,  /* a PROFILE sample was NaN/Inf */
  HK_ERR_GOLDEN_ALARM = 7  /* the fault-free golden run raised an alarm (ranges do not fit the input) */
};

enum { HK_CP = 0, HK_MRIQ = 1, HK_TPACF = 2, HK_MIXED = -1 };

/* Variants (PAPER Fig. 7, Table I): BASE = original program (overhead denominator);
 * FT = HAUBERK-NL + HAUBERK-L; FT_NL / FT_L = one detector family only (Fig. 13 columns);
 * PROFILE = accumulator/counter and per-thread samples of acc/it (no checks). */
enum { HK_BASE = 0, HK_FT = 1, HK_FT_NL = 2, HK_FT_L = 3, HK_PROFILE = 4 };

/* Outcome classes (L2377-2387). */
enum { HK_MASKED = 0, HK_DETECTED_MASKED = 1, HK_DETECTED = 2, HK_UNDETECTED = 3, HK_FAILURE = 4 };

/* hk_control.alarm bits / hk_control.fail bits. */
enum { HK_ALARM_DUP = 1, HK_ALARM_CHECKSUM = 2, HK_ALARM_RANGE = 4, HK_ALARM_COUNT = 8 };
enum { HK_FAIL_CRASH = 1, HK_FAIL_HANG = 2 };

/* Up to three correlation-point ranges per loop detector (L1489-1508). */
typedef struct { int32_t n; float lo[3], hi[3]; int32_t t_exp10; } hk_range_set;
/* Ranges of all loop detectors of one kernel; alpha widens them (L2073-2077, DESIGN R11). */
typedef struct { int32_t n_det; float alpha; hk_range_set det[8]; } hk_ranges;

/* Control block (L1202-1214): device-resident, written by the kernel, read by the caller after
 * the stream completes.  Reset by every hauberk_run_* call before its kernel. 96 bytes. */
typedef struct {
  uint32_t alarm;             /* OR of alarm bits of all threads */
  uint32_t fail;              /* FI only: modelled crash / hang (R16, R17) */
  uint32_t n_alarm_warps;     /* warps with >= 1 alarming thread */
  uint32_t first_thread;      /* smallest alarming abstract thread id (0xffffffff if none) */
  int32_t outlier_min_ord[8]; /* A11 (L1309-1313): ordinal (R8) range of out-of-range values */
  int32_t outlier_max_ord[8];
  uint32_t fault_applied;     /* FI only: the flip happened */
  uint32_t check_margin;      /* FI only: min ordinal distance of the faulted thread's checks to a bound */
  uint32_t domain;            /* FI only: faulted thread left the MUFU accuracy domain (R22c) */
  float check_gap;            /* FI only: min |check value - bound| of the faulted thread (R22a) */
} hk_control;

/* CP (K1; Fig. 9).  atoms: [n_atoms] (x, y, z, q); atoms_ws: [n_atoms] float4 scratch
 * for the (x, y, dz^2, q) pre-pass (both 16-byte aligned); grid: [ny][nx] output, every point
 * written by a whole run (the abstract program's "+=" onto a zeroed grid, R18; hauberk_run_part
 * zeroes its rows and adds).  Requires nx % (bx*unroll) == 0, ny % by == 0, bx*by <= 256 and a multiple of 32,
 * unroll in {1,2,4,8} (campaigns: unroll 4 or 8).  Detector d (maxvar = d + 1) checks the
 * self-accumulator E_{unroll-1} for d = 0, then E_0, E_1, ... (A6, DESIGN R12). */
typedef struct {
  const float* atoms; float* atoms_ws; int32_t n_atoms; float z0, h;
  int32_t nx, ny, bx, by, unroll; float* grid; int32_t exact;
} hk_cp_args;

/* MRI-Q (K2).  x,y,z: [n_vox]; kx..phi_i: [n_k]; kv_ws: [n_k] float4 scratch (PhiMag output);
 * qr, qi: [n_vox] outputs, every voxel written by a whole run (R18's "+=" onto zeroed outputs;
 * hauberk_run_part zeroes its voxels and adds). */
typedef struct {
  const float *x, *y, *z; int32_t n_vox, n_k;
  const float *kx, *ky, *kz, *phi_r, *phi_i; float* kv_ws; float *qr, *qi; int32_t exact;
} hk_mriq_args;

/* TPACF (K3).  pts: [(1+n_rand)][n][3] unit vectors (set 0 = data); edges: [n_bins+1] strictly
 * decreasing cos(angle) edges; hist: [(1+2*n_rand)][n_bins+2] u64 output (zeroed by the callee).
 * One abstract thread per (histogram h, point i) over all its partners; how the
 * kernels tile that loop is internal.  n_bins <= 30. */
typedef struct {
  const float* pts; const float* edges; int32_t n, n_rand, n_bins; unsigned long long* hist;
} hk_tpacf_args;

typedef struct { int32_t maxvar; int32_t t0_exp10; float alpha; } hk_profile_opts; /* defaults 1, -5, 1 */

/* Campaign (L2295-2305, L2370-2387).  Injections n in [first, first+count) decoded from
 * (seed, n) (DESIGN R14-R15); nbits = bits flipped per injection (0/1 = single-bit; 3, 6, 10, 15
 * reproduce Fig. 14's multi-bit masks, L2691); mode 0 = replica (every injection is a full program
 * run, the paper's definition), mode 1 = replay (one CUDA thread re-runs only the
 * faulted abstract thread and classifies the golden output patched with its writes — identical
 * outcomes; TPACF n_bins <= 32), mode 2 = unguarded replica (DESIGN R25, SURVEY
 * §8 f4: the faulted thread dereferences corrupted addresses itself and the R17 watchdog is off,
 * so a crash kills the calling process's CUDA context and a hang never returns — only for a
 * supervised child process, paper_conf_ipps_yimpski11_b200/guardian.py);
 * batch = replicas per launch (0 = auto); site_mask[b] bit s enables site s.
 * variant: HK_FIFT (0) = the FI&FT binary (HAUBERK-protected program with the injector) or
 * HK_FI_ONLY (1) = the FI binary (the original program with the injector: its
 * catalogue keeps only the original program's sites — hauberk_detector_site() — and its outcomes
 * are masked / undetected (SDC) / failure; ranges may be empty).  hang_factor: R17's T, a loop
 * running more than T x max(golden trips, 1) iterations is a hang (0 = 10). */
typedef struct {
  uint64_t seed; int64_t first, count; int32_t nbits; int32_t mode; int32_t batch; int32_t exact;
  uint64_t site_mask[3]; int32_t variant; int32_t hang_factor;
} hk_campaign;
enum { HK_FIFT = 0, HK_FI_ONLY = 1 };

/* One decoded injection (DESIGN R13-R15). */
typedef struct { int32_t site; int32_t hang; int64_t thread, inst; uint64_t mask; } hk_fault;

/* One classified injection (device array, `count` entries, slot = n - first). */
typedef struct {
  int64_t index; int32_t bench, site; int64_t thread, inst; uint64_t mask;
  int32_t cls; uint32_t alarm, fail, domain, margin; float worst; /* worst err/tol (R22b) */
  float gap; int32_t pad2;                                        /* check-value gap to a bound (R22a) */
} hk_outcome;

/* Run one benchmark kernel (plus its uninstrumented pre-pass / PhiMag) on `stream`.
 * variant: HK_BASE | HK_FT | HK_FT_NL | HK_FT_L | HK_PROFILE.  ranges: required for FT/FT_L
 * (HK_ERR_NO_RANGES otherwise), ranges->n_det detectors are checked.  d_cb: required except BASE.
 * d_samples: PROFILE only, [maxvar][threads] floats (maxvar = ranges ? ranges->n_det : 1).
 * Stream-asynchronous. */
HK_API hk_status hauberk_run_cp(const hk_cp_args* args, int32_t variant, const hk_ranges* ranges,
                         hk_control* d_cb, float* d_samples, void* stream);
HK_API hk_status hauberk_run_mriq(const hk_mriq_args* args, int32_t variant, const hk_ranges* ranges,
                           hk_control* d_cb, float* d_samples, void* stream);
HK_API hk_status hauberk_run_tpacf(const hk_tpacf_args* args, int32_t variant, const hk_ranges* ranges,
                            hk_control* d_cb, float* d_samples, void* stream);

/* Single-run sharding (the benchmarks' abstract threads are independent):
 * run only the partition units [begin, end) of one benchmark, bit-identical to the same units of
 * the whole run.  Units: CP = grid rows (begin, end multiples of by, or end = ny); MRI-Q = voxels
 * (the slice's abstract-thread ids, e.g. hk_control.first_thread, are slice-local); TPACF =
 * abstract threads g = h*n + i (histogram h in DD, RR_1..nr, DR_1..nr; point i), whose counts are
 * ADDED into a zeroed hist, so the partial histograms of a partition sum to the whole
 * (one all-reduce).  The callee zeroes only its own output part (CP rows, MRI-Q voxels; TPACF the
 * whole hist).  variant: HK_BASE / HK_FT / HK_FT_NL / HK_FT_L (profile over the whole input with
 * hauberk_profile_ranges and share the ranges).  hauberk_part_units returns the unit count and the
 * alignment granule.  HK_ERR_INVALID for a range outside [0, units) or misaligned. */
/* R-Naive's compare step: bitwise compare of two
 * device buffers of n_words 32-bit words (16-byte aligned), e.g. the outputs of two BASE runs on
 * two copies of the inputs.  d_cb is reset, then alarm |= HK_ALARM_DUP and first_thread = the
 * smallest differing word index if any word differs.  Stream-asynchronous. */
HK_API hk_status hauberk_compare(const void* d_a, const void* d_b, int64_t n_words, hk_control* d_cb, void* stream);

HK_API hk_status hauberk_part_units(int32_t bench, const void* args, int64_t* units, int64_t* granule);
HK_API hk_status hauberk_run_part(int32_t bench, const void* args, int32_t variant, const hk_ranges* ranges,
                                  hk_control* d_cb, int64_t begin, int64_t end, void* stream);

/* PROFILE run + threshold search (L1489-1508) -> out (host).  Synchronises `stream`.
 * args points to the bench's hk_*_args; opts may be NULL (defaults). */
HK_API hk_status hauberk_profile_ranges(int32_t bench, const void* args, const hk_profile_opts* opts,
                                 hk_ranges* out, void* stream);

/* Seeded injection campaign.  bench_mode: HK_CP/HK_MRIQ/HK_TPACF or HK_MIXED (bench = n mod 3).
 * args[b]/ranges[b]: per benchmark (unused ones may be NULL).  Runs the golden (fault-free FT)
 * program per benchmark, checks it raises no alarm, then launches the FI&FT replicas and the
 * classify epilogue.  d_counts: int64 [3][5] accumulated (+=); d_site_counts: nullable int64
 * [3][64][5] (+=); d_records: nullable [count].  Synchronises `stream` once at the start (golden
 * alarm check); the injections are enqueued asynchronously. */
HK_API hk_status hauberk_inject_campaign(int32_t bench_mode, const void* const args[3],
                                  const hk_ranges* const ranges[3], const hk_campaign* campaign,
                                  hk_outcome* d_records, int64_t* d_counts, int64_t* d_site_counts,
                                  void* stream);

/* The threshold search of hauberk_profile_ranges on caller-supplied HOST samples (e.g. the
 * PROFILE samples of several training inputs concatenated — the paper's multi-set training,
 * L2031-2036, L2654-2662).  Returns HK_ERR_PROFILE_NAN on a NaN/Inf sample. */
HK_API hk_status hauberk_profile_search(const float* samples, int64_t n, int32_t t0_exp10, hk_range_set* out);

/* Campaign session (the same campaign, prepared once): create validates, runs the golden programs,
 * checks they raise no alarm (synchronises `stream` once) and allocates the replica workspaces;
 * each run enqueues injections [first, first+count) on that stream without synchronising (the
 * device pointers inside the args must stay valid until destroy); destroy synchronises and frees.
 * hauberk_inject_campaign = create + run + destroy. */
typedef struct hk_campaign_session hk_campaign_session;
HK_API hk_status hauberk_campaign_create(int32_t bench_mode, const void* const args[3], const hk_ranges* const ranges[3],
                                         const hk_campaign* campaign, hk_campaign_session** out, void* stream);
HK_API hk_status hauberk_campaign_run(hk_campaign_session* session, int64_t first, int64_t count, hk_outcome* d_records,
                                      int64_t* d_counts, int64_t* d_site_counts);
HK_API void hauberk_campaign_destroy(hk_campaign_session* session);

/* Host-side decode of injections [first, first+count) (same rule the campaign uses; nbits as in
 * hk_campaign: <= 1 single-bit, k > 1 = k distinct bits, DESIGN R15 / NEXT f1; variant as in
 * hk_campaign: HK_FI_ONLY decodes over the original program's sites only). */
HK_API hk_status hauberk_decode(int32_t bench_mode, const void* const args[3], const uint64_t site_mask[3],
                         uint64_t seed, int32_t nbits, int32_t variant, int64_t first, int64_t count,
                         int32_t* bench_out, hk_fault* out);

/* Number of injection sites of a benchmark (unroll only matters for CP). */
HK_API int32_t hauberk_num_sites(int32_t bench, int32_t unroll);
/* 1 if `site` exists only because of HAUBERK (the loop detector's counter / accumulator and the
 * expected trip count: CP it, MRI-Q it, TPACF expect / acc / cnt), i.e. absent from the FI-only
 * binary's catalogue (row a7); 0 otherwise; -1 for an invalid bench / site. */
HK_API int32_t hauberk_detector_site(int32_t bench, int32_t unroll, int32_t site);

/* Device memory hauberk_campaign_create allocates for benchmark `bench` of campaign C besides the
 * caller's buffers: golden output, the batch's replica outputs and control blocks (C->batch, 0 =
 * auto; replay mode: 1), TPACF tables, MRI-Q per-replica k-space when PhiMag sites are enabled.
 * Each hauberk_campaign_run slice of `count` injections adds 40 B x count (fault records) in
 * replica mode, 81 B x count + 1 KB (device decode) in replay mode.  0 on invalid arguments. */
HK_API size_t hauberk_campaign_workspace_bytes(int32_t bench, const void* args, const hk_campaign* C);

/* ---- Evaluation and recovery arithmetic (host, no device work) ----
 * Campaign summary (R2): counts = int64 [5] of one campaign (sum the
 * rows of several benchmarks first).  coverage = P(masked or detected or failure) = 1 -
 * undetected / total; sdc = undetected / total (for an HK_FI_ONLY campaign: the unprotected SDC
 * rate of the original program, L211-213); detected = (detected + detected&masked) / total;
 * failure = failure / total.  HK_ERR_INVALID if the total is 0. */
typedef struct { double coverage, sdc, detected, failure; int64_t total; } hk_summary;
HK_API hk_status hauberk_summarize(const int64_t counts[5], hk_summary* out);
/* A11 ("calculates new ranges that include the outlier"; DESIGN R24): each of
 * the n finite values joins the range of its correlation class at the set's threshold
 * T = 10^t_exp10 (neg v < -T, zero |v| <= T, pos v > T); a class without a range gains one; ranges
 * stay in class order.  *added (nullable) = ranges created. */
HK_API hk_status hauberk_extend_ranges(hk_range_set* set, const float* values, int32_t n, int32_t* added);
/* The outlier interval a run recorded for detector d in a (host copy of a) control block: 0, 1 or
 * 2 values written to out[2] (*n); feed them to hauberk_extend_ranges on a diagnosed false alarm. */
HK_API hk_status hauberk_outliers(const hk_control* cb, int32_t d, float out[2], int32_t* n);
/* alpha controller: false-positive ratio > hi (0.10) -> alpha x 10;
 * < lo (0.05) -> alpha / 10 as long as alpha stays >= 1. */
HK_API float hauberk_alpha_update(float alpha, double fp_ratio, double hi, double lo);
/* Re-execution diagnosis of an alarm (Fig. 11): (alarm, fail) of the first run
 * and of its re-execution, and whether the two outputs are bitwise identical (hauberk_compare). */
enum { HK_DIAG_OK = 0, HK_DIAG_FALSE_ALARM = 1, HK_DIAG_TRANSIENT = 2, HK_DIAG_PERSISTENT = 3, HK_DIAG_FAILURE = 4 };
HK_API int32_t hauberk_diagnose(uint32_t alarm1, uint32_t fail1, uint32_t alarm2, uint32_t fail2, int32_t identical);

/* Free cached per-shape device tables (the TPACF single-run schedules) of the current device. */
HK_API void hauberk_release_caches(void);

HK_API const char* hauberk_strerror(hk_status s);
HK_API const char* hauberk_last_error(void);
HK_API int32_t hauberk_version(void);
/* Kernels this library has launched since load (process-wide counter, for bench accounting). */
HK_API uint64_t hauberk_launch_count(void);

/* Optional CUDA-event timing of the main kernels (cls 0: FT/BASE/PROFILE benchmark kernel,
 * cls 1: FI&FT campaign replicas, cls 2: replay kernels, cls 3: fused MRI-Q + TPACF replica
 * launches — each such launch is recorded under both benchmarks with that benchmark's work), recorded on each kernel's launch stream while enabled.
 * timing_read synchronises on the recorded events and returns the summed device time (ms),
 * the number of launches and the work (pairs / interactions) they computed, then forgets them.
 * Disabling drops unread records.  Not thread-safe; used by bench.py for roofline numbers. */
HK_API void hauberk_timing_enable(int32_t on);
HK_API hk_status hauberk_timing_read(int32_t bench, int32_t cls, double* ms, int64_t* launches, double* work);

#ifdef __cplusplus
}
#endif
#endif /* HAUBERK_H */
