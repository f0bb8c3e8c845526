// hk_internal.h — host-side declarations shared by the CUDA translation units of libhauberk.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/hauberk.h"
#include "hk_common.cuh"

namespace hk {

void count_launch();           // bumps the process-wide launch counter (hauberk_launch_count)

// Optional per-kernel CUDA-event timing (hauberk_timing_*): brackets the main / FI kernels of each
// benchmark with events on their launch stream.  cls 0 = FT/BASE/PROFILE main kernel, 1 = FI replicas.
// `work` = pairs (interactions) the launch computes, summed for the roofline numbers of bench.py.
struct TimedScope {
  TimedScope(int bench, int cls, double work, cudaStream_t s);
  ~TimedScope();
  void* start = nullptr;
  int bench, cls;
  double work;
  cudaStream_t s;
};
uint32_t opaque_zero();        // 0, read through a volatile so no compiler can fold it

// kernels of one benchmark run (pre-pass / PhiMag included); vflags = V_NL | V_L | V_PROF bits
cudaError_t cp_launch(int vflags, const hk_cp_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                      cudaStream_t s);
cudaError_t cp_launch_rows(int vflags, const hk_cp_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                           int32_t y0, int32_t y1, cudaStream_t s);
cudaError_t mriq_launch(int vflags, const hk_mriq_args& a, const DevRanges& R, int ndet, hk_control* cb,
                        float* samples, cudaStream_t s);
// TPACF: abstract threads [g0, g1) (g1 < 0: all); ws = tpacf_ws_bytes(a) bytes (bin table, single-run
// schedule counters, per-thread (acc, cnt) partial sums)
// Zeroes a.hist itself (in the table kernel) before adding the run's counts into it.
cudaError_t tpacf_launch(int vflags, const hk_tpacf_args& a, const DevRanges& R, int ndet, hk_control* cb,
                         float* samples, void* ws, cudaStream_t s, int32_t g0 = 0, int32_t g1 = -1);
size_t tpacf_ws_bytes(const hk_tpacf_args& a);
// Builds the bucket table in ws; the same launch zeroes the word ranges [z0, z0 + n0), [z1, z1 + n1).
cudaError_t tpacf_lut_build(const hk_tpacf_args& a, void* ws, cudaStream_t s, uint32_t* z0 = nullptr, int64_t n0 = 0,
                            uint32_t* z1 = nullptr, int64_t n1 = 0);
void tpacf_release_caches();
cudaError_t cp_prepass_launch(const hk_cp_args& a, cudaStream_t s);
cudaError_t mriq_phimag_launch(const hk_mriq_args& a, bool nl, hk_control* cb, cudaStream_t s);

// campaign replicas of one site kind
int cp_site_kind(int site, int U, int* sub);
int mriq_site_kind(int site);
int tpacf_site_kind(int site);
// ft = false: the FI-only binary (row a7): BASE fast CTAs, the FI program without detectors
cudaError_t cp_fi_launch(int kind, bool ft, const hk_cp_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep,
                         float* grid0, int64_t stride, hk_control* cb0, bool real, cudaStream_t s);
cudaError_t mriq_fi_launch(int kind, bool ft, const hk_mriq_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
                           int nrep, float* out0, int64_t stride, hk_control* cb0, float4* kv_rep, bool real,
                           cudaStream_t s);
constexpr int MRIQ_PHIMAG_SITE0 = 29;  // PhiMag NL sites 29-35 (replica mode only)
cudaError_t tpacf_fi_launch(int kind, bool ft, const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
                            int nrep, unsigned long long* hist0, hk_control* cb0, void* lut_ws, bool real,
                            cudaStream_t s);

// fused MRI-Q + TPACF replicas (mix.cu): rm MRI-Q replicas of Q-kernel site kinds (no PhiMag) and
// rt TPACF replicas in one launch; outputs / controls exactly as mriq_fi_launch + tpacf_fi_launch
bool mix_supported(const hk_mriq_args& m, const hk_tpacf_args& t);
cudaError_t mix_fi_launch(bool ft, const hk_mriq_args& ma, const DevRanges& mR, int mndet, const FaultRec* mfaults, int rm,
                          float* mout0, int64_t mstride, hk_control* mcb0, const hk_tpacf_args& ta, const DevRanges& tR, int tndet,
                          const FaultRec* tfaults, int rt, unsigned long long* thist0, hk_control* tcb0, void* tlut, cudaStream_t s);

// replay accelerator (one CUDA thread per injection; classification fused)
cudaError_t cp_replay_launch(int kind, bool ft, const hk_cp_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep,
                             const float* golden, const float* dM, hk_outcome* records, int64_t first, int64_t* counts,
                             int64_t* site_counts, cudaStream_t s);
cudaError_t mriq_replay_launch(int kind, bool ft, const hk_mriq_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
                               int nrep, const float* golden, const float* dM, hk_outcome* records, int64_t first,
                               int64_t* counts, int64_t* site_counts, cudaStream_t s);
cudaError_t tpacf_replay_launch(int kind, bool ft, const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
                                int nrep, const unsigned long long* golden, hk_outcome* records, int64_t first,
                                int64_t* counts, int64_t* site_counts, cudaStream_t s);

// decode.cu: device decode + counting sort by (bench, kind) for the replay path
size_t decode_ws_bytes(int64_t count);
cudaError_t decode_sort_launch(const DevCatalog cat[3], uint64_t seed, int64_t first, int64_t count, int32_t bench_mode,
                               int32_t nbits, int32_t hang, void* ws, FaultRec** sorted_out, cudaStream_t s);

// classify.cu
cudaError_t control_init_launch(hk_control* cb, int n, cudaStream_t s);
cudaError_t max_abs_launch(const float* g, int64_t n, float* d_out, cudaStream_t s);
cudaError_t compare_launch(const void* a, const void* b, int64_t n_words, hk_control* cb, cudaStream_t s);
cudaError_t classify_fp_launch(int bench, float* out0, int64_t elems, const float* golden, const float* d_M,
                               hk_control* cb0, const FaultRec* faults, int nrep, hk_outcome* records, int64_t first,
                               int64_t* counts, int64_t* site_counts, cudaStream_t s);
cudaError_t classify_tpacf_launch(unsigned long long* hist0, int nr, int nb, const unsigned long long* golden,
                                  hk_control* cb0, const FaultRec* faults, int nrep, hk_outcome* records,
                                  int64_t first, int64_t* counts, int64_t* site_counts, cudaStream_t s);

}  // namespace hk
