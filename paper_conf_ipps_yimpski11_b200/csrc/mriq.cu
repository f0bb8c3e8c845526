// mriq.cu — MRI-Q (K2: PhiMag + Q) with HAUBERK detectors, for sm_100a.
//
// Abstract programs: DESIGN.md §3.3 (benchmark: Parboil MRI-Q; the paper names it at L503 and
// reports its value distributions, Fig. 10, and correctness rule, L2598-2603).
// B200 shape: k-space packed as float4 {kx, ky, kz, |phi|^2} by PhiMag, staged into shared memory
// with double-buffered 1-D bulk async copies; one voxel per thread; MUFU.SIN + MUFU.COS per pair
// (the binding pipe); loop detector = self-accumulator Qr (and Qi at maxvar 2) + counter.
#include "mriq_dev.cuh"

namespace hk {

// PhiMag (non-loop code: HAUBERK-NL only).  kv[k] = (kx, ky, kz, fmaf(im, im, re*re)).
template <bool NL>
__global__ void __launch_bounds__(256) mriq_phimag_kernel(const float* __restrict__ kx, const float* __restrict__ ky,
                                                         const float* __restrict__ kz, const float* __restrict__ pr,
                                                         const float* __restrict__ pi, float4* __restrict__ kv, int numK,
                                                         hk_control* cb, uint32_t z) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t chk = 0, alarm = 0;
  if (k < numK) {
    if (NL) { chk ^= (uint32_t)k; alarm |= ((int)((blockIdx.x ^ z) * blockDim.x + (threadIdx.x ^ z)) != k) ? AL_DUP : 0u; }
    const float re = pr[k];
    if (NL) { chk ^= fb(re); alarm |= (fb(pr[opq(k, z)]) != fb(re)) ? AL_DUP : 0u; }
    const float im = pi[k];
    if (NL) { chk ^= fb(im); alarm |= (fb(pi[opq(k, z)]) != fb(im)) ? AL_DUP : 0u; }
    const float pm = __fmaf_rn(im, im, __fmul_rn(re, re));
    if (NL) {
      chk ^= fb(pm);
      const float re2 = bf(fb(re) + z), im2 = bf(fb(im) + z);
      alarm |= (fb(__fmaf_rn(im2, im2, __fmul_rn(re2, re2))) != fb(pm)) ? AL_DUP : 0u;
    }
    const float lx = kx[k], ly = ky[k], lz = kz[k];
    if (NL) {
      chk ^= fb(lx); alarm |= (fb(kx[opq(k, z)]) != fb(lx)) ? AL_DUP : 0u;
      chk ^= fb(ly); alarm |= (fb(ky[opq(k, z)]) != fb(ly)) ? AL_DUP : 0u;
      chk ^= fb(lz); alarm |= (fb(kz[opq(k, z)]) != fb(lz)) ? AL_DUP : 0u;
    }
    kv[k] = make_float4(lx, ly, lz, pm);
    if (NL) {
      chk ^= opqf(re, z); chk ^= opqf(im, z); chk ^= opqf(pm, z); chk ^= (uint32_t)opq(k, z);
      chk ^= opqf(lx, z); chk ^= opqf(ly, z); chk ^= opqf(lz, z);
      if (chk) alarm |= AL_CHK;
    }
  }
  if (NL) fold_alarm(cb, alarm, (uint32_t)k);
}

template <int V, bool EXACT>
__global__ void __launch_bounds__(MQ_THREADS) mriq_kernel(const MQParams p) {
  __shared__ __align__(128) float4 tile[2][MQ_TILE];
  __shared__ __align__(8) uint64_t bar[2];
  mriq_body<V, EXACT, false, MQ_VPT, MQ_UNROLL>(p, tile, bar, blockIdx.x);
}

// ============================================================================================
// FI & FT replicas (blockIdx.y = replica).  See cp.cu for the scheme.
// ============================================================================================
// PhiMag replicas for PhiMag-site injections (sites 29-35): every thread runs the
// instrumented PhiMag program; the target thread gets the flip, guarded loads/stores (R16) and
// additive kv writes into the replica's zeroed buffer (R18); alarms fold into the replica's cb.
__global__ void __launch_bounds__(256) mriq_phimag_fi_kernel(const float* __restrict__ kx, const float* __restrict__ ky,
                                                            const float* __restrict__ kz, const float* __restrict__ pr,
                                                            const float* __restrict__ pi, float4* kv0, int numK,
                                                            const FaultRec* faults, hk_control* cb0, uint32_t z,
                                                            bool ft) {
  const int r = blockIdx.y;
  const FaultRec f = faults[r];
  float* kv = reinterpret_cast<float*>(kv0 + (int64_t)r * numK);
  hk_control* cb = cb0 + r;
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= numK) return;
  const bool mine = (k == f.thread);
  const uint64_t mask = f.mask;
  const int site = mine ? f.site : -1;
  uint32_t chk = 0, alarm = 0, fail = 0;
  int64_t e;
  const int64_t nk = numK;
  const uint64_t vb = VBASE;  // PhiMag's pointers are not injection sites: only indices move
  int32_t kidx = flip_i(k, site == 29, mask);
  chk ^= (uint32_t)kidx; alarm |= ((int)((blockIdx.x ^ z) * blockDim.x + (threadIdx.x ^ z)) != kidx) ? AL_DUP : 0u;
  float v[5];
  const float* src[5] = {pr, pi, kx, ky, kz};
  const int sid[5] = {30, 31, 33, 34, 35};
#pragma unroll
  for (int a = 0; a < 5; ++a) {
    if (f.real) e = kidx;  // R25: the corrupted index is used as is
    else if (!guard(vb, vb, kidx, 4, nk, &e)) { fail |= FL_CRASH; goto done; }
    v[a] = flip_f(src[a][e], site == sid[a], mask);
    chk ^= fb(v[a]); alarm |= (fb(src[a][e + z]) != fb(v[a])) ? AL_DUP : 0u;
    if (a == 1) {
      // pm right after re, im (program order of DESIGN §3.3)
    }
  }
  {
    const float re = v[0], im = v[1];
    float pm = flip_f(__fmaf_rn(im, im, __fmul_rn(re, re)), site == 32, mask);
    chk ^= fb(pm);
    const float re2 = bf(fb(re) + z), im2 = bf(fb(im) + z);
    alarm |= (fb(__fmaf_rn(im2, im2, __fmul_rn(re2, re2))) != fb(pm)) ? AL_DUP : 0u;
    if (f.real) e = kidx;
    else if (!guard(vb, vb, kidx, 16, nk, &e)) { fail |= FL_CRASH; goto done; }
    atomicAdd(kv + 4 * e + 0, v[2]);
    atomicAdd(kv + 4 * e + 1, v[3]);
    atomicAdd(kv + 4 * e + 2, v[4]);
    atomicAdd(kv + 4 * e + 3, pm);
    chk ^= opqf(v[0], z) ^ opqf(v[1], z) ^ opqf(pm, z) ^ opqf(v[2], z) ^ opqf(v[3], z) ^ opqf(v[4], z) ^ (uint32_t)opq(kidx, z);
    if (chk) alarm |= AL_CHK;
  }
done:
  if (fail) atomicOr(&cb->fail, fail);
  if (mine) cb->fault_applied = 1u;
  if (ft) fold_alarm(cb, alarm, (uint32_t)k);  // the FI-only binary has no detectors
}

// Items L = (replica, CTA) in fi_order; by default one per CTA of a (ncta, nrep) grid.  With
// HK_MQ_FI_PERSIST = c the grid holds c CTAs per SM that walk the items (experiment: leaves room
// for TPACF replica CTAs on the same SMs); the k-space mbarriers are invalidated between items.
template <int KIND, bool EXACT, bool FT>
__global__ void __launch_bounds__(MQ_FI_THREADS) mriq_fi_kernel(const MQFIParams q) {
  __shared__ __align__(128) float4 tile[2][MQ_FI_TILE];
  __shared__ __align__(8) uint64_t bar[2];
  const int64_t ncta = q.ncta, vpc = MQ_FI_VPT * (int64_t)blockDim.x, total = ncta * q.nrep;
  const int64_t step = (int64_t)gridDim.x * gridDim.y;
  for (int64_t L = (int64_t)blockIdx.y * gridDim.x + blockIdx.x; L < total; L += step) {
    int r;
    int64_t cta;
    const bool faulted = fi_order(L, ncta, q.nrep, [&](int rr) { return clamp_cta(q.faults[rr].thread / vpc, ncta); }, &r, &cta);
    const FaultRec f = q.faults[r];
    const int bxi = (int)cta;
    MQParams p = q.base;
    p.qr = q.out0 + (int64_t)r * q.stride;
    p.qi = p.qr + p.numX;
    p.cb = q.cb0 + r;
    if (KIND == MK_PHIMAG) p.kv = q.kv0 + (int64_t)r * p.numK;  // this replica's (possibly faulted) k-space
    if (KIND == MK_PHIMAG || !faulted) {
      mriq_body<FT ? (V_NL | V_L) : 0, EXACT, true, MQ_FI_VPT, MQ_FI_UNROLL, MQ_FI_TILE>(p, tile, bar, bxi);
      if (L + step < total) {  // next item re-initialises the barriers
        __syncthreads();
        if (threadIdx.x == 0) {
          asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(&bar[0])) : "memory");
          asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(&bar[1])) : "memory");
        }
        __syncthreads();
      }
    } else {
      mq_faulted_cta<KIND, EXACT, FT>(p, f, bxi);
    }
  }
}

// Unguarded replicas for the guardian (campaign mode 2, DESIGN R25): every thread runs the
// per-voxel program with REAL = true (Q-kernel kinds; PhiMag kinds use mriq_phimag_fi_kernel,
// which reads FaultRec::real, followed by the fault-free Q kernel).
template <bool EXACT>
__global__ void __launch_bounds__(256) mriq_real_kernel(const MQFIParams q, int kind) {
  const int r = blockIdx.y;
  const FaultRec f = q.faults[r];
  MQParams p = q.base;
  p.qr = q.out0 + (int64_t)r * q.stride;
  p.qi = p.qr + p.numX;
  p.cb = q.cb0 + r;
  ReplicaSinkF S{{p.qr, p.qi}, p.cb};
  const int32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= p.numX) return;
  const int32_t t_dup = (int32_t)((blockIdx.x ^ p.zz) * blockDim.x + (threadIdx.x ^ p.zz));
  const uint64_t qr = (uint64_t)(uintptr_t)p.qr, qi = (uint64_t)(uintptr_t)p.qi;
  switch (kind) {
#define K(k) case k: mriq_fi_program<k, EXACT, true>(p, f, t, t_dup, t == f.thread, qr, qi, S); break;
    K(MK_NL) K(MK_LIVE) K(MK_K) K(MK_KX) K(MK_KY) K(MK_KZ) K(MK_PM) K(MK_T1) K(MK_T2) K(MK_T) K(MK_R) K(MK_C)
    K(MK_S) K(MK_QR) K(MK_QI) K(MK_IT)
#undef K
    default: break;
  }
}

// ============================================================================================
// Replay accelerator: one CUDA thread per injection re-runs only the faulted voxel (DESIGN R22).
// ============================================================================================
struct MQReplayParams {
  MQParams base;
  const FaultRec* faults;
  int nrep;
  const float* golden;  // [qr; qi]
  const float* dM;
  hk_outcome* records;
  int64_t first;
  int64_t* counts;
  int64_t* site_counts;
};

template <int KIND, bool EXACT, bool FT>
__device__ __forceinline__ void mriq_replay_one(const MQReplayParams& q, const FaultRec& f) {
  const MQParams& p = q.base;
  const int32_t t = (int32_t)f.thread;
  ReplaySinkF<2> S;
  const uint64_t base_real = (uint64_t)(uintptr_t)q.golden;
  mriq_fi_program<KIND, EXACT, false, FT>(p, f, t, opq(t, p.zz), true, base_real, base_real + 4ull * (uint64_t)p.numX, S);
  bool wrong = false;
  float worst = 0.f;
  if (!S.fail) {
    const float M = *q.dM;
#pragma unroll
    for (int b = 0; b < 2; ++b) {  // own elements qr[t], qi[t]
      float v = 0.f;
      for (int w = 0; w < S.n; ++w) if (S.buf[w] == b && S.idx[w] == t) v = __fadd_rn(v, S.val[w]);
      fp_judge(v, q.golden[(int64_t)b * p.numX + t], M, &wrong, &worst);
    }
    for (int w = 0; w < S.n; ++w) {  // stray writes
      if (S.idx[w] == t) continue;
      bool first_write = true;
      for (int w2 = 0; w2 < w; ++w2) first_write &= !(S.idx[w2] == S.idx[w] && S.buf[w2] == S.buf[w]);
      if (!first_write) continue;
      const int64_t ge = (int64_t)S.buf[w] * p.numX + S.idx[w];
      float v = q.golden[ge];
      for (int w2 = w; w2 < S.n; ++w2) if (S.idx[w2] == S.idx[w] && S.buf[w2] == S.buf[w]) v = __fadd_rn(v, S.val[w2]);
      fp_judge(v, q.golden[ge], M, &wrong, &worst);
    }
  }
  emit_outcome(HK_MRIQ, f, wrong, S.alarm, S.fail, S.domain, S.margin, S.gap, worst, q.records, q.first, q.counts,
               q.site_counts);
}

template <bool EXACT, bool FT>
__global__ void __launch_bounds__(128) mriq_replay_all_kernel(const MQReplayParams q) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= q.nrep) return;
  const FaultRec f = q.faults[r];
  switch (mriq_site_kind_d(f.site)) {
#define K(k) case k: mriq_replay_one<k, EXACT, FT>(q, f); break;
    K(MK_NL) K(MK_LIVE) K(MK_K) K(MK_KX) K(MK_KY) K(MK_KZ) K(MK_PM) K(MK_T1) K(MK_T2) K(MK_T) K(MK_R) K(MK_C) K(MK_S)
    K(MK_QR) K(MK_QI) K(MK_IT)
#undef K
    default: break;
  }
}

// ============================================================================================
// Host launchers
// ============================================================================================
static MQParams mq_params(const hk_mriq_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples) {
  MQParams p{};
  p.x = a.x; p.y = a.y; p.z = a.z;
  p.kv = reinterpret_cast<const float4*>(a.kv_ws);
  p.qr = a.qr; p.qi = a.qi;
  p.cb = cb;
  p.samples = samples;
  p.R = R;
  p.numX = a.n_vox;
  p.numK = a.n_k;
  p.ndet = ndet;
  p.zz = opaque_zero();
  p.one = 1 + (int32_t)opaque_zero();
  return p;
}

cudaError_t mriq_phimag_launch(const hk_mriq_args& a, bool nl, hk_control* cb, cudaStream_t s) {
  if (a.n_k <= 0) return cudaSuccess;
  const int g = (a.n_k + 255) / 256;
  float4* kv = reinterpret_cast<float4*>(a.kv_ws);
  if (nl) mriq_phimag_kernel<true><<<g, 256, 0, s>>>(a.kx, a.ky, a.kz, a.phi_r, a.phi_i, kv, a.n_k, cb, opaque_zero());
  else mriq_phimag_kernel<false><<<g, 256, 0, s>>>(a.kx, a.ky, a.kz, a.phi_r, a.phi_i, kv, a.n_k, cb, opaque_zero());
  count_launch();
  return cudaGetLastError();
}

template <int V, bool EXACT>
static cudaError_t launch_mq_v(const MQParams& p, cudaStream_t s) {
  const int g = (p.numX + MQ_THREADS * MQ_VPT - 1) / (MQ_THREADS * MQ_VPT);
  if (g == 0) return cudaSuccess;
  TimedScope ts(HK_MRIQ, 0, (double)p.numX * (double)p.numK, s);
  mriq_kernel<V, EXACT><<<g, MQ_THREADS, 0, s>>>(p);
  count_launch();
  return cudaGetLastError();
}

cudaError_t mriq_launch(int vflags, const hk_mriq_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                        cudaStream_t s) {
  cudaError_t e = mriq_phimag_launch(a, (vflags & V_NL) != 0, cb, s);
  if (e != cudaSuccess) return e;
  const MQParams p = mq_params(a, R, ndet, cb, samples);
  const bool ex = a.exact != 0;
#define VV(v) case v: return ex ? launch_mq_v<v, true>(p, s) : launch_mq_v<v, false>(p, s);
  switch (vflags) { VV(0) VV(V_NL | V_L) VV(V_NL) VV(V_L) VV(V_PROF) }
#undef VV
  return cudaErrorInvalidValue;
}

int mriq_site_kind(int site) { return mriq_site_kind_d(site); }

template <int KIND, bool EXACT, bool FT>
static cudaError_t launch_mq_fi_k(const MQFIParams& q, int nrep, cudaStream_t s) {
  constexpr int vpc = MQ_FI_VPT * MQ_FI_THREADS;
  dim3 grid((q.base.numX + vpc - 1) / vpc, nrep);
  static const int persist = [] { const char* v = getenv("HK_MQ_FI_PERSIST"); return v ? atoi(v) : 0; }();
  if (persist > 0) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t items = (int64_t)grid.x * nrep, cap = (int64_t)persist * sms;
    if (items > cap) grid = dim3((unsigned)cap, 1);
  }
  TimedScope ts(HK_MRIQ, 1, (double)q.base.numX * (double)q.base.numK * nrep, s);
  mriq_fi_kernel<KIND, EXACT, FT><<<grid, MQ_FI_THREADS, 0, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

template <bool EXACT, bool FT>
static cudaError_t launch_mq_fi_e(int kind, const MQFIParams& q, int nrep, cudaStream_t s) {
  switch (kind) {
#define K(k) case k: return launch_mq_fi_k<k, EXACT, FT>(q, nrep, s);
    K(MK_NL) K(MK_LIVE) K(MK_K) K(MK_KX) K(MK_KY) K(MK_KZ) K(MK_PM) K(MK_T1) K(MK_T2) K(MK_T) K(MK_R) K(MK_C) K(MK_S)
    K(MK_QR) K(MK_QI) K(MK_IT) K(MK_PHIMAG)
#undef K
  }
  return cudaErrorInvalidValue;
}

cudaError_t mriq_replay_launch(int kind, bool ft, const hk_mriq_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
                               int nrep, const float* golden, const float* dM, hk_outcome* records, int64_t first,
                               int64_t* counts, int64_t* site_counts, cudaStream_t s) {
  if (nrep <= 0) return cudaSuccess;
  MQReplayParams q{};
  q.base = mq_params(a, R, ndet, nullptr, nullptr);
  q.faults = faults;
  q.nrep = nrep;
  q.golden = golden; q.dM = dM; q.records = records; q.first = first; q.counts = counts; q.site_counts = site_counts;
  (void)kind;
  TimedScope ts(HK_MRIQ, 2, (double)a.n_k * nrep, s);
  const unsigned g = (unsigned)((nrep + 127) / 128);
  if (a.exact) ft ? mriq_replay_all_kernel<true, true><<<g, 128, 0, s>>>(q) : mriq_replay_all_kernel<true, false><<<g, 128, 0, s>>>(q);
  else ft ? mriq_replay_all_kernel<false, true><<<g, 128, 0, s>>>(q) : mriq_replay_all_kernel<false, false><<<g, 128, 0, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

MQFIParams mriq_fi_params(const hk_mriq_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep, float* out0,
                          int64_t stride, hk_control* cb0, int threads, int vpt) {
  MQFIParams q{};
  q.base = mq_params(a, R, ndet, nullptr, nullptr);
  q.faults = faults;
  q.out0 = out0;
  q.stride = stride;
  q.cb0 = cb0;
  q.ncta = (a.n_vox + vpt * threads - 1) / (vpt * threads);
  q.nrep = nrep;
  return q;
}

cudaError_t mriq_fi_launch(int kind, bool ft, const hk_mriq_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep,
                           float* out0, int64_t stride, hk_control* cb0, float4* kv_rep, bool real, cudaStream_t s) {
  if (kind == MK_PHIMAG) {
    if (!kv_rep) return cudaErrorInvalidValue;
    cudaError_t e = cudaMemsetAsync(kv_rep, 0, sizeof(float4) * (size_t)a.n_k * nrep, s);
    if (e != cudaSuccess) return e;
    dim3 g((a.n_k + 255) / 256, nrep);
    mriq_phimag_fi_kernel<<<g, 256, 0, s>>>(a.kx, a.ky, a.kz, a.phi_r, a.phi_i, kv_rep, a.n_k, faults, cb0, opaque_zero(), ft);
    count_launch();
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  MQFIParams q = mriq_fi_params(a, R, ndet, faults, nrep, out0, stride, cb0, MQ_FI_THREADS);
  q.kv0 = kv_rep;
  if (real && kind != MK_PHIMAG) {
    dim3 grid((a.n_vox + 255) / 256, nrep);
    if (a.exact) mriq_real_kernel<true><<<grid, 256, 0, s>>>(q, kind);
    else mriq_real_kernel<false><<<grid, 256, 0, s>>>(q, kind);
    count_launch();
    return cudaGetLastError();
  }
  if (ft) return a.exact ? launch_mq_fi_e<true, true>(kind, q, nrep, s) : launch_mq_fi_e<false, true>(kind, q, nrep, s);
  return a.exact ? launch_mq_fi_e<true, false>(kind, q, nrep, s) : launch_mq_fi_e<false, false>(kind, q, nrep, s);
}

}  // namespace hk
