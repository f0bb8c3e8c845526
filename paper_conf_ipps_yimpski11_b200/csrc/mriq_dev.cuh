// mriq_dev.cuh — device building blocks of the MRI-Q kernels (mriq.cu) and of the fused
// MRI-Q + TPACF replica kernel (mix.cu).  DESIGN.md §3.3 / §6.2.
#pragma once

#include "hk_internal.h"

namespace hk {

constexpr int MQ_TILE = 1024;  // k-samples per stage (16 KB)
#ifndef HK_MQ_FI_THREADS
#define HK_MQ_FI_THREADS 64
#endif
#ifndef HK_MQ_FI_VPT
#define HK_MQ_FI_VPT 2
#endif
#ifndef HK_MQ_FI_TILE
#define HK_MQ_FI_TILE 1024
#endif
#ifndef HK_MQ_FI_UNROLL
#define HK_MQ_FI_UNROLL 8
#endif
constexpr int MQ_FI_THREADS = HK_MQ_FI_THREADS;  // campaign replicas: CTA size
constexpr int MQ_FI_VPT = HK_MQ_FI_VPT;          // voxels per CUDA thread in the replicas
constexpr int MQ_FI_UNROLL = HK_MQ_FI_UNROLL;
constexpr int MQ_FI_TILE = HK_MQ_FI_TILE;        // k-samples per stage in the replicas
#ifndef HK_MQ_UNROLL
#define HK_MQ_UNROLL 32
#endif
constexpr int MQ_UNROLL = HK_MQ_UNROLL;  // single-run kernel
#ifndef HK_MQ_THREADS
#define HK_MQ_THREADS 256
#endif
#ifndef HK_MQ_VPT
#define HK_MQ_VPT 1
#endif
constexpr int MQ_THREADS = HK_MQ_THREADS;  // single-run CTA size
constexpr int MQ_VPT = HK_MQ_VPT;          // single-run voxels per CUDA thread
constexpr float RINT_MAGIC = 12582912.0f;  // 1.5 * 2^23
constexpr float TWO_PI_F = 6.28318548202514648f;

struct MQParams {
  const float *x, *y, *z;
  const float4* kv;
  float *qr, *qi;
  hk_control* cb;
  float* samples;
  DevRanges R;
  int32_t numX, numK, ndet;
  uint32_t zz;  // runtime 0 (opaque)
  int32_t one;
};

// VPT voxels (abstract threads) per CUDA thread: voxel j of thread t in CTA b is
// b*(blockDim*VPT) + j*blockDim + t.  Each keeps its own registers, detectors and counter; they
// share every k-space load (VPT = 2 in the campaign replicas, 1 for the single-run kernel whose
// grid is small).
template <int V, bool EXACT, bool ADD, int VPT, int UNR = (VPT == 1 ? MQ_UNROLL : MQ_FI_UNROLL), int TILE = MQ_TILE>
__device__ __forceinline__ void mriq_body(const MQParams& p, float4 (*tile)[TILE], uint64_t* bar, int bxi) {
  constexpr bool NL = (V & V_NL) != 0, L = (V & V_L) != 0, PROF = (V & V_PROF) != 0;
  constexpr bool CNT = L || PROF;
  const uint32_t z = p.zz;
  const int32_t numK = p.numK;
  // the first k-space tile is requested before the voxel prologue so its latency overlaps it
  const int ntiles = (numK + TILE - 1) / TILE;
  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
    if (ntiles > 0) bulk_g2s(tile[0], p.kv, (uint32_t)min(TILE, numK) * 16u, &bar[0]);
  }
  int32_t xIndex[VPT];
  bool active[VPT];
  uint32_t chk[VPT], alarm[VPT];
  float sX[VPT], sY[VPT], sZ[VPT], Qr[VPT], Qi[VPT];
  int32_t it[VPT];
#pragma unroll
  for (int v = 0; v < VPT; ++v) {
    xIndex[v] = bxi * (blockDim.x * VPT) + v * blockDim.x + threadIdx.x;
    active[v] = xIndex[v] < p.numX;
    chk[v] = 0; alarm[v] = 0;
    sX[v] = sY[v] = sZ[v] = 0.f;
    Qr[v] = Qi[v] = 0.f;
    it[v] = 0;
    if (active[v]) {
      const int32_t xi = xIndex[v];
      if (NL) {
        chk[v] ^= (uint32_t)numK ^ lohi_ptr(p.kv) ^ lohi_ptr(p.qr) ^ lohi_ptr(p.qi) ^ lohi_ptr(p.x) ^ lohi_ptr(p.y) ^ lohi_ptr(p.z);
        chk[v] ^= (uint32_t)xi;
        alarm[v] |= ((int32_t)((bxi ^ z) * (blockDim.x * VPT) + v * blockDim.x + (threadIdx.x ^ z)) != xi) ? AL_DUP : 0u;
      }
      sX[v] = p.x[xi];
      if (NL) { chk[v] ^= fb(sX[v]); alarm[v] |= (fb(p.x[opq(xi, z)]) != fb(sX[v])) ? AL_DUP : 0u; }
      sY[v] = p.y[xi];
      if (NL) { chk[v] ^= fb(sY[v]); alarm[v] |= (fb(p.y[opq(xi, z)]) != fb(sY[v])) ? AL_DUP : 0u; }
      sZ[v] = p.z[xi];
      if (NL) { chk[v] ^= fb(sZ[v]); alarm[v] |= (fb(p.z[opq(xi, z)]) != fb(sZ[v])) ? AL_DUP : 0u; }
    }
  }
  __syncthreads();  // barrier init (above) visible to every waiter
  bool any_active = false;
#pragma unroll
  for (int v = 0; v < VPT; ++v) any_active |= active[v];
  for (int t = 0; t < ntiles; ++t) {
    const int buf = t & 1;
    if (threadIdx.x == 0 && t + 1 < ntiles) {
      fence_proxy_async();
      bulk_g2s(tile[buf ^ 1], p.kv + (size_t)(t + 1) * TILE, (uint32_t)min(TILE, numK - (t + 1) * TILE) * 16u,
               &bar[buf ^ 1]);
    }
    mbar_wait(&bar[buf], (uint32_t)(t >> 1) & 1u);
    if (any_active) {
      const float4* A = tile[buf];
      const int cnt = min(TILE, numK - t * TILE);
      const auto step = [&](const float4 k4) {
#pragma unroll
        for (int v = 0; v < VPT; ++v) {
          const float t1 = __fmul_rn(k4.x, sX[v]);
          const float t2 = __fmaf_rn(k4.y, sY[v], t1);
          const float tt = __fmaf_rn(k4.z, sZ[v], t2);
          const float m = __fsub_rn(__fadd_rn(tt, RINT_MAGIC), RINT_MAGIC);
          const float r = __fsub_rn(tt, m);
          const float ang = __fmul_rn(r, TWO_PI_F);
          const float c = hk_cos<EXACT>(ang);
          const float s = hk_sin<EXACT>(ang);
          Qr[v] = __fmaf_rn(k4.w, c, Qr[v]);
          Qi[v] = __fmaf_rn(k4.w, s, Qi[v]);
        }
      };
      // the iteration counter advances by UNR per unrolled group (the strength reduction a
      // compiler applies to an unrolled it++; the per-thread FI program keeps one increment per
      // iteration, where a fault can hit the counter)
      int a = 0;
#pragma unroll 1
      for (; a + UNR <= cnt; a += UNR) {
#pragma unroll
        for (int u = 0; u < UNR; ++u) step(A[a + u]);
        if (CNT)
#pragma unroll
          for (int v = 0; v < VPT; ++v) it[v] = count_inc(it[v], p.one * UNR);
      }
#pragma unroll 1
      for (; a < cnt; ++a) {
        step(A[a]);
        if (CNT)
#pragma unroll
          for (int v = 0; v < VPT; ++v) it[v] = count_inc(it[v], p.one);
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int v = 0; v < VPT; ++v) {
    if (!active[v]) continue;
    const int32_t xi = xIndex[v];
    if (L && it[v] != numK) alarm[v] |= AL_COUNT;
    if (CNT && it[v] != 0) {
      const float fit = (float)it[v];
#pragma unroll
      for (int d = 0; d < 2; ++d) {
        if (d < p.ndet) {
          const float val = __fdiv_rn(d == 0 ? Qr[v] : Qi[v], fit);
          if (PROF) p.samples[(int64_t)d * p.numX + xi] = val;
          if (L && p.R.n[d] > 0 && !in_range<false>(p.R, d, val, nullptr)) {
            alarm[v] |= AL_RANGE;
            record_outlier(p.cb, d, val);
          }
        }
      }
    }
    if (NL) { chk[v] ^= opqf(sX[v], z); chk[v] ^= opqf(sY[v], z); chk[v] ^= opqf(sZ[v], z); }
    if (ADD) { atomicAdd(p.qr + xi, Qr[v]); atomicAdd(p.qi + xi, Qi[v]); }
    else { p.qr[xi] = Qr[v]; p.qi[xi] = Qi[v]; }
    if (NL) {
      chk[v] ^= (uint32_t)opq(xi, z);
      chk[v] ^= ((uint32_t)numK + z) ^ (lohi_ptr(p.kv) + z) ^ (lohi_ptr(p.qr) + z) ^ (lohi_ptr(p.qi) + z) ^
                (lohi_ptr(p.x) + z) ^ (lohi_ptr(p.y) + z) ^ (lohi_ptr(p.z) + z);
      if (chk[v] != 0) alarm[v] |= AL_CHK;
    }
  }
#pragma unroll
  for (int v = 0; v < VPT; ++v)
    if ((NL || L) && active[v]) fold_alarm(p.cb, alarm[v], (uint32_t)xIndex[v]);
}

enum MQKind : int {
  MK_NL = 0, MK_LIVE, MK_K, MK_KX, MK_KY, MK_KZ, MK_PM, MK_T1, MK_T2, MK_T, MK_R, MK_C, MK_S, MK_QR, MK_QI, MK_IT,
  MK_PHIMAG,  // sites 29-35 (PhiMag NL): replica mode only
  MK_COUNT
};

__host__ __device__ __forceinline__ int mriq_site_kind_d(int site) {
  if (site <= 3) return MK_NL;
  if (site <= 14) return MK_LIVE;
  if (site >= 29) return MK_PHIMAG;
  return MK_K + (site - 15);
}

struct MQFIParams {
  MQParams base;
  const FaultRec* faults;
  float* out0;  // replica r: qr = out0 + r*stride, qi = qr + numX
  int64_t stride;
  const float4* kv0;  // PhiMag-site replicas: per-replica k-space [nrep][numK]
  hk_control* cb0;
  int64_t ncta;  // CTAs per replica (the replica kernel walks ncta * nrep items; the grid may be smaller)
  int32_t nrep;
};

// Per-thread FI&FT program of voxel t.  t_dup: the duplicate of N0 recomputed from launch indices
// (replica) or from the abstract id (replay); qr_real / qi_real: the buffers' true base addresses.
// REAL: the guardian's unguarded variant (R25) — no R16 guards, no R17 watchdog.
// FT = false: the FI-only binary (row a7): no counter, no checks.
template <int KIND, bool EXACT, bool REAL = false, bool FT = true, class Sink>
__device__ void mriq_fi_program(const MQParams& p, const FaultRec& f, int32_t t, int32_t t_dup, bool mine,
                                uint64_t qr_real, uint64_t qi_real, Sink& S) {
  const int64_t inst = mine ? f.inst : -1;
  const uint64_t mask = f.mask;
  const int site = f.site;
  const uint32_t z = p.zz;
  const int64_t nv = p.numX, nk = p.numK;
  const uint64_t kv_real = (uint64_t)(uintptr_t)p.kv;
  const uint64_t x_real = (uint64_t)(uintptr_t)p.x, y_real = (uint64_t)(uintptr_t)p.y, z_real = (uint64_t)(uintptr_t)p.z;
  uint32_t chk = 0, alarm = 0, fail = 0, margin = 0xffffffffu, domain = 0;
  float gap = __int_as_float(0x7f800000);
  bool applied = false;
  int32_t numK = p.numK;
  uint64_t pkv = kv_real, pqr = qr_real, pqi = qi_real, px = x_real, py = y_real, pz = z_real;
  chk ^= (uint32_t)numK ^ lohi(pkv) ^ lohi(pqr) ^ lohi(pqi) ^ lohi(px) ^ lohi(py) ^ lohi(pz);
  const bool nl = (KIND == MK_NL) && mine;
  int32_t xIndex = t;
  { const bool n = nl && site == 0; applied |= n; xIndex = flip_i(xIndex, n, mask); }
  chk ^= (uint32_t)xIndex;
  alarm |= (t_dup != xIndex) ? AL_DUP : 0u;
  float sX, sY, sZ, Qr = 0.f, Qi = 0.f;
  int32_t it = 0, k = 0;
  const float* pe;
  float* po;
  const int64_t limit = fi_limit<REAL>(nk, f.hang);
  constexpr bool real = REAL;
  if (!fi_at(real, px, x_real, xIndex, nv, &pe)) { fail |= FL_CRASH; goto done; }
  sX = __ldg(pe);
  { const bool n = nl && site == 1; applied |= n; sX = flip_f(sX, n, mask); }
  chk ^= fb(sX); alarm |= (fb(__ldg(pe + z)) != fb(sX)) ? AL_DUP : 0u;
  if (!fi_at(real, py, y_real, xIndex, nv, &pe)) { fail |= FL_CRASH; goto done; }
  sY = __ldg(pe);
  { const bool n = nl && site == 2; applied |= n; sY = flip_f(sY, n, mask); }
  chk ^= fb(sY); alarm |= (fb(__ldg(pe + z)) != fb(sY)) ? AL_DUP : 0u;
  if (!fi_at(real, pz, z_real, xIndex, nv, &pe)) { fail |= FL_CRASH; goto done; }
  sZ = __ldg(pe);
  { const bool n = nl && site == 3; applied |= n; sZ = flip_f(sZ, n, mask); }
  chk ^= fb(sZ); alarm |= (fb(__ldg(pe + z)) != fb(sZ)) ? AL_DUP : 0u;

  for (int64_t i = 0;; ++i) {
    const bool now = (i == inst);
    if (KIND == MK_K) { applied |= now; k = flip_i(k, now, mask); }
    if (KIND == MK_LIVE && now) {
      applied = true;
      switch (site) {
        case 4: xIndex = flip_i(xIndex, true, mask); break;
        case 5: sX = flip_f(sX, true, mask); break;
        case 6: sY = flip_f(sY, true, mask); break;
        case 7: sZ = flip_f(sZ, true, mask); break;
        case 8: numK = flip_i(numK, true, mask); break;
        case 9: pkv = flip_p(pkv, true, mask); break;
        case 10: pqr = flip_p(pqr, true, mask); break;
        case 11: pqi = flip_p(pqi, true, mask); break;
        case 12: px = flip_p(px, true, mask); break;
        case 13: py = flip_p(py, true, mask); break;
        case 14: pz = flip_p(pz, true, mask); break;
        default: break;
      }
    }
    if (!(k < numK)) break;
    if (i >= limit) { fail |= FL_HANG; goto done; }
    const float4* pk;
    if (!fi_at(real, pkv, kv_real, k, nk, &pk)) { fail |= FL_CRASH; goto done; }
    {
      float4 k4 = __ldg(pk);
      if (KIND == MK_KX) { applied |= now; k4.x = flip_f(k4.x, now, mask); }
      if (KIND == MK_KY) { applied |= now; k4.y = flip_f(k4.y, now, mask); }
      if (KIND == MK_KZ) { applied |= now; k4.z = flip_f(k4.z, now, mask); }
      if (KIND == MK_PM) { applied |= now; k4.w = flip_f(k4.w, now, mask); }
      float t1 = __fmul_rn(k4.x, sX);
      if (KIND == MK_T1) { applied |= now; t1 = flip_f(t1, now, mask); }
      float t2 = __fmaf_rn(k4.y, sY, t1);
      if (KIND == MK_T2) { applied |= now; t2 = flip_f(t2, now, mask); }
      float tt = __fmaf_rn(k4.z, sZ, t2);
      if (KIND == MK_T) { applied |= now; tt = flip_f(tt, now, mask); }
      const float m = __fsub_rn(__fadd_rn(tt, RINT_MAGIC), RINT_MAGIC);
      float r = __fsub_rn(tt, m);
      if (KIND == MK_R) { applied |= now; r = flip_f(r, now, mask); }
      if (!EXACT && fabsf(r) > 0.5f && fabsf(r) != __int_as_float(0x7f800000)) domain = 1;
      const float ang = __fmul_rn(r, TWO_PI_F);
      float c = hk_cos<EXACT>(ang);
      if (KIND == MK_C) { applied |= now; c = flip_f(c, now, mask); }
      float s = hk_sin<EXACT>(ang);
      if (KIND == MK_S) { applied |= now; s = flip_f(s, now, mask); }
      Qr = __fmaf_rn(k4.w, c, Qr);
      if (KIND == MK_QR) { applied |= now; Qr = flip_f(Qr, now, mask); }
      Qi = __fmaf_rn(k4.w, s, Qi);
      if (KIND == MK_QI) { applied |= now; Qi = flip_f(Qi, now, mask); }
    }
    if (FT) it = count_inc(it, p.one);
    if (KIND == MK_IT) { applied |= now; it = flip_i(it, now, mask); }
    k = (int32_t)((uint32_t)k + 1u);
  }
  if (FT && it != numK) alarm |= AL_COUNT;
  if (FT && it != 0) {
    const float fit = (float)it;
#pragma unroll
    for (int d = 0; d < 2; ++d) {
      if (d < p.ndet && p.R.n[d] > 0) {
        const float v = __fdiv_rn(d == 0 ? Qr : Qi, fit);
        if (!in_range<true>(p.R, d, v, &margin, &gap)) { alarm |= AL_RANGE; S.outlier(d, v); }
      }
    }
  }
  chk ^= opqf(sX, z); chk ^= opqf(sY, z); chk ^= opqf(sZ, z);
  if (!fi_at(real, pqr, qr_real, xIndex, nv, &po)) { fail |= FL_CRASH; goto done; }
  S.store_p(0, po, reinterpret_cast<const float*>(qr_real), Qr);
  if (!fi_at(real, pqi, qi_real, xIndex, nv, &po)) { fail |= FL_CRASH; goto done; }
  S.store_p(1, po, reinterpret_cast<const float*>(qi_real), Qi);
  chk ^= (uint32_t)opq(xIndex, z);
  chk ^= ((uint32_t)numK + z) ^ (lohi(pkv) + z) ^ (lohi(pqr) + z) ^ (lohi(pqi) + z) ^ (lohi(px) + z) ^ (lohi(py) + z) ^
         (lohi(pz) + z);
  if (chk != 0) alarm |= AL_CHK;
done:
  if (!FT) alarm = 0;
  S.finish(mine, alarm, fail, margin, gap, domain, applied, (uint32_t)t);
}


// The faulted CTA of a replica: every CUDA thread runs the per-voxel FI program for its MQ_FI_VPT
// voxels (the one holding the faulted abstract thread applies the fault).
template <int KIND, bool EXACT, bool FT, int VPT = MQ_FI_VPT>
__device__ __forceinline__ void mq_faulted_cta(const MQParams& p, const FaultRec& f, int bxi) {
  ReplicaSinkF S{{p.qr, p.qi}, p.cb};
#pragma unroll 1
  for (int vox = 0; vox < VPT; ++vox) {
    const int32_t t = bxi * (VPT * blockDim.x) + vox * blockDim.x + threadIdx.x;
    if (t < p.numX) {
      const int32_t t_dup = (int32_t)((bxi ^ p.zz) * (VPT * blockDim.x) + vox * blockDim.x + (threadIdx.x ^ p.zz));
      mriq_fi_program<KIND, EXACT, false, FT>(p, f, t, t_dup, t == f.thread, (uint64_t)(uintptr_t)p.qr, (uint64_t)(uintptr_t)p.qi, S);
    }
  }
}

// Replica-kernel parameters (mriq.cu; `threads` = CTA size of the kernel that will use them).
MQFIParams mriq_fi_params(const hk_mriq_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep, float* out0,
                          int64_t stride, hk_control* cb0, int threads, int vpt = MQ_FI_VPT);

}  // namespace hk
