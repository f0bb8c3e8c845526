// cp.cu — Coulombic potential (CP, K1) with HAUBERK detectors, for sm_100a.
//
// Per abstract thread (PAPER Fig. 9 L1242-1258 and the detector code at
// L1422-1429): U grid points of one row, E_j = sum_a q_a * rsqrt(dx_j^2 + dy^2 + dz^2).
// The B200 shape: atoms staged in shared memory by 1-D bulk async copies (TMA engine,
// cp.async.bulk + mbarrier, double buffered); every thread reads them with broadcast LDS.128;
// FP32 FADD/FFMA + MUFU.RSQ per interaction; detector state lives in registers; alarms are folded
// with warp votes and one atomic per warp.  MUFU.RSQ is the binding pipe (16/clk/SM).
#include "hk_internal.h"

namespace hk {

constexpr int CP_TILE = 1024;  // atoms per stage (16 KB); 2 stages

#ifndef HK_CP_AUNROLL
#define HK_CP_AUNROLL 16
#endif
constexpr int CP_AUNROLL = HK_CP_AUNROLL;  // atom-loop unroll of the protected loop

struct CPParams {
  const float4* atoms;  // (x, y, dz^2, q)
  float* grid;
  hk_control* cb;
  float* samples;
  DevRanges R;
  int32_t numatoms;
  float h;
  int32_t ndet;
  uint32_t z;    // runtime 0 (opaque)
  int32_t one;   // runtime 1 (opaque)
  int64_t nthreads;
  int32_t by0;  // single run: first block row of this launch (row sharding, hauberk_run_part)
};

// One CTA's worth of the protected loop.  V: variant flags; ADD: additive stores (R18, FI replicas).
template <int V, int U, bool EXACT, bool ADD>
__device__ __forceinline__ void cp_body(const CPParams& p, float4 (*tile)[CP_TILE], uint64_t* bar, int bxi, int byi) {
  constexpr bool NL = (V & V_NL) != 0, L = (V & V_L) != 0, PROF = (V & V_PROF) != 0;
  constexpr bool CNT = L || PROF;
  const int BX = blockDim.x, BY = blockDim.y;
  const int tx = threadIdx.x, ty = threadIdx.y;
  const uint32_t z = p.z;
  const uint32_t tid = (uint32_t)(((int64_t)byi * gridDim.x + bxi) * (BX * BY) + ty * BX + tx);
  uint32_t chk = 0, alarm = 0;
  const int32_t numatoms = p.numatoms;
  const float h = p.h;
  if (NL) chk ^= (uint32_t)numatoms ^ fb(h) ^ lohi_ptr(p.grid) ^ lohi_ptr(p.atoms);

  // ---- non-loop virtual variables: def; chk ^= v; duplicate; compare (L1017-1042)
  const int32_t xindex = bxi * (BX * U) + tx;
  if (NL) { chk ^= (uint32_t)xindex; alarm |= ((int32_t)((bxi ^ z) * (BX * U) + (tx ^ z)) != xindex) ? AL_DUP : 0u; }
  const int32_t yindex = byi * BY + ty;
  if (NL) { chk ^= (uint32_t)yindex; alarm |= ((int32_t)((byi ^ z) * BY + (ty ^ z)) != yindex) ? AL_DUP : 0u; }
  const int32_t nx = gridDim.x * BX * U;
  const int32_t outaddr = nx * yindex + xindex;
  if (NL) { chk ^= (uint32_t)outaddr; alarm |= ((int32_t)(nx * opq(yindex, z) + opq(xindex, z)) != outaddr) ? AL_DUP : 0u; }
  const float coorx = __fmul_rn(h, (float)xindex);
  if (NL) { chk ^= fb(coorx); alarm |= (fb(__fmul_rn(bf(fb(h) + z), (float)opq(xindex, z))) != fb(coorx)) ? AL_DUP : 0u; }
  const float coory = __fmul_rn(h, (float)yindex);
  if (NL) { chk ^= fb(coory); alarm |= (fb(__fmul_rn(bf(fb(h) + z), (float)opq(yindex, z))) != fb(coory)) ? AL_DUP : 0u; }
  const float gu = __fmul_rn(h, (float)BX);
  if (NL) { chk ^= fb(gu); alarm |= (fb(__fmul_rn(bf(fb(h) + z), (float)opq(BX, z))) != fb(gu)) ? AL_DUP : 0u; }
  if (NL) { chk ^= (uint32_t)opq(xindex, z); chk ^= (uint32_t)opq(yindex, z); }  // (iv) after last use

  // ---- the loop: self-accumulators E_j (no accumulator needed, L1277) + counter it (L1286)
  float E[U];
#pragma unroll
  for (int j = 0; j < U; ++j) E[j] = 0.0f;
  int32_t it = 0;
  const int lin = ty * BX + tx;
  const int ntiles = (numatoms + CP_TILE - 1) / CP_TILE;
  if (lin == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (lin == 0 && ntiles > 0) {
    const int cnt0 = min(CP_TILE, numatoms);
    bulk_g2s(tile[0], p.atoms, (uint32_t)cnt0 * 16u, &bar[0]);
  }
  for (int t = 0; t < ntiles; ++t) {
    const int buf = t & 1;
    if (lin == 0 && t + 1 < ntiles) {
      const int cnt1 = min(CP_TILE, numatoms - (t + 1) * CP_TILE);
      fence_proxy_async();
      bulk_g2s(tile[buf ^ 1], p.atoms + (size_t)(t + 1) * CP_TILE, (uint32_t)cnt1 * 16u, &bar[buf ^ 1]);
    }
    mbar_wait(&bar[buf], (uint32_t)(t >> 1) & 1u);
    const float4* A = tile[buf];
    const int cnt = min(CP_TILE, numatoms - t * CP_TILE);
#pragma unroll(CP_AUNROLL)
    for (int a = 0; a < cnt; ++a) {
      const float4 at = A[a];
      const float dy = __fsub_rn(coory, at.y);
      const float dyz2 = __fmaf_rn(dy, dy, at.z);
      float dx = __fsub_rn(coorx, at.x);
#pragma unroll
      for (int j = 0; j < U; ++j) {
        if (j) dx = __fadd_rn(dx, gu);
        const float r2 = __fmaf_rn(dx, dx, dyz2);
        const float s = hk_rsqrt<EXACT>(r2);
        E[j] = __fmaf_rn(at.w, s, E[j]);
      }
      if (CNT) it = count_inc(it, p.one);
    }
    __syncthreads();
  }

  // ---- after the loop: HauberkCheckEqual / HauberkCheckRange (L1428-1429)
  if (L && it != numatoms) alarm |= AL_COUNT;
  if (CNT && it != 0) {
    const float fit = (float)it;
#pragma unroll
    for (int d = 0; d < U; ++d) {
      if (d < p.ndet) {
        const float v = __fdiv_rn(E[d == 0 ? U - 1 : d - 1], fit);
        if (PROF) p.samples[(int64_t)d * p.nthreads + tid] = v;
        if (L && p.R.n[d] > 0 && !in_range<false>(p.R, d, v, nullptr)) {
          alarm |= AL_RANGE;
          record_outlier(p.cb, d, v);
        }
      }
    }
  }
  if (NL) { chk ^= opqf(coorx, z); chk ^= opqf(coory, z); chk ^= opqf(gu, z); }
#pragma unroll
  for (int j = 0; j < U; ++j) {
    float* dst = p.grid + (outaddr + j * BX);
    if (ADD) atomicAdd(dst, E[j]);
    else *dst = E[j];
  }
  if (NL) {
    chk ^= (uint32_t)opq(outaddr, z);
    chk ^= ((uint32_t)numatoms + z) ^ (fb(h) + z) ^ (lohi_ptr(p.grid) + z) ^ (lohi_ptr(p.atoms) + z);
    if (chk != 0) alarm |= AL_CHK;
  }
  if (NL || L) fold_alarm(p.cb, alarm, tid);
}

template <int V, int U, bool EXACT>
__global__ void __launch_bounds__(256) cp_kernel(const CPParams p) {
  __shared__ __align__(128) float4 tile[2][CP_TILE];
  __shared__ __align__(8) uint64_t bar[2];
  cp_body<V, U, EXACT, false>(p, tile, bar, blockIdx.x, blockIdx.y + p.by0);
}

// Uninstrumented pre-pass (row a1): (x, y, z, q) -> (x, y, (z - z0)^2, q).
__global__ void cp_prepass_kernel(const float4* __restrict__ in, float4* __restrict__ out, int n, float z0) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) {
    float4 a = in[i];
    const float dz = __fsub_rn(a.z, z0);
    a.z = __fmul_rn(dz, dz);
    out[i] = a;
  }
}

// ============================================================================================
// FI & FT campaign kernel (replica mode): blockIdx.z = replica.  CTAs that do not hold the
// faulted thread run the FT body unchanged (additive stores, R18); the faulted CTA runs the
// per-thread program with the single-kind hook, guarded accesses (R16) and the watchdog (R17).
// ============================================================================================
enum CPKind : int {
  CK_NL = 0, CK_LIVE, CK_ATOMID, CK_AX, CK_AY, CK_AZ, CK_AW, CK_DY, CK_DYZ2, CK_DX0, CK_DXJ, CK_R2, CK_S, CK_E, CK_IT,
  CK_COUNT
};

struct CPFIParams {
  CPParams base;       // grid/cb point at replica 0; per replica strides below
  const FaultRec* faults;
  int64_t grid_elems;  // replica stride (>= nx * ny)
  float* grid0;
  hk_control* cb0;
};

// Launch geometry of one abstract CP thread (CUDA indices of its replica CTA, or reconstructed
// from the abstract id in replay mode).
struct CPGeo {
  int tx, ty, bxi, byi, BX, BY, gx, gy;
};
__device__ __forceinline__ CPGeo cp_geo_here(int bxi, int byi) {
  return CPGeo{(int)threadIdx.x, (int)threadIdx.y, bxi, byi, (int)blockDim.x, (int)blockDim.y, (int)gridDim.x,
               (int)gridDim.y};
}
__device__ __forceinline__ CPGeo cp_geo_of(int64_t t, int BX, int BY, int gx, int gy) {
  const int64_t per = (int64_t)BX * BY, blk = t / per, r = t % per;
  return CPGeo{(int)(r % BX), (int)(r / BX), (int)(blk % gx), (int)(blk / gx), BX, BY, gx, gy};
}

// REAL: the guardian's unguarded variant (R25) — no R16 guards, no R17 watchdog.
// FT = false: the FI-only binary (row a7) — the same program without HAUBERK: no
// counter, no checks (the duplicate / checksum arithmetic feeds nothing and is removed).
template <int KIND, int U, bool EXACT, bool REAL = false, bool FT = true, class Sink>
__device__ void cp_fi_program(const CPParams& p, const FaultRec& f, const CPGeo& G, bool mine, uint64_t grid_real,
                              Sink& S) {
  const int BX = G.BX, BY = G.BY;
  const int tx = G.tx, ty = G.ty;
  const int bxi = G.bxi, byi = G.byi;
  const int64_t t = ((int64_t)byi * G.gx + bxi) * (BX * BY) + ty * BX + tx;
  const int64_t inst = mine ? f.inst : -1;
  const uint64_t mask = f.mask;
  const int site = f.site, sub = f.sub;
  const uint32_t z = p.z;
  const int64_t n_atoms = p.numatoms;
  const int64_t n_grid = (int64_t)G.gx * BX * U * G.gy * BY;
  const uint64_t atoms_real = (uint64_t)(uintptr_t)p.atoms;
  uint32_t chk = 0, alarm = 0, fail = 0, margin = 0xffffffffu;
  float gap = __int_as_float(0x7f800000);
  bool applied = false;

  int32_t numatoms = p.numatoms;
  float h = p.h;
  uint64_t pgrid = grid_real, patoms = atoms_real;
  chk ^= (uint32_t)numatoms ^ fb(h) ^ lohi(pgrid) ^ lohi(patoms);

  const bool nl = (KIND == CK_NL) && mine;
#define NLF(v, s) do { const bool _n = nl && site == (s); applied |= _n; v = flip_i(v, _n, mask); } while (0)
#define NLFF(v, s) do { const bool _n = nl && site == (s); applied |= _n; v = flip_f(v, _n, mask); } while (0)
  int32_t xindex = bxi * (BX * U) + tx;
  NLF(xindex, 0);
  chk ^= (uint32_t)xindex; alarm |= ((int32_t)((bxi ^ z) * (BX * U) + (tx ^ z)) != xindex) ? AL_DUP : 0u;
  int32_t yindex = byi * BY + ty;
  NLF(yindex, 1);
  chk ^= (uint32_t)yindex; alarm |= ((int32_t)((byi ^ z) * BY + (ty ^ z)) != yindex) ? AL_DUP : 0u;
  const int32_t nx = G.gx * BX * U;
  int32_t outaddr = (int32_t)((uint32_t)nx * (uint32_t)yindex + (uint32_t)xindex);
  NLF(outaddr, 2);
  chk ^= (uint32_t)outaddr;
  alarm |= ((int32_t)((uint32_t)nx * (uint32_t)opq(yindex, z) + (uint32_t)opq(xindex, z)) != outaddr) ? AL_DUP : 0u;
  float coorx = __fmul_rn(h, (float)xindex);
  NLFF(coorx, 3);
  chk ^= fb(coorx); alarm |= (fb(__fmul_rn(bf(fb(h) + z), (float)opq(xindex, z))) != fb(coorx)) ? AL_DUP : 0u;
  float coory = __fmul_rn(h, (float)yindex);
  NLFF(coory, 4);
  chk ^= fb(coory); alarm |= (fb(__fmul_rn(bf(fb(h) + z), (float)opq(yindex, z))) != fb(coory)) ? AL_DUP : 0u;
  float gu = __fmul_rn(h, (float)BX);
  NLFF(gu, 5);
  chk ^= fb(gu); alarm |= (fb(__fmul_rn(bf(fb(h) + z), (float)opq(BX, z))) != fb(gu)) ? AL_DUP : 0u;
  chk ^= (uint32_t)opq(xindex, z); chk ^= (uint32_t)opq(yindex, z);
#undef NLF
#undef NLFF

  float E[U];
#pragma unroll
  for (int j = 0; j < U; ++j) E[j] = 0.0f;
  int32_t it = 0;
  int32_t atomid = 0;
  const int64_t limit = fi_limit<REAL>(n_atoms, f.hang);
  constexpr bool real = REAL;
  for (int64_t i = 0;; ++i) {
    const bool now = (i == inst);
    if (KIND == CK_ATOMID) { applied |= now; atomid = flip_i(atomid, now, mask); }
    if (KIND == CK_LIVE && now) {
      applied = true;
      switch (site) {
        case 6: outaddr = flip_i(outaddr, true, mask); break;
        case 7: coorx = flip_f(coorx, true, mask); break;
        case 8: coory = flip_f(coory, true, mask); break;
        case 9: gu = flip_f(gu, true, mask); break;
        case 10: numatoms = flip_i(numatoms, true, mask); break;
        case 11: h = flip_f(h, true, mask); break;
        case 12: pgrid = flip_p(pgrid, true, mask); break;
        case 13: patoms = flip_p(patoms, true, mask); break;
        default: break;
      }
    }
    if (!(atomid < numatoms)) break;
    if (i >= limit) { fail |= FL_HANG; goto done; }
    const float4* pa;
    if (!fi_at(real, patoms, atoms_real, atomid, n_atoms, &pa)) { fail |= FL_CRASH; goto done; }
    {
      float4 at = __ldg(pa);
      if (KIND == CK_AX) { applied |= now; at.x = flip_f(at.x, now, mask); }
      if (KIND == CK_AY) { applied |= now; at.y = flip_f(at.y, now, mask); }
      if (KIND == CK_AZ) { applied |= now; at.z = flip_f(at.z, now, mask); }
      if (KIND == CK_AW) { applied |= now; at.w = flip_f(at.w, now, mask); }
      float dy = __fsub_rn(coory, at.y);
      if (KIND == CK_DY) { applied |= now; dy = flip_f(dy, now, mask); }
      float dyz2 = __fmaf_rn(dy, dy, at.z);
      if (KIND == CK_DYZ2) { applied |= now; dyz2 = flip_f(dyz2, now, mask); }
      float dx = __fsub_rn(coorx, at.x);
      if (KIND == CK_DX0) { applied |= now; dx = flip_f(dx, now, mask); }
#pragma unroll
      for (int j = 0; j < U; ++j) {
        const bool nj = now && (j == sub);
        if (j) {
          dx = __fadd_rn(dx, gu);
          if (KIND == CK_DXJ) { applied |= nj; dx = flip_f(dx, nj, mask); }
        }
        float r2 = __fmaf_rn(dx, dx, dyz2);
        if (KIND == CK_R2) { applied |= nj; r2 = flip_f(r2, nj, mask); }
        float s = hk_rsqrt<EXACT>(r2);
        if (KIND == CK_S) { applied |= nj; s = flip_f(s, nj, mask); }
        E[j] = __fmaf_rn(at.w, s, E[j]);
        if (KIND == CK_E) { applied |= nj; E[j] = flip_f(E[j], nj, mask); }
      }
    }
    if (FT) it = count_inc(it, p.one);
    if (KIND == CK_IT) { applied |= now; it = flip_i(it, now, mask); }
    atomid = (int32_t)((uint32_t)atomid + 1u);
  }
  if (FT && it != numatoms) alarm |= AL_COUNT;
  if (FT && it != 0) {
    const float fit = (float)it;
#pragma unroll
    for (int d = 0; d < U; ++d) {
      if (d < p.ndet && p.R.n[d] > 0) {
        const float v = __fdiv_rn(E[d == 0 ? U - 1 : d - 1], fit);
        if (!in_range<true>(p.R, d, v, &margin, &gap)) { alarm |= AL_RANGE; S.outlier(d, v); }
      }
    }
  }
  chk ^= opqf(coorx, z); chk ^= opqf(coory, z); chk ^= opqf(gu, z);
#pragma unroll
  for (int j = 0; j < U; ++j) {
    float* po;
    if (!fi_at(real, pgrid, grid_real, outaddr + j * BX, n_grid, &po)) { fail |= FL_CRASH; goto done; }
    S.store_p(0, po, reinterpret_cast<const float*>(grid_real), E[j]);
  }
  chk ^= (uint32_t)opq(outaddr, z);
  chk ^= ((uint32_t)numatoms + z) ^ (fb(h) + z) ^ (lohi(pgrid) + z) ^ (lohi(patoms) + z);
  if (chk != 0) alarm |= AL_CHK;
done:
  if (!FT) alarm = 0;
  S.finish(mine, alarm, fail, margin, gap, 0u, applied, (uint32_t)t);
}

template <int KIND, int U, bool EXACT, bool FT>
__global__ void __launch_bounds__(256) cp_fi_kernel(const CPFIParams q) {
  __shared__ __align__(128) float4 tile[2][CP_TILE];
  __shared__ __align__(8) uint64_t bar[2];
  const int64_t tpb = (int64_t)blockDim.x * blockDim.y, ncta = (int64_t)gridDim.x * gridDim.y;
  const int64_t L = ((int64_t)blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
  int r;
  int64_t cta;
  const bool faulted = fi_order(L, ncta, (int)gridDim.z, [&](int rr) { return clamp_cta(q.faults[rr].thread / tpb, ncta); },
                                &r, &cta);
  const FaultRec f = q.faults[r];
  CPParams p = q.base;
  p.grid = q.grid0 + (int64_t)r * q.grid_elems;
  p.cb = q.cb0 + r;
  const int bxi = (int)(cta % gridDim.x), byi = (int)(cta / gridDim.x);
  if (!faulted) {
    cp_body<FT ? (V_NL | V_L) : 0, U, EXACT, true>(p, tile, bar, bxi, byi);
  } else {
    const CPGeo G = cp_geo_here(bxi, byi);
    const int64_t t = ((int64_t)G.byi * G.gx + G.bxi) * (G.BX * G.BY) + G.ty * G.BX + G.tx;
    ReplicaSinkF S{{p.grid, nullptr}, p.cb};
    cp_fi_program<KIND, U, EXACT, false, FT>(p, f, G, t == f.thread, (uint64_t)(uintptr_t)p.grid, S);
  }
}

// Unguarded replicas for the guardian (campaign mode 2, DESIGN R25): every CTA runs the per-thread
// program with REAL = true; the site kind is a runtime switch (one injection per launch).
template <int U, bool EXACT>
__global__ void __launch_bounds__(256) cp_real_kernel(const CPFIParams q, int kind) {
  const int r = blockIdx.z;
  const FaultRec f = q.faults[r];
  CPParams p = q.base;
  p.grid = q.grid0 + (int64_t)r * q.grid_elems;
  p.cb = q.cb0 + r;
  const CPGeo G = cp_geo_here(blockIdx.x, blockIdx.y);
  const int64_t t = ((int64_t)G.byi * G.gx + G.bxi) * (G.BX * G.BY) + G.ty * G.BX + G.tx;
  ReplicaSinkF S{{p.grid, nullptr}, p.cb};
  const uint64_t gr = (uint64_t)(uintptr_t)p.grid;
  switch (kind) {
#define K(k) case k: cp_fi_program<k, U, EXACT, true>(p, f, G, t == f.thread, gr, S); break;
    K(CK_NL) K(CK_LIVE) K(CK_ATOMID) K(CK_AX) K(CK_AY) K(CK_AZ) K(CK_AW) K(CK_DY) K(CK_DYZ2) K(CK_DX0)
    K(CK_DXJ) K(CK_R2) K(CK_S) K(CK_E) K(CK_IT)
#undef K
    default: break;
  }
}

// ============================================================================================
// Replay accelerator (DESIGN R22): one CUDA thread per injection re-runs only the
// faulted abstract thread and classifies against the golden output patched with its writes
// (the thread's own elements lose the golden contribution, R18) — identical to the replica
// outcome because no other thread is affected by the fault.
// ============================================================================================
struct CPReplayParams {
  CPParams base;
  const FaultRec* faults;
  int nrep, BX, BY, gx, gy, bench;
  const float* golden;
  const float* dM;
  hk_outcome* records;
  int64_t first;
  int64_t* counts;
  int64_t* site_counts;
  uint8_t kind_of_site[64];
};

template <int KIND, int U, bool EXACT, bool FT>
__device__ __forceinline__ void cp_replay_one(const CPReplayParams& q, const FaultRec& f) {
  const CPGeo G = cp_geo_of(f.thread, q.BX, q.BY, q.gx, q.gy);
  ReplaySinkF<U> S;
  cp_fi_program<KIND, U, EXACT, false, FT>(q.base, f, G, true, (uint64_t)(uintptr_t)q.golden, S);
  bool wrong = false;
  float worst = 0.f;
  if (!S.fail) {
    const float M = *q.dM;
    const int32_t nx = q.gx * q.BX * U;
    const int64_t own0 = (int64_t)nx * (G.byi * q.BY + G.ty) + G.bxi * (q.BX * U) + G.tx;
    // own elements: golden contribution removed, then the faulted writes added (in program order)
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const int64_t e = own0 + (int64_t)j * q.BX;
      float v = 0.f;
      for (int w = 0; w < S.n; ++w) if (S.idx[w] == e) v = __fadd_rn(v, S.val[w]);
      fp_judge(v, q.golden[e], M, &wrong, &worst);
    }
    // stray writes into elements owned by other threads
    for (int w = 0; w < S.n; ++w) {
      const int64_t e = S.idx[w];
      const int64_t d = e - own0;
      if (d >= 0 && d % q.BX == 0 && d / q.BX < U) continue;  // own element (handled above)
      bool first_write = true;
      for (int w2 = 0; w2 < w; ++w2) first_write &= (S.idx[w2] != e);
      if (!first_write) continue;
      float v = q.golden[e];
      for (int w2 = w; w2 < S.n; ++w2) if (S.idx[w2] == e) v = __fadd_rn(v, S.val[w2]);
      fp_judge(v, q.golden[e], M, &wrong, &worst);
    }
  }
  emit_outcome(q.bench, f, wrong, S.alarm, S.fail, S.domain, S.margin, S.gap, worst, q.records, q.first, q.counts,
               q.site_counts);
}

// One CUDA thread per injection; the records arrive sorted by site kind (decode.cu), so warps
// take one branch of the switch.
template <int U, bool EXACT, bool FT>
__global__ void __launch_bounds__(128) cp_replay_all_kernel(const CPReplayParams q) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= q.nrep) return;
  const FaultRec f = q.faults[r];
  switch (q.kind_of_site[f.site & 63]) {
#define K(k) case k: cp_replay_one<k, U, EXACT, FT>(q, f); break;
    K(CK_NL) K(CK_LIVE) K(CK_ATOMID) K(CK_AX) K(CK_AY) K(CK_AZ) K(CK_AW) K(CK_DY) K(CK_DYZ2) K(CK_DX0)
    K(CK_DXJ) K(CK_R2) K(CK_S) K(CK_E) K(CK_IT)
#undef K
    default: break;
  }
}

// ============================================================================================
// Host launchers
// ============================================================================================
template <int V, int U, bool EXACT>
static cudaError_t launch_cp_v(const CPParams& p, dim3 grid, dim3 block, cudaStream_t s) {
  TimedScope ts(HK_CP, 0, (double)p.numatoms * (double)grid.x * grid.y * block.x * block.y * U, s);
  cp_kernel<V, U, EXACT><<<grid, block, 0, s>>>(p);
  count_launch();
  return cudaGetLastError();
}

template <int U, bool EXACT>
static cudaError_t launch_cp_u(int v, const CPParams& p, dim3 grid, dim3 block, cudaStream_t s) {
  switch (v) {
    case 0: return launch_cp_v<0, U, EXACT>(p, grid, block, s);
    case V_NL | V_L: return launch_cp_v<V_NL | V_L, U, EXACT>(p, grid, block, s);
    case V_NL: return launch_cp_v<V_NL, U, EXACT>(p, grid, block, s);
    case V_L: return launch_cp_v<V_L, U, EXACT>(p, grid, block, s);
    case V_PROF: return launch_cp_v<V_PROF, U, EXACT>(p, grid, block, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t cp_launch(int vflags, const hk_cp_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                      cudaStream_t s) {
  return cp_launch_rows(vflags, a, R, ndet, cb, samples, 0, a.ny, s);
}

// Grid rows [y0, y1) only (multiples of by): the same abstract threads as the whole run, by
// global block row (blockIdx.y + by0), so the rows come out bit-identical (single-run sharding).
cudaError_t cp_launch_rows(int vflags, const hk_cp_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                           int32_t y0, int32_t y1, cudaStream_t s) {
  if (a.n_atoms > 0) {
    cp_prepass_kernel<<<(a.n_atoms + 255) / 256, 256, 0, s>>>(reinterpret_cast<const float4*>(a.atoms),
                                                               reinterpret_cast<float4*>(a.atoms_ws), a.n_atoms, a.z0);
    count_launch();
  }
  CPParams p{};
  p.atoms = reinterpret_cast<const float4*>(a.atoms_ws);
  p.grid = a.grid;
  p.cb = cb;
  p.samples = samples;
  p.R = R;
  p.numatoms = a.n_atoms;
  p.h = a.h;
  p.ndet = ndet;
  p.z = opaque_zero();
  p.one = 1 + (int32_t)opaque_zero();
  p.nthreads = (int64_t)(a.nx / a.unroll) * a.ny;
  p.by0 = y0 / a.by;
  dim3 block(a.bx, a.by), grid(a.nx / (a.bx * a.unroll), (y1 - y0) / a.by);
  if (grid.y == 0) return cudaSuccess;
  const bool ex = a.exact != 0;
  switch (a.unroll) {
    case 1: return ex ? launch_cp_u<1, true>(vflags, p, grid, block, s) : launch_cp_u<1, false>(vflags, p, grid, block, s);
    case 2: return ex ? launch_cp_u<2, true>(vflags, p, grid, block, s) : launch_cp_u<2, false>(vflags, p, grid, block, s);
    case 4: return ex ? launch_cp_u<4, true>(vflags, p, grid, block, s) : launch_cp_u<4, false>(vflags, p, grid, block, s);
    case 8: return ex ? launch_cp_u<8, true>(vflags, p, grid, block, s) : launch_cp_u<8, false>(vflags, p, grid, block, s);
  }
  return cudaErrorInvalidValue;
}

// site -> (kind, sub) for U = 4 (DESIGN §3.2 catalogue)
int cp_site_kind(int site, int U, int* sub) {
  *sub = 0;
  if (site <= 5) return CK_NL;
  if (site <= 13) return CK_LIVE;
  if (site <= 21) return CK_ATOMID + (site - 14);
  const int S_DX = 22, S_R2 = 22 + (U - 1), S_S = S_R2 + U, S_E = S_S + U, S_IT = S_E + U;
  if (site < S_R2) { *sub = site - S_DX + 1; return CK_DXJ; }
  if (site < S_S) { *sub = site - S_R2; return CK_R2; }
  if (site < S_E) { *sub = site - S_S; return CK_S; }
  if (site < S_IT) { *sub = site - S_E; return CK_E; }
  return CK_IT;
}

template <int KIND, int U, bool EXACT, bool FT>
static cudaError_t launch_cp_fi_k(const CPFIParams& q, dim3 grid, dim3 block, cudaStream_t s) {
  TimedScope ts(HK_CP, 1, (double)q.base.numatoms * (double)q.base.nthreads * U * grid.z, s);
  cp_fi_kernel<KIND, U, EXACT, FT><<<grid, block, 0, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

template <int U, bool EXACT, bool FT>
static cudaError_t launch_cp_fi_e(int kind, const CPFIParams& q, dim3 grid, dim3 block, cudaStream_t s) {
  switch (kind) {
#define K(k) case k: return launch_cp_fi_k<k, U, EXACT, FT>(q, grid, block, s);
    K(CK_NL) K(CK_LIVE) K(CK_ATOMID) K(CK_AX) K(CK_AY) K(CK_AZ) K(CK_AW) K(CK_DY) K(CK_DYZ2) K(CK_DX0)
    K(CK_DXJ) K(CK_R2) K(CK_S) K(CK_E) K(CK_IT)
#undef K
  }
  return cudaErrorInvalidValue;
}

// One batch of `nrep` replicas of one kind: faults[0..nrep), outputs grid0[r], control blocks cb0[r].
cudaError_t cp_fi_launch(int kind, bool ft, const hk_cp_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep,
                         float* grid0, int64_t stride, hk_control* cb0, bool real, cudaStream_t s) {
  CPFIParams q{};
  q.base.atoms = reinterpret_cast<const float4*>(a.atoms_ws);
  q.base.R = R;
  q.base.numatoms = a.n_atoms;
  q.base.h = a.h;
  q.base.ndet = ndet;
  q.base.z = opaque_zero();
  q.base.one = 1 + (int32_t)opaque_zero();
  q.base.nthreads = (int64_t)(a.nx / a.unroll) * a.ny;
  q.faults = faults;
  q.grid_elems = stride;
  q.grid0 = grid0;
  q.cb0 = cb0;
  dim3 block(a.bx, a.by), grid(a.nx / (a.bx * a.unroll), a.ny / a.by, nrep);
  if (real) {
    if (a.unroll == 8) {
      if (a.exact) cp_real_kernel<8, true><<<grid, block, 0, s>>>(q, kind);
      else cp_real_kernel<8, false><<<grid, block, 0, s>>>(q, kind);
    } else if (a.unroll == 4) {
      if (a.exact) cp_real_kernel<4, true><<<grid, block, 0, s>>>(q, kind);
      else cp_real_kernel<4, false><<<grid, block, 0, s>>>(q, kind);
    } else {
      return cudaErrorInvalidValue;
    }
    count_launch();
    return cudaGetLastError();
  }
  if (a.unroll != 8 && a.unroll != 4) return cudaErrorInvalidValue;
  if (ft) {
    if (a.unroll == 8)
      return a.exact ? launch_cp_fi_e<8, true, true>(kind, q, grid, block, s) : launch_cp_fi_e<8, false, true>(kind, q, grid, block, s);
    return a.exact ? launch_cp_fi_e<4, true, true>(kind, q, grid, block, s) : launch_cp_fi_e<4, false, true>(kind, q, grid, block, s);
  }
  if (a.unroll == 8)
    return a.exact ? launch_cp_fi_e<8, true, false>(kind, q, grid, block, s) : launch_cp_fi_e<8, false, false>(kind, q, grid, block, s);
  return a.exact ? launch_cp_fi_e<4, true, false>(kind, q, grid, block, s) : launch_cp_fi_e<4, false, false>(kind, q, grid, block, s);
}

cudaError_t cp_replay_launch(int kind, bool ft, const hk_cp_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep,
                             const float* golden, const float* dM, hk_outcome* records, int64_t first, int64_t* counts,
                             int64_t* site_counts, cudaStream_t s) {
  if (nrep <= 0) return cudaSuccess;
  CPReplayParams q{};
  q.base.atoms = reinterpret_cast<const float4*>(a.atoms_ws);
  q.base.R = R;
  q.base.numatoms = a.n_atoms;
  q.base.h = a.h;
  q.base.ndet = ndet;
  q.base.z = opaque_zero();
  q.base.one = 1 + (int32_t)opaque_zero();
  q.base.nthreads = (int64_t)(a.nx / a.unroll) * a.ny;
  q.faults = faults;
  q.nrep = nrep;
  q.BX = a.bx; q.BY = a.by; q.gx = a.nx / (a.bx * a.unroll); q.gy = a.ny / a.by;
  q.bench = HK_CP;
  q.golden = golden; q.dM = dM; q.records = records; q.first = first; q.counts = counts; q.site_counts = site_counts;
  for (int site = 0; site < 64; ++site) {
    int sub = 0;
    q.kind_of_site[site] = (uint8_t)cp_site_kind(site, a.unroll, &sub);
  }
  (void)kind;
  const unsigned g = (unsigned)((nrep + 127) / 128);
  TimedScope ts(HK_CP, 2, (double)a.n_atoms * a.unroll * nrep, s);
  if (a.unroll == 8) {
    if (a.exact) ft ? cp_replay_all_kernel<8, true, true><<<g, 128, 0, s>>>(q) : cp_replay_all_kernel<8, true, false><<<g, 128, 0, s>>>(q);
    else ft ? cp_replay_all_kernel<8, false, true><<<g, 128, 0, s>>>(q) : cp_replay_all_kernel<8, false, false><<<g, 128, 0, s>>>(q);
  } else if (a.unroll == 4) {
    if (a.exact) ft ? cp_replay_all_kernel<4, true, true><<<g, 128, 0, s>>>(q) : cp_replay_all_kernel<4, true, false><<<g, 128, 0, s>>>(q);
    else ft ? cp_replay_all_kernel<4, false, true><<<g, 128, 0, s>>>(q) : cp_replay_all_kernel<4, false, false><<<g, 128, 0, s>>>(q);
  } else {
    return cudaErrorInvalidValue;
  }
  count_launch();
  return cudaGetLastError();
}

cudaError_t cp_prepass_launch(const hk_cp_args& a, cudaStream_t s) {
  if (a.n_atoms <= 0) return cudaSuccess;
  cp_prepass_kernel<<<(a.n_atoms + 255) / 256, 256, 0, s>>>(reinterpret_cast<const float4*>(a.atoms),
                                                             reinterpret_cast<float4*>(a.atoms_ws), a.n_atoms, a.z0);
  count_launch();
  return cudaGetLastError();
}

}  // namespace hk
