// tpacf_dev.cuh — device building blocks of the TPACF kernels (tpacf.cu) and of the fused
// MRI-Q + TPACF replica kernel (mix.cu).  DESIGN.md §3.4 / §6.3.
#pragma once

#include "hk_internal.h"

namespace hk {

#ifndef HK_TP_NP_FI
#define HK_TP_NP_FI 4  // points per CUDA thread, campaign replicas
#endif
#ifndef HK_TP_NP_SR
#define HK_TP_NP_SR 4  // points per CUDA thread, single run
#endif
#ifndef HK_TP_MINB
#define HK_TP_MINB 6     // replicas: 37 KB of shared memory per CTA -> 6 CTAs per SM, 80 registers
#endif
#ifndef HK_TP_SR_T
#define HK_TP_SR_T 128  // single run: threads per CTA (128: six CTAs per SM; 256 / 512 measured slower)
#endif
#ifndef HK_TP_MINB_SR
#define HK_TP_MINB_SR (HK_TP_SR_T == 128 ? 6 : 1)  // single run BASE: CTAs per SM (128 threads: 37 KB, 80 registers)
#endif
#ifndef HK_TP_STASH
#define HK_TP_STASH 0x2  // single-run variants (bit V) that keep the points' exit state in local memory:
                         // FT_NL (its loop otherwise runs out of registers for independent lookups,
                         // 77.8 -> 67.6 us); FT and FT_L measured 2 us slower with it
#endif
#ifndef HK_TP_MINB_SR_NL
#define HK_TP_MINB_SR_NL (HK_TP_SR_T == 128 ? 6 : 1)  // FT_NL (its exit state in local memory, HK_TP_STASH):
                                                       // 80 registers, 6 CTAs per SM (61.4 vs 63.5 us at 5)
#endif
#ifndef HK_TP_MINB_SR_FT
#define HK_TP_MINB_SR_FT (HK_TP_SR_T == 128 ? 5 : 1)  // with detectors: 96 registers at 128 threads (at 80 the
                                                       // NL / L state spills)
#endif
#ifndef HK_TP_GROUP
#define HK_TP_GROUP 0  // partners per group of the unmasked loop (0: 4 for NP >= 4, else 8)
#endif
constexpr int TP_THREADS = 128;
constexpr int TP_WARPS = TP_THREADS / 32;
constexpr int TP_SR_T = HK_TP_SR_T;
constexpr int TP_TILE = 512;                // partners per shared-memory tile (6 KB)
constexpr int TP_LUT = 2048;                // u-buckets: sign, 8 exponent bits, 2 mantissa bits

struct TPParams {
  const float* pts;
  const float* edges;
  const uint8_t* lut;     // [TP_LUT] 4 * bmin per u-bucket; built by tpacf_lut_kernel
  const int* lut_ok;      // 1: every bucket holds at most one edge (else the binary search is used)
  unsigned long long* hist;
  hk_control* cb;
  float* samples;
  DevRanges R;
  int32_t* accg;          // single run: per abstract thread partial sums of acc and cnt (zeroed per run)
  int32_t* cntg;
  int32_t n, nr, nb, ndet;
  int32_t nblk;           // point blocks per histogram for the launching kernel's NP
  int32_t g0, g1;         // abstract threads [g0, g1) of this run (single-run sharding)
  uint32_t z;
  int32_t one, four, eight;  // runtime 1, 4 and 8 (opaque to the compiler)
};

// ---------------------------------------------------------------------------------------------
// Binning.  Definition: bin = #{e in [0, nb] : dot < edge[e]}, edges decreasing.
//  * tp_bin_search: branch-free 5-step binary search over the edges (padded with -inf).
//  * table: u = fl(1 - dot) is monotone (non-increasing) in dot and so is bin, so every bucket q of
//    u's top 11 bits maps to a contiguous dot interval [dmin, dmax].  The device builds
//    bmin = bin(dmax) per bucket and checks bin(dmin) <= bmin + 1; then bin = bmin + (dot < edge[bmin])
//    exactly (edge[bmin] = -inf past the last edge; NaN dots compare false, and the canonical NaN u
//    lands in a bucket whose bmin is bin(NaN) = 0).  The table holds 4 * bmin, the byte offset of
//    edge[bmin], so the edge load needs no address arithmetic.
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ int32_t tp_bin_search(const float* Es, float dot) {
  int32_t b = 0;
#pragma unroll
  for (int s = 16; s >= 1; s >>= 1) b += (dot < Es[b + s - 1]) ? s : 0;
  return b;
}
// 4 * bin through the byte table L and the edges at the shared byte address eb (uniform)
__device__ __forceinline__ uint32_t tp_b4_lut(const uint8_t* __restrict__ L, uint32_t eb, float dot) {
  const float u = __fsub_rn(1.0f, dot);
  const uint32_t b4 = L[fb(u) >> 21];
  float e;
  asm("ld.shared.f32 %0, [%1];" : "=f"(e) : "r"(eb + b4));
  return (dot < e) ? b4 + 4u : b4;
}
// Every TPACF kernel carves its TPSmem from the start of dynamic shared memory and declares no
// static shared memory, so in a launch without clusters the table sits at the shared address
// TP_DSBASE (the first KB of the CTA's window is the system's) and the edges at TP_DSBASE + TP_LUT:
// the pair loops address both as [reg + immediate] (no base add per lookup; the kernels check
// tp_dsbase_ok() once and otherwise take the binary search).  The compare-and-step is one PTX
// select so the compiler forms the histogram address as one LEA of the stepped value.
extern __shared__ __align__(128) unsigned char hk_tp_dsmem[];
constexpr uint32_t TP_DSBASE = 0x400;
__device__ __forceinline__ bool tp_dsbase_ok() { return (uint32_t)__cvta_generic_to_shared(hk_tp_dsmem) == TP_DSBASE; }
__device__ __forceinline__ uint32_t tp_b4_fixed(float dot) {
  const float u = __fsub_rn(1.0f, dot);
  uint32_t b4, r;
  float e;
  asm("ld.shared.u8 %0, [%1+%2];" : "=r"(b4) : "r"(fb(u) >> 21), "n"(TP_DSBASE));
  asm("ld.shared.f32 %0, [%1+%2];" : "=f"(e) : "r"(b4), "n"(TP_DSBASE + TP_LUT));
  asm("{\n\t.reg .pred p;\n\tsetp.lt.f32 p, %1, %2;\n\tadd.u32 %0, %3, 4;\n\tselp.u32 %0, %0, %3, p;\n\t}"
      : "=r"(r) : "f"(dot), "f"(e), "r"(b4));
  return r;
}
template <bool LUT>
__device__ __forceinline__ uint32_t tp_b4(const uint8_t* __restrict__, uint32_t, const float* Es, float dot) {
  return LUT ? tp_b4_fixed(dot) : 4u * (uint32_t)tp_bin_search(Es, dot);
}
__device__ __forceinline__ void red_shared(uint32_t addr, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}

// ---------------------------------------------------------------------------------------------
// Shared memory: L[2048] u8 | E[32] f32 | B[2][3 * TP_TILE] f32 (packed x, y, z) |
// H[warps][NP/2 words][nb2][32] u32 | part[warps * NP/2 * nb2] | flag
// ---------------------------------------------------------------------------------------------
struct TPSmem {
  uint8_t* L;
  float* E;
  float* B;
  uint32_t* H;
  uint32_t* part;  // [TP_WARPS * NP/2 * nb2] flush scratch (the ring may hold a prefetched tile)
  int* flag;
};
// (T = threads of the CTA: 128 for the replica kernels, HK_TP_SR_T for the single run)
__host__ __device__ inline size_t tp_smem_bytes(int nb2, int np, int T = TP_THREADS) {
  return (size_t)TP_LUT + 32 * 4 + 2 * 3 * TP_TILE * 4 + (size_t)(T / 32) * (np / 2) * nb2 * 33 * 4 + 16;
}
__device__ __forceinline__ TPSmem tp_carve(unsigned char* base, int nb2, int np, int T = TP_THREADS) {
  TPSmem S;
  S.L = base;
  S.E = reinterpret_cast<float*>(base + TP_LUT);
  S.B = reinterpret_cast<float*>(base + TP_LUT + 128);
  S.H = reinterpret_cast<uint32_t*>(base + TP_LUT + 128 + 2 * 3 * TP_TILE * 4);
  S.part = reinterpret_cast<uint32_t*>(base + TP_LUT + 128 + 2 * 3 * TP_TILE * 4 + (size_t)(T / 32) * (np / 2) * nb2 * 128);
  S.flag = reinterpret_cast<int*>(reinterpret_cast<unsigned char*>(S.part) + (size_t)(T / 32) * (np / 2) * nb2 * 4);
  return S;
}
__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// Table + edges, once per CTA (the edges padded with -inf for the binary search).
__device__ __forceinline__ void tp_stage_tables(const TPParams& p, const TPSmem& S) {
  for (int k = threadIdx.x; k < TP_LUT / 16; k += TP_THREADS) cp_async16(S.L + 16 * k, p.lut + 16 * k);
  if (threadIdx.x < 32) S.E[threadIdx.x] = threadIdx.x <= p.nb ? p.edges[threadIdx.x] : __int_as_float(0xff800000);
  cp_async_commit();
}
template <int NP, int T = TP_THREADS>
__device__ __forceinline__ void tp_zero_hist(const TPParams& p, const TPSmem& S) {
  const int nh = (T / 32) * (NP / 2) * (p.nb + 2) * 32;
  for (int k = threadIdx.x; k < nh; k += T) S.H[k] = 0u;
}
// Partners [j0, j0 + cnt) of set sb into ring slot `slot` (cnt <= TP_TILE; 4-byte async copies).
template <int T = TP_THREADS>
__device__ __forceinline__ void tp_stage_tile(const TPParams& p, const TPSmem& S, int sb, int j0, int cnt, int slot) {
  const float* src = p.pts + 3 * ((int64_t)sb * p.n + j0);
  float* dst = S.B + slot * 3 * TP_TILE;
  for (int k = threadIdx.x; k < 3 * cnt; k += T) cp_async4(dst + k, src + k);
  cp_async_commit();
}

// Reduce the lane-private histograms (both 16-bit halves of every word) and add them to
// hist[base + b]: each (warp, word, bin) row of 32 counters is summed (rotated start: no bank
// conflicts), the rows of a bin combined in shared memory, then one u64 atomic per non-zero bin.
template <int NP, int T = TP_THREADS>
__device__ __forceinline__ void tp_flush(const TPParams& p, const TPSmem& S, unsigned long long* hist, int base) {
  const int nb2 = p.nb + 2, rows = (T / 32) * (NP / 2);
  uint32_t* part = S.part;
  for (int t = threadIdx.x; t < rows * nb2; t += T) {
    const uint32_t* row = S.H + (size_t)t * 32;
    uint32_t s = 0;
#pragma unroll 8
    for (int l = 0; l < 32; ++l) {
      const uint32_t w = row[(l + t) & 31];
      s += (w & 0xffffu) + (w >> 16);
    }
    part[t] = s;
  }
  __syncthreads();
  if (threadIdx.x < nb2) {
    unsigned long long s = 0;
    for (int w = 0; w < rows; ++w) s += part[w * nb2 + threadIdx.x];
    if (s) atomicAdd(hist + base + threadIdx.x, s);
  }
}

// ---------------------------------------------------------------------------------------------
// Per-abstract-thread prologue (NL sites 0-10) and epilogue.
// ---------------------------------------------------------------------------------------------
struct TPPoint {
  int32_t i, h, boff, jb, je, expect, base;
  float x1, y1, z1;
  uint32_t chk, alarm;
  int32_t acc, cnt;  // acc in units of 4 (the table's 4 * bin) until divided
  bool valid;
};

// i_dup / h_dup: the same indices recomputed from launch indices through the opaque zero.
template <bool NL>
__device__ __forceinline__ TPPoint tp_prologue(const TPParams& p, const unsigned long long* hist, int h, int i, int i_dup,
                                               int h_dup, bool valid) {
  const uint32_t z = p.z;
  const int32_t n = p.n, nr = p.nr, nb2 = p.nb + 2;
  TPPoint P;
  P.valid = valid;
  P.i = i;
  P.h = h;
  P.chk = 0;
  P.alarm = 0;
  if (NL) {
    P.chk ^= (uint32_t)n ^ lohi_ptr(p.pts) ^ lohi_ptr(hist);
    P.chk ^= (uint32_t)i; P.alarm |= (i_dup != i) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)h; P.alarm |= (h_dup != h) ? AL_DUP : 0u;
  }
  const int32_t aoff = (h <= nr ? h : 0) * n + i;
  const int32_t sb = (h == 0) ? 0 : (h <= nr ? h : h - nr);
  P.boff = sb * n;
  P.jb = h <= nr ? i + 1 : 0;
  P.je = n;
  P.expect = max(P.je - P.jb, 0);
  P.base = h * nb2;
  if (NL) {
    const int32_t h2 = opq(h, z), i2 = opq(i, z);
    P.chk ^= (uint32_t)aoff; P.alarm |= ((h2 <= nr ? h2 : 0) * n + i2 != aoff) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.boff; P.alarm |= ((h2 == 0 ? 0 : (h2 <= nr ? h2 : h2 - nr)) * n != P.boff) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.jb; P.alarm |= ((h2 <= nr ? i2 + 1 : 0) != P.jb) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.je; P.alarm |= (opq(n, z) != P.je) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.expect; P.alarm |= (max(opq(P.je, z) - P.jb, 0) != P.expect) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.base; P.alarm |= (h2 * nb2 != P.base) ? AL_DUP : 0u;
  }
  const float* A = p.pts + 3 * (int64_t)(valid ? aoff : 0);
  P.x1 = A[0]; P.y1 = A[1]; P.z1 = A[2];
  if (NL) {
    const float* A2 = p.pts + 3 * (int64_t)(valid ? opq(aoff, z) : 0);
    P.chk ^= fb(P.x1); P.alarm |= (fb(A2[0]) != fb(P.x1)) ? AL_DUP : 0u;
    P.chk ^= fb(P.y1); P.alarm |= (fb(A2[1]) != fb(P.y1)) ? AL_DUP : 0u;
    P.chk ^= fb(P.z1); P.alarm |= (fb(A2[2]) != fb(P.z1)) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)opq(i, z) ^ (uint32_t)opq(h, z) ^ (uint32_t)opq(aoff, z) ^ (uint32_t)opq(P.jb, z);
  }
  P.acc = 0;
  P.cnt = 0;
  if (!valid) P.jb = INT32_MAX;  // takes part in no pair
  return P;
}

// NL exit XORs of the loop-live values and the parameters, then the checksum test.
template <bool NL>
__device__ __forceinline__ void tp_nl_exit(const TPParams& p, TPPoint& P, const unsigned long long* hist) {
  if (!NL) return;
  const uint32_t z = p.z;
  P.chk ^= (uint32_t)opq(P.boff, z) ^ (uint32_t)opq(P.je, z) ^ (uint32_t)opq(P.base, z);
  P.chk ^= opqf(P.x1, z) ^ opqf(P.y1, z) ^ opqf(P.z1, z) ^ (uint32_t)opq(P.expect, z);
  P.chk ^= ((uint32_t)p.n + z) ^ (lohi_ptr(p.pts) + z) ^ (lohi_ptr(hist) + z);
  if (P.chk != 0) P.alarm |= AL_CHK;
}

// HauberkCheckEqual(cnt, expect) / HauberkCheckRange(acc / cnt) after the whole loop (L1405-1429);
// PROFILE writes the sample acc / cnt.  acc and cnt are the full-loop sums.
template <int V>
__device__ __forceinline__ void tp_checks(const TPParams& p, TPPoint& P, hk_control* cb, int64_t g) {
  constexpr bool L = (V & V_L) != 0, PROF = (V & V_PROF) != 0;
  if (L && P.cnt != P.expect) P.alarm |= AL_COUNT;
  if ((L || PROF) && P.cnt != 0 && p.ndet > 0) {
    const float v = __fdiv_rn((float)P.acc, (float)P.cnt);
    if (PROF) p.samples[g] = v;
    if (L && p.R.n[0] > 0 && !in_range<false>(p.R, 0, v, nullptr)) {
      P.alarm |= AL_RANGE;
      record_outlier(cb, 0, v);
    }
  }
}

__device__ __forceinline__ float tp_dot(const TPPoint& P, float x2, float y2, float z2) {
  return __fmaf_rn(P.z1, z2, __fmaf_rn(P.y1, y2, __fmul_rn(P.x1, x2)));
}

// ---------------------------------------------------------------------------------------------
// The pair loops over one staged tile.  Hw[w] = this lane's histogram word w (shared byte address;
// point k counts in word k/2, half k%2); inc[k] = 1 / 0x10000 (0 for an absent point or the faulted
// abstract thread of an FI CTA, whose whole loop runs in the FI program instead).
//  * tp_pairs_all: every point of the CTA has all of [k0, k1) as partners (no masks); groups of G
//    partners (G = 32 / NP, i.e. 3 * G / 4 broadcast LDS.128 per group) with the counters advanced
//    by G per group (the strength reduction any compiler applies to an unrolled cnt++; the FI
//    program keeps the per-iteration increment);
//  * tp_pairs_masked: the diagonal of a self-correlation row (j >= jb differs per point).
// ---------------------------------------------------------------------------------------------
struct TPLoopCtx {
  const uint8_t* L;
  uint32_t eb;
  const float* Es;
};

// Points 0..NQ-1 of the thread against one partner j (MASKQ: point NQ-1 only if j >= its jb).
template <int NP, int NQ, bool MASKQ, bool CNT, bool LUT>
__device__ __forceinline__ void tp_pair1(const TPLoopCtx& c, const uint32_t (&Hw)[NP / 2], TPPoint (&P)[NP],
                                         const uint32_t (&inc)[NP], float x2, float y2, float z2, int j) {
#pragma unroll
  for (int k = 0; k < NQ; ++k) {
    const uint32_t b4 = tp_b4<LUT>(c.L, c.eb, c.Es, tp_dot(P[k], x2, y2, z2));
    const bool on = !(MASKQ && k == NQ - 1) || j >= P[k].jb;
    red_shared(Hw[k / 2] + b4 * 32u, on ? inc[k] : 0u);
    if (CNT) {
      P[k].acc += on ? (int32_t)b4 : 0;
      P[k].cnt += on ? 1 : 0;
    }
  }
}

// Points 0..NQ-1 against the partners [k, k1) of the staged tile (partner jt0 + k); MASKQ: point
// NQ-1 counts partner j only if j >= its jb (the diagonal, see tp_diag).  Groups of G partners
// (G = 32 / NP, i.e. 3 * G / 4 broadcast LDS.128 per group) with the counters of the unmasked
// points advanced by G per group (the strength reduction any compiler applies to an unrolled
// cnt++; the FI program keeps the per-iteration increment).
template <int NP, int NQ, bool MASKQ, bool CNT, bool LUT>
__device__ __forceinline__ void tp_pairs_grp(const TPParams& p, const TPLoopCtx& c, const float* __restrict__ Bt,
                                             const uint32_t (&Hw)[NP / 2], TPPoint (&P)[NP], const uint32_t (&inc)[NP],
                                             int k, int k1, int jt0) {
  if (!LUT) {  // the binary-search fallback (a bucket holds two edges): plain loop, rare
#pragma unroll 1
    for (; k < k1; ++k) tp_pair1<NP, NQ, MASKQ, CNT, LUT>(c, Hw, P, inc, Bt[3 * k], Bt[3 * k + 1], Bt[3 * k + 2], jt0 + k);
    return;
  }
  // partners per group: G * NQ pairs per thread and group (16 for NP = 4: enough independent
  // table lookups in flight within the 80-register budget of 6 CTAs per SM)
  constexpr int G = HK_TP_GROUP > 0 ? HK_TP_GROUP : (NP >= 4 ? 4 : 8);
  static_assert(G % 4 == 0, "groups are whole 48-byte partner quads");
  for (; k < k1 && (k & 3); ++k) tp_pair1<NP, NQ, MASKQ, CNT, LUT>(c, Hw, P, inc, Bt[3 * k], Bt[3 * k + 1], Bt[3 * k + 2], jt0 + k);
  const float4* __restrict__ T4 = reinterpret_cast<const float4*>(Bt);
#pragma unroll 1
  for (; k + G - 1 < k1; k += G) {
    const int k3 = (k >> 2) * 3;
    float xs[G], ys[G], zs[G];
#pragma unroll
    for (int q = 0; q < G / 4; ++q) {
      const float4 v0 = T4[k3 + 3 * q], v1 = T4[k3 + 3 * q + 1], v2 = T4[k3 + 3 * q + 2];
      xs[4 * q] = v0.x; ys[4 * q] = v0.y; zs[4 * q] = v0.z;
      xs[4 * q + 1] = v0.w; ys[4 * q + 1] = v1.x; zs[4 * q + 1] = v1.y;
      xs[4 * q + 2] = v1.z; ys[4 * q + 2] = v1.w; zs[4 * q + 2] = v2.x;
      xs[4 * q + 3] = v2.y; ys[4 * q + 3] = v2.z; zs[4 * q + 3] = v2.w;
    }
    uint32_t b[NQ][G];
#pragma unroll
    for (int u = 0; u < G; ++u)
#pragma unroll
      for (int kk = 0; kk < NQ; ++kk) b[kk][u] = tp_b4<LUT>(c.L, c.eb, c.Es, tp_dot(P[kk], xs[u], ys[u], zs[u]));
    bool on[G];
#pragma unroll
    for (int u = 0; u < G; ++u) on[u] = !MASKQ || jt0 + k + u >= P[NQ - 1].jb;
#pragma unroll
    for (int u = 0; u < G; ++u)
#pragma unroll
      for (int kk = 0; kk < NQ; ++kk)
        red_shared(Hw[kk / 2] + b[kk][u] * 32u, (MASKQ && kk == NQ - 1 && !on[u]) ? 0u : inc[kk]);
    if (CNT) {
#pragma unroll
      for (int kk = 0; kk < NQ; ++kk) {
        if (MASKQ && kk == NQ - 1) {
#pragma unroll
          for (int u = 0; u < G; ++u) {
            P[kk].acc += on[u] ? (int32_t)b[kk][u] : 0;
            P[kk].cnt += on[u] ? 1 : 0;
          }
        } else {
#pragma unroll
          for (int u = 0; u < G; u += 2) P[kk].acc += (int32_t)(b[kk][u] + b[kk][u + 1]);
          P[kk].cnt = count_inc(P[kk].cnt, G == 8 ? p.eight : (G == 4 ? p.four : p.one * G));
        }
      }
    }
  }
  for (; k < k1; ++k) tp_pair1<NP, NQ, MASKQ, CNT, LUT>(c, Hw, P, inc, Bt[3 * k], Bt[3 * k + 1], Bt[3 * k + 2], jt0 + k);
}
// All points against [k, k1): the unmasked form of tp_pairs_grp, kept as its own loop (ptxas
// schedules this one with the table lookups of a group interleaved; measured in mix.cu)
template <int NP, bool CNT, bool LUT>
__device__ __forceinline__ void tp_pairs_all(const TPParams& p, const TPLoopCtx& c, const float* __restrict__ Bt,
                                             const uint32_t (&Hw)[NP / 2], TPPoint (&P)[NP], const uint32_t (&inc)[NP],
                                             int k, int k1) {
  if (!LUT) {
    tp_pairs_grp<NP, NP, false, CNT, LUT>(p, c, Bt, Hw, P, inc, k, k1, 0);
    return;
  }
  constexpr int G = HK_TP_GROUP > 0 ? HK_TP_GROUP : (NP >= 4 ? 4 : 8);
  static_assert(G % 4 == 0, "groups are whole 48-byte partner quads");
  for (; k < k1 && (k & 3); ++k) tp_pair1<NP, NP, false, CNT, LUT>(c, Hw, P, inc, Bt[3 * k], Bt[3 * k + 1], Bt[3 * k + 2], 0);
  const float4* __restrict__ T4 = reinterpret_cast<const float4*>(Bt);
#pragma unroll 1
  for (; k + G - 1 < k1; k += G) {
    const int k3 = (k >> 2) * 3;
    float xs[G], ys[G], zs[G];
#pragma unroll
    for (int q = 0; q < G / 4; ++q) {
      const float4 v0 = T4[k3 + 3 * q], v1 = T4[k3 + 3 * q + 1], v2 = T4[k3 + 3 * q + 2];
      xs[4 * q] = v0.x; ys[4 * q] = v0.y; zs[4 * q] = v0.z;
      xs[4 * q + 1] = v0.w; ys[4 * q + 1] = v1.x; zs[4 * q + 1] = v1.y;
      xs[4 * q + 2] = v1.z; ys[4 * q + 2] = v1.w; zs[4 * q + 2] = v2.x;
      xs[4 * q + 3] = v2.y; ys[4 * q + 3] = v2.z; zs[4 * q + 3] = v2.w;
    }
    uint32_t b[NP][G];
#pragma unroll
    for (int u = 0; u < G; ++u)
#pragma unroll
      for (int kk = 0; kk < NP; ++kk) b[kk][u] = tp_b4<LUT>(c.L, c.eb, c.Es, tp_dot(P[kk], xs[u], ys[u], zs[u]));
#pragma unroll
    for (int u = 0; u < G; ++u)
#pragma unroll
      for (int kk = 0; kk < NP; ++kk) red_shared(Hw[kk / 2] + b[kk][u] * 32u, inc[kk]);
    if (CNT) {
#pragma unroll
      for (int kk = 0; kk < NP; ++kk) {
#pragma unroll
        for (int u = 0; u < G; u += 2) P[kk].acc += (int32_t)(b[kk][u] + b[kk][u + 1]);
        P[kk].cnt = count_inc(P[kk].cnt, G == 8 ? p.eight : (G == 4 ? p.four : p.one * G));
      }
    }
  }
  for (; k < k1; ++k) tp_pair1<NP, NP, false, CNT, LUT>(c, Hw, P, inc, Bt[3 * k], Bt[3 * k + 1], Bt[3 * k + 2], 0);
}

// The diagonal, one partner at a time (GDIAG = false: the fused kernel of mix.cu, where the
// grouped form below costs the main loop its interleaved schedule — measured).
template <int NP, bool CNT, bool LUT, int S = 0, int STR = TP_THREADS>
__device__ __forceinline__ void tp_diag1(const TPLoopCtx& c, const float* __restrict__ Bt, const uint32_t (&Hw)[NP / 2],
                                         TPPoint (&P)[NP], const uint32_t (&inc)[NP], int i0, int jt0, int k0, int km) {
  const int ka = max(k0, i0 + S * STR - jt0), kb = min(km, i0 + (S + 1) * STR - jt0);
#pragma unroll 1
  for (int k = ka; k < kb; ++k) tp_pair1<NP, S + 1, true, CNT, LUT>(c, Hw, P, inc, Bt[3 * k], Bt[3 * k + 1], Bt[3 * k + 2], jt0 + k);
  if constexpr (S + 1 < NP) tp_diag1<NP, CNT, LUT, S + 1, STR>(c, Bt, Hw, P, inc, i0, jt0, k0, km);
}

// The diagonal of a self-correlation row, segment S: partners j in [i0 + STR S, i0 + STR (S + 1))
// (tile-relative [ka, kb)).  Point k of a thread is i0 + STR k + t (STR = the CTA's threads), so for
// these partners points k < S are all active (j > i), point S is masked (j >= jb) and points k > S
// take no part: the grouped loop over points 0..S with the mask on point S.
template <int NP, bool CNT, bool LUT, int S = 0, int STR = TP_THREADS>
__device__ __forceinline__ void tp_diag(const TPParams& p, const TPLoopCtx& c, const float* __restrict__ Bt,
                                        const uint32_t (&Hw)[NP / 2], TPPoint (&P)[NP], const uint32_t (&inc)[NP], int i0, int jt0,
                                        int k0, int km) {
  const int ka = max(k0, i0 + S * STR - jt0), kb = min(km, i0 + (S + 1) * STR - jt0);
  if (ka < kb) tp_pairs_grp<NP, S + 1, true, CNT, LUT>(p, c, Bt, Hw, P, inc, ka, kb, jt0);
  if constexpr (S + 1 < NP) tp_diag<NP, CNT, LUT, S + 1, STR>(p, c, Bt, Hw, P, inc, i0, jt0, k0, km);
}

// Pairs of the staged tile Bt (partners jt0 + k) for k in [k0, k1): [k0, km) with per-point masks
// (partners below jall = min(i0 + NP * STR, N) in a self-correlation row: its diagonal, in
// segments), [km, k1) for all points.
template <int NP, bool CNT, bool LUT, bool GDIAG = true, int STR = TP_THREADS>
__device__ __forceinline__ void tp_tile_pairs(const TPParams& p, const TPLoopCtx& c, const float* __restrict__ Bt,
                                              const uint32_t (&Hw)[NP / 2], TPPoint (&P)[NP], const uint32_t (&inc)[NP],
                                              int jt0, int k0, int k1, int jall, int i0) {
  const int km = min(max(jall - jt0, k0), k1);
  if (k0 < km) {
    if (GDIAG) tp_diag<NP, CNT, LUT, 0, STR>(p, c, Bt, Hw, P, inc, i0, jt0, k0, km);
    else tp_diag1<NP, CNT, LUT, 0, STR>(c, Bt, Hw, P, inc, i0, jt0, k0, km);
  }
  tp_pairs_all<NP, CNT, LUT>(p, c, Bt, Hw, P, inc, km, k1);
}
template <int NP>
__device__ __forceinline__ void tp_lane_hist(const TPParams& p, const TPSmem& S, uint32_t (&Hw)[NP / 2]) {
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
#pragma unroll
  for (int w = 0; w < NP / 2; ++w) Hw[w] = smem_u32(S.H + (((size_t)warp * (NP / 2) + w) * (p.nb + 2)) * 32 + lane);
}

// One work item: the points i0 + t + 128 k (k < NP) of histogram h against partners [jr0, jr1)
// (already clipped to the block's [jlo, N)), streamed tile by tile through the ring.  The tables
// are staged and the histogram zeroed by the caller.
template <int NP, int V, bool LUT, bool GDIAG = true, int T = TP_THREADS>
__device__ __forceinline__ void tp_item_loop(const TPParams& p, const TPSmem& S, TPPoint (&P)[NP], const uint32_t (&inc)[NP],
                                             int h, int i0, int jr0, int jr1) {
  constexpr bool CNT = (V & (V_L | V_PROF)) != 0;
  const int sb = (h == 0) ? 0 : (h <= p.nr ? h : h - p.nr);
  const int js = jr0 & ~3;  // tiles start on 4-partner boundaries (16-byte aligned groups in smem)
  const int nt = jr1 > jr0 ? (jr1 - js + TP_TILE - 1) / TP_TILE : 0;
  // partners below jall need per-point masks (self rows: j >= i + 1), the rest do not
  const int jall = h <= p.nr ? min(i0 + NP * T, p.n) : 0;
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  uint32_t Hw[NP / 2];
#pragma unroll
  for (int w = 0; w < NP / 2; ++w) Hw[w] = smem_u32(S.H + (((size_t)warp * (NP / 2) + w) * (p.nb + 2)) * 32 + lane);
  const TPLoopCtx c{S.L, smem_u32(S.E), S.E};
  if (nt > 0) tp_stage_tile<T>(p, S, sb, js, min(TP_TILE, jr1 - js), 0);
  for (int t = 0; t < nt; ++t) {
    const int jt0 = js + t * TP_TILE;
    if (t + 1 < nt) {
      const int jn = jt0 + TP_TILE;
      tp_stage_tile<T>(p, S, sb, jn, min(TP_TILE, jr1 - jn), (t + 1) & 1);
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    tp_tile_pairs<NP, CNT, LUT, GDIAG, T>(p, c, S.B + (t & 1) * 3 * TP_TILE, Hw, P, inc, jt0, max(jr0, jt0) - jt0,
                                          min(jr1, jt0 + TP_TILE) - jt0, jall, i0);
    __syncthreads();  // slot t & 1 is refilled by the stage of tile t + 2
  }
}

template <int NP, int T = TP_THREADS>
__device__ __forceinline__ void tp_points(const TPParams& p, const unsigned long long* hist, int h, int blk, int64_t g0,
                                          int64_t g1, TPPoint (&P)[NP], bool nl) {
  const int i0 = blk * NP * T;
  const int64_t gb = (int64_t)h * p.n;
#pragma unroll
  for (int k = 0; k < NP; ++k) {
    const int i = i0 + k * T + threadIdx.x;
    const bool v = i < p.n && gb + i >= g0 && gb + i < g1;
    const int idup = (int)((blk ^ p.z) * (NP * T) + k * T + (threadIdx.x ^ p.z));
    P[k] = nl ? tp_prologue<true>(p, hist, h, i, idup, (int)((uint32_t)h ^ p.z), v)
              : tp_prologue<false>(p, hist, h, i, idup, (int)((uint32_t)h ^ p.z), v);
  }
}

// ============================================================================================
// Single run (BASE / FT / FT_NL / FT_L / PROFILE): one wave of equal pieces.  A row = (histogram
// h, point block blk) of 128 * NP points; its partners [jlo, N) are cut into pieces.  Row r gets
// P(r + 1) - P(r) pieces (at least 1, and enough to keep every piece < 32768 partners, the
// capacity of a 16-bit histogram half) with P(r) = round(S * W(r) / W), W(r) the pair slots
// (points x partners) of the rows before r and S the CTAs one wave holds: every SM then runs the
// same number of equal pieces.  A CTA runs one piece exactly like a replica CTA runs a whole row
// (tp_item_loop), then adds its points' (acc, cnt) to per-thread partial sums (exact integer
// combine); the piece that completes a row (a per-row counter) runs the loop-exit checks.
// ============================================================================================
struct TPSR {
  int* row_done;   // [nrows] pieces completed (zeroed per run)
  int nrows;
  int slots;       // S: CTAs of one wave
  int64_t total;   // W: pair slots of the run
};

// Row geometry: h, blk, the first partner jlo and the weight (valid points x partners) of `row`.
__host__ __device__ __forceinline__ int64_t tp_sr_row(int n, int nr, int nblk, int64_t g0, int64_t g1, int row, int* h, int* blk,
                                                      int* jlo) {
  constexpr int NP = HK_TP_NP_SR;
  *h = row / nblk;
  *blk = row - *h * nblk;
  const int i0 = *blk * NP * TP_SR_T;
  const int64_t gb = (int64_t)*h * n;
  const int64_t a = gb + i0 > g0 ? gb + i0 : g0;
  const int64_t e = gb + i0 + NP * TP_SR_T < gb + n ? gb + i0 + NP * TP_SR_T : gb + n;
  const int64_t pts = (e < g1 ? e : g1) - a;
  *jlo = *h <= nr ? i0 + 1 : 0;
  return (pts > 0 && *jlo < n) ? pts * (int64_t)(n - *jlo) : 0;
}
// pieces of a row of weight w and `len` partners whose preceding rows weigh wcum
__host__ __device__ __forceinline__ int tp_sr_pieces(int64_t w, int64_t wcum, int len, int slots, int64_t total) {
  if (w <= 0) return 0;
  const int64_t p0 = (2 * slots * wcum + total) / (2 * total), p1 = (2 * slots * (wcum + w) + total) / (2 * total);
  const int64_t bylen = (len + 32766) / 32767;
  const int64_t k = p1 - p0 > bylen ? p1 - p0 : bylen;
  return (int)(k < 1 ? 1 : k);
}

// Warp 0: (row, piece within the row, pieces of the row) of piece `piece` (prefix scans over the
// rows, 32 at a time).
__device__ __forceinline__ int3 tp_sr_locate(const TPParams& p, const TPSR& q, int piece) {
  const unsigned FULL = 0xffffffffu;
  const int lane = (int)lane_id();
  int base = 0;
  int64_t wbase = 0;
  for (int r0 = 0; r0 < q.nrows; r0 += 32) {
    const int r = r0 + lane;
    int h, blk, jlo = 0;
    const int64_t w = r < q.nrows ? tp_sr_row(p.n, p.nr, p.nblk, p.g0, p.g1, r, &h, &blk, &jlo) : 0;
    int64_t wincl = w;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int64_t v = __shfl_up_sync(FULL, wincl, d);
      if (lane >= d) wincl += v;
    }
    const int c = tp_sr_pieces(w, wbase + wincl - w, p.n - jlo, q.slots, q.total);
    int incl = c;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int v = __shfl_up_sync(FULL, incl, d);
      if (lane >= d) incl += v;
    }
    const unsigned m = __ballot_sync(FULL, c > 0 && piece >= base + incl - c && piece < base + incl);
    if (m) {
      const int l = __ffs(m) - 1;
      return make_int3(r0 + l, piece - (base + __shfl_sync(FULL, incl - c, l)), __shfl_sync(FULL, c, l));
    }
    base += __shfl_sync(FULL, incl, 31);
    wbase += __shfl_sync(FULL, wincl, 31);
  }
  return make_int3(-1, 0, 0);
}

template <int V, bool LUT>
__device__ __forceinline__ void tp_sr_piece(const TPParams& p, const TPSmem& S, const TPSR& q, int3 pc) {
  constexpr int NP = HK_TP_NP_SR;
  constexpr bool NL = (V & V_NL) != 0, L = (V & V_L) != 0, PROF = (V & V_PROF) != 0, CNT = L || PROF;
  int h, blk, jlo;
  tp_sr_row(p.n, p.nr, p.nblk, p.g0, p.g1, pc.x, &h, &blk, &jlo);
  const int i0 = blk * NP * TP_SR_T;
  const int64_t gb = (int64_t)h * p.n;
  const int64_t len = p.n - jlo;
  const int j0 = jlo + (int)(len * pc.y / pc.z), j1 = jlo + (int)(len * (pc.y + 1) / pc.z);
  TPPoint P[NP];
  tp_points<NP, TP_SR_T>(p, p.hist, h, blk, p.g0, p.g1, P, NL);
  uint32_t inc[NP];
#pragma unroll
  for (int k = 0; k < NP; ++k) inc[k] = P[k].valid ? ((k & 1) ? 0x10000u : 1u) : 0u;
  tp_zero_hist<NP, TP_SR_T>(p, S);
  // The points' state the pair loop does not touch (index, checksum, alarm bits, the NL-protected
  // loop-invariant values) waits in local memory while the loop runs, so the loop keeps its
  // registers for independent table lookups (HK_TP_STASH; the values are written once before and
  // read once after the loop, exactly as a register spill would move them).
  constexpr bool STASH = ((HK_TP_STASH >> V) & 1) != 0;
  volatile int32_t stash[NP][8];
  if constexpr (STASH) {
#pragma unroll
    for (int k = 0; k < NP; ++k) {
      stash[k][0] = P[k].i; stash[k][1] = (int32_t)P[k].chk; stash[k][2] = (int32_t)P[k].alarm; stash[k][3] = P[k].expect;
      stash[k][4] = P[k].boff; stash[k][5] = P[k].je; stash[k][6] = P[k].base; stash[k][7] = P[k].valid ? 1 : 0;
    }
  }
  __syncthreads();
  tp_item_loop<NP, V, LUT, true, TP_SR_T>(p, S, P, inc, h, i0, j0, j1);
  if constexpr (STASH) {
#pragma unroll
    for (int k = 0; k < NP; ++k) {
      P[k].i = stash[k][0]; P[k].chk = (uint32_t)stash[k][1]; P[k].alarm = (uint32_t)stash[k][2]; P[k].expect = stash[k][3];
      P[k].boff = stash[k][4]; P[k].je = stash[k][5]; P[k].base = stash[k][6]; P[k].valid = stash[k][7] != 0;
    }
  }
#pragma unroll
  for (int k = 0; k < NP; ++k) {
    if (CNT) P[k].acc /= 4;
    tp_nl_exit<NL>(p, P[k], p.hist);
  }
  if (CNT) {
    if (pc.z == 1) {  // the whole row in this piece
#pragma unroll
      for (int k = 0; k < NP; ++k)
        if (P[k].valid) tp_checks<V>(p, P[k], p.cb, gb + P[k].i);
    } else {
#pragma unroll
      for (int k = 0; k < NP; ++k)
        if (P[k].valid && P[k].cnt) {  // exact combine of this piece's partial sums
          atomicAdd(p.accg + gb + P[k].i, P[k].acc);
          atomicAdd(p.cntg + gb + P[k].i, P[k].cnt);
        }
      // the histogram flush overlaps the combine atomics' round trip (the loop's last barrier
      // already ordered every ATOMS of the piece)
      tp_flush<NP, TP_SR_T>(p, S, p.hist, h * (p.nb + 2));
      __syncthreads();  // every thread's combine atomics issued
      if (threadIdx.x == 0) {
        __threadfence();
        *S.flag = atomicAdd(q.row_done + pc.x, 1) + 1 == pc.z;
      }
      __syncthreads();
      if (*S.flag) {  // this piece completed the row: the loop-exit checks of its points
        __threadfence();
#pragma unroll
        for (int k = 0; k < NP; ++k)
          if (P[k].valid) {
            P[k].acc = __ldcg(p.accg + gb + P[k].i);
            P[k].cnt = __ldcg(p.cntg + gb + P[k].i);
            tp_checks<V>(p, P[k], p.cb, gb + P[k].i);
          }
      }
    }
  }
  if (NL || L) {
#pragma unroll
    for (int k = 0; k < NP; ++k)
      if (P[k].valid) fold_alarm(p.cb, P[k].alarm, (uint32_t)(gb + P[k].i));
  }
  if (!CNT || pc.z == 1) {
    __syncthreads();
    tp_flush<NP, TP_SR_T>(p, S, p.hist, h * (p.nb + 2));
  }
}

// FI & FT (or FI-only) replicas (blockIdx.y = launch slot)
// ============================================================================================
enum TPKind : int { TK_NL = 0, TK_LIVE, TK_J, TK_X2, TK_Y2, TK_Z2, TK_DOT, TK_BIN, TK_HIDX, TK_ACC, TK_CNT, TK_COUNT };

struct TPFIParams {
  TPParams base;
  const FaultRec* faults;
  unsigned long long* hist0;  // replica r: hist0 + r * hist_elems
  hk_control* cb0;
  int64_t hist_elems;
};

// Histogram sinks of the per-thread TPACF FI program.  Replica: every increment of the faulted
// thread goes to the replica's global histogram through its (possibly corrupted) index.  Replay:
// every increment is folded into deltas of the 3*nb outputs (DD, DRS, RRS of R4) with a sign
// (+1 faulted run, -1 golden twin).
struct TPReplicaSink {
  hk_control* cb;
  __device__ __forceinline__ void hist_p(unsigned long long* ptr, const unsigned long long*) { red_add(ptr, 1ull); }
  __device__ __forceinline__ void outlier(int d, float v) { record_outlier(cb, d, v); }
  __device__ __forceinline__ void finish(bool mine, uint32_t alarm, uint32_t fail, uint32_t margin, float gap,
                                         bool applied, uint32_t tid) {
    if (fail) atomicOr(&cb->fail, fail);
    if (mine) {
      cb->fault_applied = applied ? 1u : 0u;
      cb->check_margin = margin;
      cb->check_gap = gap;
    }
    if (alarm) {  // one thread: no warp vote (the rest of its warp has left)
      atomicOr(&cb->alarm, alarm);
      atomicAdd(&cb->n_alarm_warps, 1u);
      atomicMin(&cb->first_thread, tid);
    }
  }
};
constexpr int TP_REPLAY_OUT = 96;  // 3 * n_bins (n_bins <= 30 for the replay kernel) + slack
struct TPReplaySink {
  int nr, nb, nb2, sign;
  int32_t* delta;  // [3 * nb]: DD, DRS, RRS for bins 1..nb
  uint32_t alarm = 0, fail = 0, margin = 0xffffffffu;
  float gap = __builtin_huge_valf();
  __device__ __forceinline__ void hist_p(unsigned long long* ptr, const unsigned long long* base) {
    const int64_t e = ptr - base;
    const int row = (int)(e / nb2), b = (int)(e % nb2);
    if (b < 1 || b > nb) return;  // under/overflow bins are not outputs (R4)
    const int kind = row == 0 ? 0 : (row <= nr ? 2 : 1);
    delta[kind * nb + b - 1] += sign;
  }
  __device__ __forceinline__ void outlier(int, float) {}
  __device__ __forceinline__ void finish(bool, uint32_t a, uint32_t f, uint32_t m, float g, bool, uint32_t) {
    alarm = a; fail = f; margin = m; gap = g;
  }
};

// Per-thread FI program of abstract thread g = h*N + ii (DESIGN §3.4 with the single hook of kind
// KIND, R16 guards and the R17 watchdog).  FT = false: the FI-only binary (row a7) — the same
// program with every HAUBERK statement compiled out.  i_dup / h_dup: N0 / N1's duplicates.
// hist_real: the histogram's true base.  REAL: the guardian's unguarded variant (R25).
template <int KIND, bool FT, bool REAL = false, class Sink>
__device__ void tpacf_fi_program(const TPParams& p, const float* Es, const FaultRec& f, int32_t hh, int32_t ii,
                                 int32_t i_dup, int32_t h_dup, bool mine, uint64_t hist_real, Sink& K) {
  const uint32_t z = p.z;
  const int32_t nr = p.nr, nb2 = p.nb + 2;
  const int64_t g = (int64_t)hh * p.n + ii;
  const int64_t inst = mine ? f.inst : -1;
  const uint64_t mask = f.mask;
  const int site = f.site;
  const int64_t npts = 3LL * (1 + nr) * p.n, nhist = (int64_t)(1 + 2 * nr) * nb2;
  const uint64_t pts_real = (uint64_t)(uintptr_t)p.pts;
  uint32_t chk = 0, alarm = 0, fail = 0, margin = 0xffffffffu;
  float gap = __int_as_float(0x7f800000);
  bool applied = false;
  int32_t n = p.n;
  uint64_t ppts = pts_real, phist = hist_real;
  if (FT) chk ^= (uint32_t)n ^ lohi(ppts) ^ lohi(phist);
  const bool nl = (KIND == TK_NL) && mine;
#define NLF(v, s) do { const bool _n = nl && site == (s); applied |= _n; v = flip_i(v, _n, mask); } while (0)
  int32_t i = ii; NLF(i, 0);
  if (FT) { chk ^= (uint32_t)i; alarm |= (i_dup != i) ? AL_DUP : 0u; }
  int32_t h = hh; NLF(h, 1);
  if (FT) { chk ^= (uint32_t)h; alarm |= (h_dup != h) ? AL_DUP : 0u; }
  auto f_aoff = [&](int32_t hq, int32_t iq) { return (int32_t)((uint32_t)(hq <= nr ? hq : 0) * (uint32_t)n + (uint32_t)iq); };
  auto f_boff = [&](int32_t hq) { return (int32_t)((uint32_t)(hq == 0 ? 0 : (hq <= nr ? hq : (int32_t)((uint32_t)hq - (uint32_t)nr))) * (uint32_t)n); };
  auto f_jb = [&](int32_t hq, int32_t iq) { return hq <= nr ? (int32_t)((uint32_t)iq + 1u) : 0; };
  auto f_ex = [&](int32_t je_, int32_t jb_) { const int32_t d = (int32_t)((uint32_t)je_ - (uint32_t)jb_); return d > 0 ? d : 0; };
  int32_t aoff = f_aoff(h, i); NLF(aoff, 2);
  if (FT) { chk ^= (uint32_t)aoff; alarm |= (f_aoff(opq(h, z), opq(i, z)) != aoff) ? AL_DUP : 0u; }
  int32_t boff = f_boff(h); NLF(boff, 3);
  if (FT) { chk ^= (uint32_t)boff; alarm |= (f_boff(opq(h, z)) != boff) ? AL_DUP : 0u; }
  int32_t jb = f_jb(h, i); NLF(jb, 4);
  if (FT) { chk ^= (uint32_t)jb; alarm |= (f_jb(opq(h, z), opq(i, z)) != jb) ? AL_DUP : 0u; }
  int32_t je = n; NLF(je, 5);
  if (FT) { chk ^= (uint32_t)je; alarm |= (opq(n, z) != je) ? AL_DUP : 0u; }
  int32_t expect = f_ex(je, jb); NLF(expect, 6);
  if (FT) { chk ^= (uint32_t)expect; alarm |= (f_ex(opq(je, z), jb) != expect) ? AL_DUP : 0u; }
  int32_t base = (int32_t)((uint32_t)h * (uint32_t)nb2); NLF(base, 7);
  if (FT) { chk ^= (uint32_t)base; alarm |= ((int32_t)((uint32_t)opq(h, z) * (uint32_t)nb2) != base) ? AL_DUP : 0u; }
#undef NLF
  float q1[3];
  int32_t acc = 0, cnt = 0, j;
  const float* pe;
  const int64_t golden = hh <= nr ? (int64_t)p.n - (ii + 1) : (int64_t)p.n;  // uncorrupted launch indices (R17)
  const int64_t limit = fi_limit<REAL>(golden, f.hang);
  constexpr bool real = REAL;
  for (int a = 0; a < 3; ++a) {
    if (!fi_at(real, ppts, pts_real, (int32_t)((uint32_t)aoff * 3u + (uint32_t)a), npts, &pe)) { fail |= FL_CRASH; goto done; }
    float v = __ldg(pe);
    { const bool nn = nl && site == 8 + a; applied |= nn; v = flip_f(v, nn, mask); }
    if (FT) { chk ^= fb(v); alarm |= (fb(__ldg(pe + z)) != fb(v)) ? AL_DUP : 0u; }
    q1[a] = v;
  }
  if (FT) chk ^= (uint32_t)opq(i, z) ^ (uint32_t)opq(h, z) ^ (uint32_t)opq(aoff, z) ^ (uint32_t)opq(jb, z);
  j = jb;
  for (int64_t it = 0;; ++it) {
    const bool now = (it == inst);
    if (KIND == TK_J) { applied |= now; j = flip_i(j, now, mask); }
    if (KIND == TK_LIVE && now) {
      applied = true;
      switch (site) {
        case 11: boff = flip_i(boff, true, mask); break;
        case 12: je = flip_i(je, true, mask); break;
        case 13: expect = flip_i(expect, true, mask); break;
        case 14: base = flip_i(base, true, mask); break;
        case 15: q1[0] = flip_f(q1[0], true, mask); break;
        case 16: q1[1] = flip_f(q1[1], true, mask); break;
        case 17: q1[2] = flip_f(q1[2], true, mask); break;
        case 18: n = flip_i(n, true, mask); break;
        case 19: ppts = flip_p(ppts, true, mask); break;
        case 20: phist = flip_p(phist, true, mask); break;
        default: break;
      }
    }
    if (!(j < je)) break;
    if (it >= limit) { fail |= FL_HANG; goto done; }
    {
      const int32_t pb = (int32_t)(3u * (uint32_t)((uint32_t)boff + (uint32_t)j));
      float q2[3];
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        if (!fi_at(real, ppts, pts_real, (int32_t)((uint32_t)pb + (uint32_t)a), npts, &pe)) { fail |= FL_CRASH; goto done; }
        q2[a] = __ldg(pe);
      }
      if (KIND == TK_X2) { applied |= now; q2[0] = flip_f(q2[0], now, mask); }
      if (KIND == TK_Y2) { applied |= now; q2[1] = flip_f(q2[1], now, mask); }
      if (KIND == TK_Z2) { applied |= now; q2[2] = flip_f(q2[2], now, mask); }
      float dot = __fmaf_rn(q1[2], q2[2], __fmaf_rn(q1[1], q2[1], __fmul_rn(q1[0], q2[0])));
      if (KIND == TK_DOT) { applied |= now; dot = flip_f(dot, now, mask); }
      int32_t bin = tp_bin_search(Es, dot);
      if (KIND == TK_BIN) { applied |= now; bin = flip_i(bin, now, mask); }
      int32_t hidx = (int32_t)((uint32_t)base + (uint32_t)bin);
      if (KIND == TK_HIDX) { applied |= now; hidx = flip_i(hidx, now, mask); }
      unsigned long long* ph;
      if (!fi_at(real, phist, hist_real, hidx, nhist, &ph)) { fail |= FL_CRASH; goto done; }
      K.hist_p(ph, reinterpret_cast<const unsigned long long*>(hist_real));
      acc = (int32_t)((uint32_t)acc + (uint32_t)bin);
      if (KIND == TK_ACC) { applied |= now; acc = flip_i(acc, now, mask); }
    }
    cnt = count_inc(cnt, p.one);
    if (KIND == TK_CNT) { applied |= now; cnt = flip_i(cnt, now, mask); }
    j = (int32_t)((uint32_t)j + 1u);
  }
  if (FT) {
    if (cnt != expect) alarm |= AL_COUNT;
    if (cnt != 0 && p.ndet > 0 && p.R.n[0] > 0) {
      const float v = __fdiv_rn((float)acc, (float)cnt);
      if (!in_range<true>(p.R, 0, v, &margin, &gap)) { alarm |= AL_RANGE; K.outlier(0, v); }
    }
    chk ^= (uint32_t)opq(boff, z) ^ (uint32_t)opq(je, z) ^ (uint32_t)opq(base, z);
    chk ^= opqf(q1[0], z) ^ opqf(q1[1], z) ^ opqf(q1[2], z) ^ (uint32_t)opq(expect, z);
    chk ^= ((uint32_t)n + z) ^ (lohi(ppts) + z) ^ (lohi(phist) + z);
    if (chk != 0) alarm |= AL_CHK;
  }
done:
  K.finish(mine, alarm, fail, margin, gap, applied, (uint32_t)g);
}

// The same per-thread FI program, evaluated by the 32 lanes of one warp: lane l evaluates loop
// iteration it0 + l of the ONE faulted abstract thread.  The program's state at iteration `it` is
// a closed form of it (j = jb + it, the live values constant) except for the single flip at
// iteration f.inst, which changes the live state from then on (kinds J / LIVE) or one iteration's
// temporaries (X2 .. HIDX) or the running sums (ACC, CNT); so every lane can compute its own
// iteration directly.  The first iteration E (ballot) holding an event — loop exit, R17 watchdog,
// R16 crash, in the sequential order of the checks — ends the program exactly where the sequential
// loop would: iterations before E add their histogram increment and their bin; acc and cnt are
// rebuilt from the per-lane sums with the flip applied at its instance.  Results are identical to
// tpacf_fi_program (the replay kernel runs that one; GPU replay == replica is tested) at ~1/32 of
// its latency-bound time — a corrupted loop may run 10x the golden trips before the watchdog.
template <int KIND, bool FT, bool LUT>
__device__ void tpacf_fi_warp(const TPParams& p, const TPSmem& S, const FaultRec& f, int32_t hh, int32_t ii, int32_t i_dup,
                              int32_t h_dup, uint64_t hist_real, hk_control* cb) {
  const unsigned FULL = 0xffffffffu;
  const uint32_t lane = lane_id();
  const uint32_t z = p.z;
  const int32_t nr = p.nr, nb2 = p.nb + 2;
  const int64_t g = (int64_t)hh * p.n + ii;
  const int64_t inst = f.inst;
  const uint64_t mask = f.mask;
  const int site = f.site;
  const int64_t npts = 3LL * (1 + nr) * p.n, nhist = (int64_t)(1 + 2 * nr) * nb2;
  const uint64_t pts_real = (uint64_t)(uintptr_t)p.pts;
  uint32_t chk = 0, alarm = 0, fail = 0, margin = 0xffffffffu;
  float gap = __int_as_float(0x7f800000);
  bool applied = false;
  int32_t n = p.n;
  uint64_t ppts = pts_real, phist = hist_real;
  // ---- prologue (uniform over the warp; DESIGN §3.4 NL sites 0-10)
  if (FT) chk ^= (uint32_t)n ^ lohi(ppts) ^ lohi(phist);
  const bool nl = (KIND == TK_NL);
#define NLF(v, s) do { const bool _n = nl && site == (s); applied |= _n; v = flip_i(v, _n, mask); } while (0)
  int32_t i = ii; NLF(i, 0);
  if (FT) { chk ^= (uint32_t)i; alarm |= (i_dup != i) ? AL_DUP : 0u; }
  int32_t h = hh; NLF(h, 1);
  if (FT) { chk ^= (uint32_t)h; alarm |= (h_dup != h) ? AL_DUP : 0u; }
  auto f_aoff = [&](int32_t hq, int32_t iq) { return (int32_t)((uint32_t)(hq <= nr ? hq : 0) * (uint32_t)n + (uint32_t)iq); };
  auto f_boff = [&](int32_t hq) { return (int32_t)((uint32_t)(hq == 0 ? 0 : (hq <= nr ? hq : (int32_t)((uint32_t)hq - (uint32_t)nr))) * (uint32_t)n); };
  auto f_jb = [&](int32_t hq, int32_t iq) { return hq <= nr ? (int32_t)((uint32_t)iq + 1u) : 0; };
  auto f_ex = [&](int32_t je_, int32_t jb_) { const int32_t d = (int32_t)((uint32_t)je_ - (uint32_t)jb_); return d > 0 ? d : 0; };
  int32_t aoff = f_aoff(h, i); NLF(aoff, 2);
  if (FT) { chk ^= (uint32_t)aoff; alarm |= (f_aoff(opq(h, z), opq(i, z)) != aoff) ? AL_DUP : 0u; }
  int32_t boff = f_boff(h); NLF(boff, 3);
  if (FT) { chk ^= (uint32_t)boff; alarm |= (f_boff(opq(h, z)) != boff) ? AL_DUP : 0u; }
  int32_t jb = f_jb(h, i); NLF(jb, 4);
  if (FT) { chk ^= (uint32_t)jb; alarm |= (f_jb(opq(h, z), opq(i, z)) != jb) ? AL_DUP : 0u; }
  int32_t je = n; NLF(je, 5);
  if (FT) { chk ^= (uint32_t)je; alarm |= (opq(n, z) != je) ? AL_DUP : 0u; }
  int32_t expect = f_ex(je, jb); NLF(expect, 6);
  if (FT) { chk ^= (uint32_t)expect; alarm |= (f_ex(opq(je, z), jb) != expect) ? AL_DUP : 0u; }
  int32_t base = (int32_t)((uint32_t)h * (uint32_t)nb2); NLF(base, 7);
  if (FT) { chk ^= (uint32_t)base; alarm |= ((int32_t)((uint32_t)opq(h, z) * (uint32_t)nb2) != base) ? AL_DUP : 0u; }
#undef NLF
  float q1[3] = {0.f, 0.f, 0.f};
  for (int a = 0; a < 3; ++a) {
    const float* pe;
    if (!fi_at(false, ppts, pts_real, (int32_t)((uint32_t)aoff * 3u + (uint32_t)a), npts, &pe)) { fail |= FL_CRASH; break; }
    float v = __ldg(pe);
    { const bool nn = nl && site == 8 + a; applied |= nn; v = flip_f(v, nn, mask); }
    if (FT) { chk ^= fb(v); alarm |= (fb(__ldg(pe + z)) != fb(v)) ? AL_DUP : 0u; }
    q1[a] = v;
  }
  if (!fail) {
    if (FT) chk ^= (uint32_t)opq(i, z) ^ (uint32_t)opq(h, z) ^ (uint32_t)opq(aoff, z) ^ (uint32_t)opq(jb, z);
    // ---- the live state after the flip (kinds J / LIVE), in force from iteration inst on
    int32_t boff2 = boff, je2 = je, expect2 = expect, base2 = base, n2 = n;
    float q12[3] = {q1[0], q1[1], q1[2]};
    uint64_t ppts2 = ppts, phist2 = phist;
    if (KIND == TK_LIVE) {
      switch (site) {
        case 11: boff2 = flip_i(boff, true, mask); break;
        case 12: je2 = flip_i(je, true, mask); break;
        case 13: expect2 = flip_i(expect, true, mask); break;
        case 14: base2 = flip_i(base, true, mask); break;
        case 15: q12[0] = flip_f(q1[0], true, mask); break;
        case 16: q12[1] = flip_f(q1[1], true, mask); break;
        case 17: q12[2] = flip_f(q1[2], true, mask); break;
        case 18: n2 = flip_i(n, true, mask); break;
        case 19: ppts2 = flip_p(ppts, true, mask); break;
        case 20: phist2 = flip_p(phist, true, mask); break;
        default: break;
      }
    }
    const int32_t jflip = (int32_t)((uint32_t)jb + (uint32_t)inst) ^ (int32_t)(uint32_t)mask;  // J: j at iteration inst
    const int64_t golden = hh <= nr ? (int64_t)p.n - (ii + 1) : (int64_t)p.n;  // uncorrupted launch indices (R17)
    const int64_t limit = fi_limit<false>(golden, f.hang);
    int64_t E = -1;
    int etype = 0;      // 1 exit, 2 hang, 3 crash in the partner loads, 4 crash at the histogram
    uint32_t s_le = 0, s_gt = 0;  // this lane's bins of iterations <= inst / > inst (before E)
    const uint32_t lb = smem_u32(S.E);
    for (int64_t it0 = 0; E < 0; it0 += 32) {
      const int64_t it = it0 + lane;
      const bool post = (KIND == TK_J || KIND == TK_LIVE) && it >= inst;
      const bool now = it == inst;
      int32_t j = (int32_t)((uint32_t)jb + (uint32_t)it);
      if (KIND == TK_J && post) j = (int32_t)((uint32_t)jflip + (uint32_t)(it - inst));
      const int32_t bo = post ? boff2 : boff, jee = post ? je2 : je, ba = post ? base2 : base;
      const uint64_t pp = post ? ppts2 : ppts, ph = post ? phist2 : phist;
      const float x1 = post ? q12[0] : q1[0], y1 = post ? q12[1] : q1[1], z1 = post ? q12[2] : q1[2];
      int ev = 0;
      uint32_t bin = 0;
      unsigned long long* hp = nullptr;
      if (!(j < jee)) ev = 1;
      else if (it >= limit) ev = 2;
      else {
        const int32_t pb = (int32_t)(3u * (uint32_t)((uint32_t)bo + (uint32_t)j));
        // x2, y2, z2 in order; the first out-of-bounds load ends the thread (crash model)
        float x2 = 0.f, y2 = 0.f, z2 = 0.f;
        const float* pe;
        if (!fi_at(false, pp, pts_real, pb, npts, &pe)) ev = 3;
        else x2 = __ldg(pe);
        if (!ev) {
          if (!fi_at(false, pp, pts_real, (int32_t)((uint32_t)pb + 1u), npts, &pe)) ev = 3;
          else y2 = __ldg(pe);
        }
        if (!ev) {
          if (!fi_at(false, pp, pts_real, (int32_t)((uint32_t)pb + 2u), npts, &pe)) ev = 3;
          else z2 = __ldg(pe);
        }
        if (!ev) {
          if (KIND == TK_X2) x2 = flip_f(x2, now, mask);
          if (KIND == TK_Y2) y2 = flip_f(y2, now, mask);
          if (KIND == TK_Z2) z2 = flip_f(z2, now, mask);
          float dot = __fmaf_rn(z1, z2, __fmaf_rn(y1, y2, __fmul_rn(x1, x2)));
          if (KIND == TK_DOT) dot = flip_f(dot, now, mask);
          bin = LUT ? tp_b4_lut(S.L, lb, dot) / 4u : (uint32_t)tp_bin_search(S.E, dot);
          if (KIND == TK_BIN) bin = (uint32_t)flip_i((int32_t)bin, now, mask);
          int32_t hidx = (int32_t)((uint32_t)ba + bin);
          if (KIND == TK_HIDX) hidx = flip_i(hidx, now, mask);
          if (!fi_at(false, ph, hist_real, hidx, nhist, &hp)) ev = 4;
        }
      }
      const unsigned evs = __ballot_sync(FULL, ev != 0);
      const int first = evs ? __ffs(evs) - 1 : 32;
      if ((int)lane < first) {  // iterations before the first event: executed in full
        red_add(hp, 1ull);
        if (it <= inst) s_le += bin;
        else s_gt += bin;
      }
      if (evs) {
        E = it0 + first;
        etype = __shfl_sync(FULL, ev, first);
      }
    }
    s_le = __reduce_add_sync(FULL, s_le);
    s_gt = __reduce_add_sync(FULL, s_gt);
    // hooks of iteration inst that ran (the checks of iteration E precede its loads / increment)
    if (KIND == TK_J || KIND == TK_LIVE) applied = inst <= E;
    if (KIND == TK_X2 || KIND == TK_Y2 || KIND == TK_Z2 || KIND == TK_DOT || KIND == TK_BIN || KIND == TK_HIDX)
      applied = inst < E || (inst == E && etype == 4);
    if (KIND == TK_ACC || KIND == TK_CNT) applied = inst < E;
    if (etype == 2) fail |= FL_HANG;
    if (etype >= 3) fail |= FL_CRASH;
    if (!fail && FT) {
      const bool in_force = (KIND == TK_J || KIND == TK_LIVE) && inst <= E;  // the exit sees the flipped state
      const int32_t boffx = in_force ? boff2 : boff, jex = in_force ? je2 : je, basex = in_force ? base2 : base;
      const int32_t expx = in_force ? expect2 : expect, nx = in_force ? n2 : n;
      const float x1x = in_force ? q12[0] : q1[0], y1x = in_force ? q12[1] : q1[1], z1x = in_force ? q12[2] : q1[2];
      const uint64_t ppx = in_force ? ppts2 : ppts, phx = in_force ? phist2 : phist;
      const int32_t acc = (KIND == TK_ACC && inst < E) ? (int32_t)(((s_le) ^ (uint32_t)mask) + s_gt) : (int32_t)(s_le + s_gt);
      const int32_t cnt = (KIND == TK_CNT && inst < E) ? (int32_t)((((uint32_t)inst + 1u) ^ (uint32_t)mask) + (uint32_t)(E - 1 - inst))
                                                        : (int32_t)E;
      if (cnt != expx) alarm |= AL_COUNT;
      if (cnt != 0 && p.ndet > 0 && p.R.n[0] > 0) {
        const float v = __fdiv_rn((float)acc, (float)cnt);
        if (!in_range<true>(p.R, 0, v, &margin, &gap)) {
          alarm |= AL_RANGE;
          if (lane == 0) record_outlier(cb, 0, v);
        }
      }
      chk ^= (uint32_t)opq(boffx, z) ^ (uint32_t)opq(jex, z) ^ (uint32_t)opq(basex, z);
      chk ^= opqf(x1x, z) ^ opqf(y1x, z) ^ opqf(z1x, z) ^ (uint32_t)opq(expx, z);
      chk ^= ((uint32_t)nx + z) ^ (lohi(ppx) + z) ^ (lohi(phx) + z);
      if (chk != 0) alarm |= AL_CHK;
    }
  }
  if (!FT) alarm = 0;
  if (lane == 0) {
    TPReplicaSink K{cb};
    K.finish(true, alarm, fail, margin, gap, applied, (uint32_t)g);
  }
}

// Replica CTA (h, point block) of the FI kernel, whole partner loops, fast part.  The faulted
// abstract thread (if this CTA holds it) takes no part in the fast loop (increment 0, no exit
// checks); returns (point index, N0 duplicate) of it in the warp that holds it, else (-1, 0).
template <bool FT, bool LUT, bool GDIAG = true>
__device__ __forceinline__ int2 tp_replica_fast(const TPFIParams& q, const TPSmem& S, const FaultRec& f, unsigned long long* hist,
                                                hk_control* cb, int h, int blk, bool faulted) {
  constexpr int NP = HK_TP_NP_FI;
  constexpr int V = FT ? (V_NL | V_L) : 0;
  constexpr bool NL = FT, L = FT;
  TPParams p = q.base;
  p.hist = hist;
  p.cb = cb;
  const int i0 = blk * NP * TP_THREADS;
  const int64_t gb = (int64_t)h * p.n;
  TPPoint P[NP];
  tp_points<NP>(p, hist, h, blk, 0, INT64_MAX, P, NL);
  uint32_t inc[NP];
  int fk = -1;  // which of this thread's points is the faulted abstract thread
#pragma unroll
  for (int k = 0; k < NP; ++k) {
    const bool mine = faulted && P[k].valid && gb + P[k].i == f.thread;
    if (mine) fk = k;
    inc[k] = (P[k].valid && !mine) ? ((k & 1) ? 0x10000u : 1u) : 0u;
  }
  tp_zero_hist<NP>(p, S);
  __syncthreads();
  const int jlo = h <= p.nr ? i0 + 1 : 0;
  tp_item_loop<NP, V, LUT, GDIAG>(p, S, P, inc, h, i0, jlo, p.n);
#pragma unroll
  for (int k = 0; k < NP; ++k) {
    if (!P[k].valid || k == fk) continue;
    if (L) P[k].acc /= 4;
    tp_nl_exit<NL>(p, P[k], hist);
    tp_checks<V>(p, P[k], cb, gb + P[k].i);
  }
  if (NL || L) {
#pragma unroll
    for (int k = 0; k < NP; ++k)
      if (P[k].valid) fold_alarm(cb, k == fk ? 0u : P[k].alarm, (uint32_t)(gb + P[k].i));
  }
  __syncthreads();
  tp_flush<NP>(p, S, hist, h * (p.nb + 2));
  // the warp holding the faulted abstract thread learns its point index and N0 duplicate
  const unsigned own = __ballot_sync(0xffffffffu, fk >= 0);
  if (!own) return make_int2(-1, 0);
  const int src = __ffs(own) - 1;
  const int fkw = __shfl_sync(0xffffffffu, fk, src);
  const int t = (int)(threadIdx.x & ~31u) + src;
  return make_int2(i0 + fkw * TP_THREADS + t, (int)((blk ^ p.z) * (NP * TP_THREADS) + fkw * TP_THREADS + (t ^ (int)p.z)));
}

// Replica CTA (h, point block) of the FI kernel: the fast loop over every abstract thread but the
// faulted one, then that one's FI program on the 32 lanes of its warp.
template <int KIND, bool FT, bool LUT>
__device__ __forceinline__ void tp_replica_cta(const TPFIParams& q, const TPSmem& S, const FaultRec& f, unsigned long long* hist,
                                               hk_control* cb, int h, int blk, bool faulted) {
  const int2 fi = tp_replica_fast<FT, LUT>(q, S, f, hist, cb, h, blk, faulted);
  if (fi.x >= 0) {
    TPParams p = q.base;
    p.hist = hist;
    p.cb = cb;
    tpacf_fi_warp<KIND, FT, LUT>(p, S, f, h, fi.x, fi.y, (int)((uint32_t)h ^ p.z), (uint64_t)(uintptr_t)hist, cb);
  }
}

// Launch slots: the first nrep slots run the faulted CTA of replica 0..nrep-1 (the FI program
// makes them the longest, so they start first); the rest go CTA-major in decreasing loop length
// (DR rows, then the self rows block by block), replica-minor; the slot of a replica's faulted
// CTA in that order does nothing.
__device__ __forceinline__ void tp_cta_of_rank(int rank, int nr, int nblk, int* h, int* blk) {
  const int ndr = nr * nblk;
  if (rank < ndr) { *h = nr + 1 + rank / nblk; *blk = rank % nblk; }
  else { const int r2 = rank - ndr; *blk = r2 / (nr + 1); *h = r2 % (nr + 1); }
}

__host__ __device__ __forceinline__ int tpacf_site_kind_d(int site) {
  if (site <= 10) return TK_NL;
  if (site <= 20) return TK_LIVE;
  return TK_J + (site - 21);
}


// Replica-kernel parameters (tpacf.cu); ws holds the bucket table built by tpacf_lut_build.
TPFIParams tpacf_fi_params(const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults, unsigned long long* hist0,
                           hk_control* cb0, void* ws);

}  // namespace hk
