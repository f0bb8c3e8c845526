// tpacf.cu — two-point angular correlation histograms (K3) with HAUBERK detectors, sm_100a.
//
// Abstract program: DESIGN.md §3.4 (benchmark: Parboil TPACF; the paper cites its 1 % output rule,
// L80-84, its shared-memory footprint, L2428-2431, and its retry-until-written histogram loop that
// could hang, L2643-2649 — not reproduced: B200 shared memory increments need no retry).
// B200 shape: one CTA per (histogram h, partner chunk c, 256 points i); the chunk's partners staged
// once in shared memory as float4; bin = 5-step branch-free binary search over edges in shared
// memory (distinct entries sit in distinct banks); lane-private shared histograms [warp][bin][lane]
// (bank = lane: conflict-free), reduced per CTA and flushed with one u64 atomic per (warp, bin).
// Loop detector: accumulator acc += bin and counter cnt++ (the "two addition instructions", L679-680).
#include <algorithm>
#include <array>
#include <map>
#include <mutex>
#include <queue>
#include <vector>

#include "hk_internal.h"

namespace hk {

#ifndef HK_TP_THREADS
#define HK_TP_THREADS 128
#endif
constexpr int TP_THREADS = HK_TP_THREADS;
// Minimum resident CTAs per SM for the register allocator (measured, tools/ab_time.py): with
// 8-partner groups (HK_TP_G8) both the replicas and the single run are fastest at 9 (56
// registers; the single run spills at 10).  8-partner groups: 13.4 SASS instructions per pair
// instead of 14 (loop overhead and partner loads amortised over 16 pairs); measured FT single
// run 74.7 -> 70.7 us, replicas 52.6 -> 51.8 us.
#ifndef HK_TP_MINB
#define HK_TP_MINB 9
#endif
#ifndef HK_TP_G8
#define HK_TP_G8 1
#endif
#ifndef HK_TP_STD_MINB
#define HK_TP_STD_MINB 9
#endif
constexpr int TP_CTA_PTS = 2 * TP_THREADS;  // two abstract threads per CUDA thread
constexpr int TP_WARPS = TP_THREADS / 32;

struct TPParams {
  const float* pts;
  const float* edges;
  const uint8_t* lut;  // [TP_LUT] bmin per u-bucket; built by tpacf_lut_kernel
  const int* lut_ok;   // 1 if every bucket holds at most one edge (else: binary search)
  unsigned long long* hist;
  hk_control* cb;
  float* samples;
  DevRanges R;
  int32_t n, nr, nb, C, nC, ndet;
  uint32_t z;
  int32_t one, four, eight;  // runtime 1, 4 and 8 (opaque)
};

// ---------------------------------------------------------------------------------------------
// Binning.  Definition: bin = #{e in [0, nb] : dot < edge[e]}, edges decreasing.
//  * tp_bin: branch-free 5-step binary search over the edges (padded with -inf) in shared memory.
//  * LUT path: u = fl(1 - dot) is monotone in dot, and so is bin; bucket u by its top 11 bits
//    (sign, exponent, 2 mantissa bits).  For every bucket q the device builds
//    bmin = bin(largest dot mapping into q) and checks that the smallest dot of q has
//    bin <= bmin + 1, so bin = bmin + (dot < edge[bmin]) exactly.  The compare is taken as the
//    sign bit of fl(dot - edge[bmin]) (one FADD + one shift-add): with gradual underflow the
//    difference of two finite floats is zero only when they are equal, rounding never flips its
//    sign, a NaN result is the canonical (positive) NaN and dot - (-inf) = +inf; the one
//    disagreement, dot = -0 against an edge of +0, is removed by staging +0 edges as -0 (equal
//    under every compare).  2 loads + 5 ops per pair.
// ---------------------------------------------------------------------------------------------
constexpr int TP_LUT = 2048;
constexpr int TP_SCHED_MAX_SM = 1024;

__device__ __forceinline__ int32_t tp_bin(const float* Es, float dot) {
  int32_t b = 0;
#pragma unroll
  for (int s = 16; s >= 1; s >>= 1) b += (dot < Es[b + s - 1]) ? s : 0;
  return b;
}
// Returns 4 * bin.  The table holds 4 * bmin, the byte offset of E[bmin], so the edge load is
// [offset + shared base] with no address arithmetic; `eb` = 32-bit shared address of E (uniform).
__device__ __forceinline__ int32_t tp_bin_lut(const uint8_t* L, uint32_t eb, float dot) {
  const float u = __fsub_rn(1.0f, dot);
  const uint32_t b4 = L[fb(u) >> 21];
  float e;
  asm("ld.shared.f32 %0, [%1];" : "=f"(e) : "r"(eb + b4));
  return (int32_t)((dot < e) ? b4 + 4u : b4);
}

__device__ __forceinline__ float nup(float x) {
  const uint32_t b = fb(x);
  if ((b & 0x7fffffffu) == 0) return bf(1u);
  return (b & 0x80000000u) ? bf(b - 1) : bf(b + 1);
}
__device__ __forceinline__ float ndown(float x) {
  const uint32_t b = fb(x);
  if ((b & 0x7fffffffu) == 0) return bf(0x80000001u);
  return (b & 0x80000000u) ? bf(b + 1) : bf(b - 1);
}
__device__ __forceinline__ int32_t bin_def(const float* edges, int nb, float dot) {
  int32_t b = 0;
  for (int e = 0; e <= nb; ++e) b += (dot < edges[e]) ? 1 : 0;
  return b;
}

// One thread per bucket q.  Buckets whose u range holds no finite value (inf/NaN exponents) map
// to bin 0 for NaN (the definition: every compare with NaN is false) and nb+1 for +inf.
__global__ void tpacf_lut_kernel(const float* __restrict__ edges, int nb, uint8_t* __restrict__ lut, int* ok) {
  const int q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= TP_LUT) return;
  const float e0 = edges[0];
  int2 out = make_int2(0, fb(e0));
  bool good = true;
  const uint32_t lo_bits = (uint32_t)q << 21, hi_bits = lo_bits | 0x1fffffu;
  const bool neg = (lo_bits & 0x80000000u) != 0;
  const bool special = ((lo_bits >> 23) & 0xffu) == 0xffu;  // inf / NaN exponent
  if (neg) {
    out = make_int2(0, fb(e0));  // u <= -0: dot >= 1 > every edge -> bin 0 (and -NaN: bin 0)
  } else if (special) {
    out = (q == (int)(0x7f800000u >> 21)) ? make_int2(nb + 1, (int)0xff800000u) : make_int2(0, (int)fb(e0));
  } else {
    const float ulo = bf(lo_bits), uhi = bf(hi_bits);
    // largest dot with fl(1 - dot) >= ulo, smallest dot with fl(1 - dot) <= uhi
    float dmax = __fsub_rn(1.0f, ulo);
    for (int k = 0; k < 64 && __fsub_rn(1.0f, nup(dmax)) >= ulo; ++k) dmax = nup(dmax);
    for (int k = 0; k < 64 && __fsub_rn(1.0f, dmax) < ulo; ++k) dmax = ndown(dmax);
    float dmin = __fsub_rn(1.0f, uhi);
    for (int k = 0; k < 64 && __fsub_rn(1.0f, ndown(dmin)) <= uhi; ++k) dmin = ndown(dmin);
    for (int k = 0; k < 64 && __fsub_rn(1.0f, dmin) > uhi; ++k) dmin = nup(dmin);
    const int bmin = bin_def(edges, nb, dmax), bmax = bin_def(edges, nb, dmin);
    good = (__fsub_rn(1.0f, dmax) >= ulo) && (__fsub_rn(1.0f, dmin) <= uhi) && (bmax - bmin <= 1);
    out = make_int2(bmin, (int)(bmin <= nb ? fb(edges[bmin]) : 0xff800000u));
  }
  lut[q] = (uint8_t)(4 * out.x);  // byte offset of E[b] (padded with -inf beyond nb): the compare value
  if (!good) atomicExch(ok, 0);
}

// Dynamic shared memory: E[32] | LUT[2048] u8 | B[3 * C4] float (packed x, y, z) | H[warps][nb2][32] u32
// The partner tile keeps the global AoS layout without padding: 4 partners = 3 float4, i.e. three
// 128-bit broadcast loads (2 wavefronts each) per 4 partners instead of four (ncu source page:
// LDS.128 costs 2.1 wavefronts even as a broadcast).
__host__ __device__ inline int tp_c4(int C) { return (C + 3) & ~3; }
struct TPSmem {
  float* E;
  uint8_t* L;
  float* B;
  uint32_t* H;
};
__host__ __device__ inline size_t tp_smem_bytes(int C, int nb2) {
  return 32 * sizeof(float) + TP_LUT + (size_t)tp_c4(C) * 12 + (size_t)TP_WARPS * nb2 * 32 * 4;
}
__device__ __forceinline__ TPSmem tp_carve(unsigned char* base, int C) {
  TPSmem S;
  S.E = reinterpret_cast<float*>(base);
  S.L = base + 128;
  S.B = reinterpret_cast<float*>(base + 128 + TP_LUT);
  S.H = reinterpret_cast<uint32_t*>(base + 128 + TP_LUT + (size_t)tp_c4(C) * 12);
  return S;
}

// Does any thread of this CTA have partners?  (self rows: chunks left of the diagonal are empty)
__device__ __forceinline__ bool tp_cta_has_work(const TPParams& p, int h, int c, int bxi) {
  const int i0 = bxi * TP_CTA_PTS;
  const int jb = (h <= p.nr) ? max(i0 + 1, c * p.C) : c * p.C;
  const int je = min((c + 1) * p.C, p.n);
  return i0 < p.n && je > jb;
}

// Stage chunk c of partner set sb, the edges, the bucket table; clear the histograms.
__device__ __forceinline__ void tp_stage(const TPParams& p, const TPSmem& S, int sb, int c, bool work) {
  if (threadIdx.x < 32) {  // +0 staged as -0 (tp_bin_lut); -inf pads past the last edge
    const float e = threadIdx.x <= p.nb ? p.edges[threadIdx.x] : __int_as_float(0xff800000);
    S.E[threadIdx.x] = fb(e) == 0u ? __int_as_float(0x80000000) : e;
  }
  if (!work) return;
  const int j0 = c * p.C;
  const int cnt = min(p.C, p.n - j0);
  const float* P = p.pts + 3 * ((int64_t)sb * p.n + j0);
  for (int k = threadIdx.x; k < 3 * cnt; k += TP_THREADS) S.B[k] = P[k];
  const int4* Lg = reinterpret_cast<const int4*>(p.lut);
  int4* Ls = reinterpret_cast<int4*>(S.L);
  for (int k = threadIdx.x; k < TP_LUT / 16; k += TP_THREADS) Ls[k] = Lg[k];
  const int nh = TP_WARPS * (p.nb + 2) * 32;
  for (int k = threadIdx.x; k < nh; k += TP_THREADS) S.H[k] = 0u;
}

// Reduce the lane-private histograms and add them to hist[base + b].
__device__ __forceinline__ void tp_flush(const TPParams& p, const TPSmem& S, unsigned long long* hist, int base) {
  const int nb2 = p.nb + 2;
  for (int t = threadIdx.x; t < TP_WARPS * nb2; t += TP_THREADS) {
    const uint32_t* row = S.H + (size_t)t * 32;  // t = w * nb2 + b
    uint32_t s = 0;
#pragma unroll 8
    for (int l = 0; l < 32; ++l) s += row[(l + t) & 31];
    if (s) atomicAdd(hist + base + (t % nb2), (unsigned long long)s);
  }
}

// Per-abstract-thread prologue state (NL sites 0-11).
struct TPPoint {
  int32_t i, row, boff, jb, je, expect, base;
  float x1, y1, z1;
  uint32_t chk, alarm;
  int32_t acc, cnt;
};

template <bool NL>
__device__ __forceinline__ TPPoint tp_prologue(const TPParams& p, const unsigned long long* hist, int k, int bxi, int byi) {
  const uint32_t z = p.z;
  const int32_t n = p.n, nr = p.nr, C = p.C, nC = p.nC, nb2 = p.nb + 2;
  TPPoint P;
  P.row = byi;
  P.i = bxi * TP_CTA_PTS + k * TP_THREADS + threadIdx.x;
  const int32_t h = P.row / nC, c = P.row - h * nC;
  P.chk = 0;
  P.alarm = 0;
  if (NL) {
    P.chk ^= (uint32_t)n ^ lohi_ptr(p.pts) ^ lohi_ptr(hist);
    P.chk ^= (uint32_t)P.i;
    P.alarm |= ((int32_t)((bxi ^ z) * TP_CTA_PTS + k * TP_THREADS + (threadIdx.x ^ z)) != P.i) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)h; P.alarm |= ((int32_t)(byi ^ z) / nC != h) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)c; P.alarm |= ((int32_t)(P.row - opq(h, z) * nC) != c) ? AL_DUP : 0u;
  }
  const int32_t aoff = (h <= nr ? h : 0) * n + P.i;
  const int32_t sb = (h == 0) ? 0 : (h <= nr ? h : h - nr);
  P.boff = sb * n;
  P.jb = h <= nr ? max(P.i + 1, c * C) : c * C;
  P.je = min((c + 1) * C, n);
  P.expect = max(P.je - P.jb, 0);
  P.base = h * nb2;
  if (NL) {
    const int32_t h2 = opq(h, z), i2 = opq(P.i, z), c2 = opq(c, z);
    P.chk ^= (uint32_t)aoff; P.alarm |= ((h2 <= nr ? h2 : 0) * n + i2 != aoff) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.boff; P.alarm |= ((h2 == 0 ? 0 : (h2 <= nr ? h2 : h2 - nr)) * n != P.boff) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.jb; P.alarm |= ((h2 <= nr ? max(i2 + 1, c2 * C) : c2 * C) != P.jb) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.je; P.alarm |= (min((c2 + 1) * C, n) != P.je) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.expect; P.alarm |= (max(opq(P.je, z) - P.jb, 0) != P.expect) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)P.base; P.alarm |= (h2 * nb2 != P.base) ? AL_DUP : 0u;
  }
  const float* A = p.pts + 3 * (int64_t)aoff;
  P.x1 = A[0]; P.y1 = A[1]; P.z1 = A[2];
  if (NL) {
    const float* A2 = p.pts + 3 * (int64_t)opq(aoff, z);
    P.chk ^= fb(P.x1); P.alarm |= (fb(A2[0]) != fb(P.x1)) ? AL_DUP : 0u;
    P.chk ^= fb(P.y1); P.alarm |= (fb(A2[1]) != fb(P.y1)) ? AL_DUP : 0u;
    P.chk ^= fb(P.z1); P.alarm |= (fb(A2[2]) != fb(P.z1)) ? AL_DUP : 0u;
    P.chk ^= (uint32_t)opq(P.i, z) ^ (uint32_t)opq(h, z) ^ (uint32_t)opq(c, z) ^ (uint32_t)opq(aoff, z) ^
             (uint32_t)opq(P.jb, z);
  }
  P.acc = 0;
  P.cnt = 0;
  return P;
}

template <int V>
__device__ __forceinline__ void tp_epilogue(const TPParams& p, TPPoint& P, const unsigned long long* hist, hk_control* cb) {
  constexpr bool NL = (V & V_NL) != 0, L = (V & V_L) != 0, PROF = (V & V_PROF) != 0;
  const uint32_t z = p.z;
  if (L && P.cnt != P.expect) P.alarm |= AL_COUNT;
  if ((L || PROF) && P.cnt != 0 && p.ndet > 0) {
    const float v = __fdiv_rn((float)P.acc, (float)P.cnt);
    if (PROF) p.samples[(int64_t)P.row * p.n + P.i] = v;
    if (L && p.R.n[0] > 0 && !in_range<false>(p.R, 0, v, nullptr)) {
      P.alarm |= AL_RANGE;
      record_outlier(cb, 0, v);
    }
  }
  if (NL) {
    P.chk ^= (uint32_t)opq(P.boff, z) ^ (uint32_t)opq(P.je, z) ^ (uint32_t)opq(P.base, z);
    P.chk ^= opqf(P.x1, z) ^ opqf(P.y1, z) ^ opqf(P.z1, z) ^ (uint32_t)opq(P.expect, z);
    P.chk ^= ((uint32_t)p.n + z) ^ (lohi_ptr(p.pts) + z) ^ (lohi_ptr(hist) + z);
    if (P.chk != 0) P.alarm |= AL_CHK;
  }
}

__device__ __forceinline__ float tp_dot(const TPPoint& P, const float3 q) {
  return __fmaf_rn(P.z1, q.z, __fmaf_rn(P.y1, q.y, __fmul_rn(P.x1, q.x)));
}
template <bool LUT>
__device__ __forceinline__ int32_t tp_binof(const uint8_t* __restrict__ L, const float* __restrict__ E, uint32_t eb, float dot) {
  return LUT ? tp_bin_lut(L, eb, dot) : 4 * tp_bin(E, dot);  // 4 * bin
}
// bin4 = 4 * bin (tp_binof).  The fast path accumulates acc4 = sum of 4 * bin; tp_loops divides
// by 4 at the end: the same integer as the abstract acc (acc <= 31 * C <= 31 * 1024, no wrap).
template <bool CNT, bool INC = true>
__device__ __forceinline__ void tp_count(const TPParams& p, uint32_t* Hw, TPPoint& P, int32_t bin4) {
  // lane-private counter: no contention; the shared-memory atomic (ATOMS.POPC.INC) has no
  // register round trip, so consecutive increments do not serialise (microbenchmark: 1.34x the
  // LDS/IADD/STS read-modify-write, tools/microbench/smem_hist.cu)
  atomicAdd(Hw + bin4 * 8, 1u);
  if (CNT) {
    P.acc += bin4;
    if (INC) P.cnt = count_inc(P.cnt, p.one);
  }
}

// CTA = (row h*nC + c, 512 points); each CUDA thread runs TWO abstract threads (points i and
// i + 256, same row and chunk), each in its own ascending-j order, sharing every partner load.
// Within a group of 4 partners all loads (partner, bucket table, edge) are issued before the
// histogram read-modify-writes, which the compiler must otherwise serialise (possible aliasing).
template <int V, bool LUT>
__device__ __forceinline__ void tp_loops4(const TPParams& p, const TPSmem& S, uint32_t* Hw, TPPoint& A, TPPoint& B,
                                         bool va, bool vb) {
  constexpr bool CNT = (V & (V_L | V_PROF)) != 0;
  const uint8_t* __restrict__ L = S.L;
  const float* __restrict__ E = S.E;
  const uint32_t eb = (uint32_t)__cvta_generic_to_shared(S.E);
  const int32_t k0 = -(A.row % p.nC) * p.C;  // tile index k = j + k0
  const float* __restrict__ Pb = S.B;
  auto part = [&](int32_t k) { return make_float3(Pb[3 * k], Pb[3 * k + 1], Pb[3 * k + 2]); };
  const int32_t je = A.je;
  const int32_t ja = va ? A.jb : je, jbb = vb ? B.jb : je;  // ja <= jbb (i_a < i_b, same chunk)
  const int32_t j1 = min(jbb, je);
  // phase 1: only point A has partners
  for (int32_t j = ja; j < j1; ++j) tp_count<CNT>(p, Hw, A, tp_binof<LUT>(L, E, eb, tp_dot(A, part(j + k0))));
  if (!va) {
    for (int32_t j = jbb; j < je; ++j) tp_count<CNT>(p, Hw, B, tp_binof<LUT>(L, E, eb, tp_dot(B, part(j + k0))));
    return;
  }
  // phase 2: both points, one shared partner load; the partner pointer walks the tile and the
  // counters advance by 4 per group of 4 iterations (the strength reduction any compiler applies
  // to an unrolled it++; the FI program keeps the per-iteration increment as the injection site)
  int32_t k = max(jbb, ja) + k0;
  const int32_t kend = je + k0;
  auto both = [&](int32_t kk) {
    const float3 q = part(kk);
    const int32_t a = tp_binof<LUT>(L, E, eb, tp_dot(A, q)), b = tp_binof<LUT>(L, E, eb, tp_dot(B, q));
    tp_count<CNT>(p, Hw, A, a);
    tp_count<CNT>(p, Hw, B, b);
  };
  for (; k < kend && (k & 3); ++k) both(k);  // align to a 48-byte group (chunk starts are aligned when C % 4 == 0)
  const float4* __restrict__ T4 = reinterpret_cast<const float4*>(Pb);
#if HK_TP_G8
  for (; k + 7 < kend; k += 8) {
    const int32_t k3 = (k >> 2) * 3;
    const float4 v0 = T4[k3], v1 = T4[k3 + 1], v2 = T4[k3 + 2], v3 = T4[k3 + 3], v4 = T4[k3 + 4], v5 = T4[k3 + 5];
    const float3 q[8] = {make_float3(v0.x, v0.y, v0.z), make_float3(v0.w, v1.x, v1.y), make_float3(v1.z, v1.w, v2.x),
                         make_float3(v2.y, v2.z, v2.w), make_float3(v3.x, v3.y, v3.z), make_float3(v3.w, v4.x, v4.y),
                         make_float3(v4.z, v4.w, v5.x), make_float3(v5.y, v5.z, v5.w)};
    int32_t a[8], b[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      a[u] = tp_binof<LUT>(L, E, eb, tp_dot(A, q[u]));
      b[u] = tp_binof<LUT>(L, E, eb, tp_dot(B, q[u]));
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      tp_count<CNT, false>(p, Hw, A, a[u]);
      tp_count<CNT, false>(p, Hw, B, b[u]);
    }
    if (CNT) {
      A.cnt = count_inc(A.cnt, p.eight);
      B.cnt = count_inc(B.cnt, p.eight);
    }
  }
#endif
  for (; k + 3 < kend; k += 4) {
    const int32_t k3 = (k >> 2) * 3;
    const float4 v0 = T4[k3], v1 = T4[k3 + 1], v2 = T4[k3 + 2];
    const float3 q0 = make_float3(v0.x, v0.y, v0.z), q1 = make_float3(v0.w, v1.x, v1.y);
    const float3 q2 = make_float3(v1.z, v1.w, v2.x), q3 = make_float3(v2.y, v2.z, v2.w);
    const int32_t a0 = tp_binof<LUT>(L, E, eb, tp_dot(A, q0)), b0 = tp_binof<LUT>(L, E, eb, tp_dot(B, q0));
    const int32_t a1 = tp_binof<LUT>(L, E, eb, tp_dot(A, q1)), b1 = tp_binof<LUT>(L, E, eb, tp_dot(B, q1));
    const int32_t a2 = tp_binof<LUT>(L, E, eb, tp_dot(A, q2)), b2 = tp_binof<LUT>(L, E, eb, tp_dot(B, q2));
    const int32_t a3 = tp_binof<LUT>(L, E, eb, tp_dot(A, q3)), b3 = tp_binof<LUT>(L, E, eb, tp_dot(B, q3));
    tp_count<CNT, false>(p, Hw, A, a0); tp_count<CNT, false>(p, Hw, B, b0);
    tp_count<CNT, false>(p, Hw, A, a1); tp_count<CNT, false>(p, Hw, B, b1);
    tp_count<CNT, false>(p, Hw, A, a2); tp_count<CNT, false>(p, Hw, B, b2);
    tp_count<CNT, false>(p, Hw, A, a3); tp_count<CNT, false>(p, Hw, B, b3);
    if (CNT) {
      A.cnt = count_inc(A.cnt, p.four);
      B.cnt = count_inc(B.cnt, p.four);
    }
  }
  for (; k < kend; ++k) both(k);
}

template <int V, bool LUT>
__device__ __forceinline__ void tp_loops(const TPParams& p, const TPSmem& S, uint32_t* Hw, TPPoint& A, TPPoint& B,
                                         bool va, bool vb) {
  tp_loops4<V, LUT>(p, S, Hw, A, B, va, vb);
  A.acc >>= 2;
  B.acc >>= 2;
}

template <int V>
__device__ __forceinline__ void tpacf_body(const TPParams& p, const TPSmem& S, unsigned long long* hist, hk_control* cb,
                                           int bxi, int byi) {
  constexpr bool NL = (V & V_NL) != 0, L = (V & V_L) != 0;
  const int32_t nr = p.nr, nC = p.nC, nb2 = p.nb + 2;
  const int32_t row = byi;
  const int32_t h = row / nC, c = row - h * nC;
  const int32_t sb = (h == 0) ? 0 : (h <= nr ? h : h - nr);
  const bool work = tp_cta_has_work(p, h, c, bxi);
  const bool use_lut = *p.lut_ok != 0;
  tp_stage(p, S, sb, c, work);
  __syncthreads();
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  uint32_t* Hw = S.H + (size_t)warp * nb2 * 32 + lane;
  TPPoint A = tp_prologue<NL>(p, hist, 0, bxi, byi);
  TPPoint B = tp_prologue<NL>(p, hist, 1, bxi, byi);
  const bool va = A.i < p.n, vb = B.i < p.n;
  if (use_lut) tp_loops<V, true>(p, S, Hw, A, B, va, vb);
  else tp_loops<V, false>(p, S, Hw, A, B, va, vb);
  if (va) {
    tp_epilogue<V>(p, A, hist, cb);
    if (NL || L) fold_alarm(cb, A.alarm, (uint32_t)((int64_t)row * p.n + A.i));
  }
  if (vb) {
    tp_epilogue<V>(p, B, hist, cb);
    if (NL || L) fold_alarm(cb, B.alarm, (uint32_t)((int64_t)row * p.n + B.i));
  }
  if (work) {
    __syncthreads();
    tp_flush(p, S, hist, h * nb2);
  }
}

// Single-run schedule.  At the configs' sizes the single run is one wave whose CTAs carry very
// different work (full chunks, diagonal triangles, empty chunks left of the diagonal), so the
// block scheduler's placement left the busiest SM with ~1.3x the mean work (ncu
// sm__cycles_active max/avg).  The host assigns the (point block, row) work items to SMs by
// longest-processing-time greedy on their exact pair counts; a persistent grid of k CTAs per SM
// claims the items of its own SM's list (%smid).  The claim of the next item is issued before the
// current item runs, so its latency overlaps the work.  Completion does not depend on placement:
// the last CTA to finish sweeps every list for items nobody claimed (an SM that received no CTA).
// Same abstract threads, same per-thread order: only which CTA runs an item changes.
struct TPSched {
  const int2* items;  // (bxi, row), grouped by SM
  const int* off;     // [nsm + 1] list offsets
  int* next;          // [nsm] claim counters (zeroed per run)
  int* claimed;       // items claimed so far (zeroed per run)
  int* exited;        // CTAs finished (zeroed per run)
  int nsm, total;
};

__device__ __forceinline__ int tp_claim(const TPSched& q, int sl) {
  const int k = atomicAdd(q.next + sl, 1);
  if (q.off[sl] + k >= q.off[sl + 1]) return -1;
  atomicAdd(q.claimed, 1);
  return q.off[sl] + k;
}

template <int V>
__device__ __forceinline__ void tp_drain(const TPParams& p, const TPSmem& S, const TPSched& q, int sl, int* item_s) {
  if (threadIdx.x == 0) *item_s = tp_claim(q, sl);
  for (;;) {
    __syncthreads();
    const int it = *item_s;
    __syncthreads();  // everyone has read the current item before thread 0 overwrites it
    if (it < 0) break;
    int nxt = -1;
    if (threadIdx.x == 0) nxt = tp_claim(q, sl);  // result consumed after the item: latency hidden
    const int2 xy = q.items[it];
    tpacf_body<V>(p, S, p.hist, p.cb, xy.x, xy.y);
    if (threadIdx.x == 0) *item_s = nxt;
  }
}

template <int V>
// the NL-only variant (Fig. 13 decomposition) spills at 56 registers: it gets 64 (8 CTAs per SM)
__global__ void __launch_bounds__(TP_THREADS, V == V_NL ? 8 : HK_TP_STD_MINB) tpacf_kernel(const TPParams p, const TPSched q) {
  extern __shared__ __align__(16) unsigned char tp_smem[];
  __shared__ int item_s, last_s;
  const TPSmem S = tp_carve(tp_smem, p.C);
  uint32_t smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  tp_drain<V>(p, S, q, (int)(smid % (uint32_t)q.nsm), &item_s);
  if (threadIdx.x == 0) {
    __threadfence();
    last_s = (atomicAdd(q.exited, 1) == (int)gridDim.x - 1) && (*(volatile int*)q.claimed < q.total);
  }
  __syncthreads();
  if (last_s)
    for (int sl = 0; sl < q.nsm; ++sl) tp_drain<V>(p, S, q, sl, &item_s);
}

// ============================================================================================
// FI & FT replicas (blockIdx.z = replica)
// ============================================================================================
enum TPKind : int { TK_NL = 0, TK_LIVE, TK_J, TK_X2, TK_Y2, TK_Z2, TK_DOT, TK_BIN, TK_HIDX, TK_ACC, TK_CNT, TK_COUNT };

struct TPFIParams {
  TPParams base;
  const FaultRec* faults;
  unsigned long long* hist0;  // replica r: hist0 + r * nh * nb2
  hk_control* cb0;
  int64_t hist_elems;
};

// Histogram sinks of the per-thread TPACF FI program.  Replica: the faulted thread adds to the
// replica's global histogram through its (possibly corrupted) index, the CTA's fault-free threads
// use their lane-private shared counters.  Replay: every increment of the one thread is folded
// into deltas of the 3*nb outputs (DD, DRS, RRS of R4) with a sign (+1 faulted run, -1 golden twin).
struct TPReplicaSink {
  unsigned long long* hist;
  hk_control* cb;
  uint32_t* H;  // lane-private counters of this CTA's row
  int nb2;
  __device__ __forceinline__ bool global_path(bool mine) const { return mine; }
  __device__ __forceinline__ void hist_global(int64_t e) { atomicAdd(hist + e, 1ull); }
  __device__ __forceinline__ void hist_p(unsigned long long* ptr, const unsigned long long*) { red_add(ptr, 1ull); }
  __device__ __forceinline__ void hist_local(uint32_t warp, int32_t bin, uint32_t lane) {
    H[((size_t)warp * nb2 + bin) * 32 + lane] += 1u;
  }
  __device__ __forceinline__ void outlier(int d, float v) { record_outlier(cb, d, v); }
  __device__ __forceinline__ void finish(bool mine, uint32_t alarm, uint32_t fail, uint32_t margin, float gap,
                                         bool applied, uint32_t tid) {
    if (fail) atomicOr(&cb->fail, fail);
    if (mine) {
      cb->fault_applied = applied ? 1u : 0u;
      cb->check_margin = margin;
      cb->check_gap = gap;
    }
    fold_alarm(cb, alarm, tid);
  }
};
constexpr int TP_REPLAY_OUT = 96;  // 3 * n_bins (n_bins <= 30 for the replay kernel) + slack
struct TPReplaySink {
  int nr, nb, nb2, sign;
  int32_t* delta;  // [3 * nb]: DD, DRS, RRS for bins 1..nb
  uint32_t alarm = 0, fail = 0, margin = 0xffffffffu;
  float gap = __builtin_huge_valf();
  __device__ __forceinline__ bool global_path(bool) const { return true; }
  __device__ __forceinline__ void hist_global(int64_t e) {
    const int row = (int)(e / nb2), b = (int)(e % nb2);
    if (b < 1 || b > nb) return;  // under/overflow bins are not outputs (R4)
    const int kind = row == 0 ? 0 : (row <= nr ? 2 : 1);
    delta[kind * nb + b - 1] += sign;
  }
  __device__ __forceinline__ void hist_p(unsigned long long* ptr, const unsigned long long* base) { hist_global(ptr - base); }
  __device__ __forceinline__ void hist_local(uint32_t, int32_t, uint32_t) {}
  __device__ __forceinline__ void outlier(int, float) {}
  __device__ __forceinline__ void finish(bool, uint32_t a, uint32_t f, uint32_t m, float g, bool, uint32_t) {
    alarm = a; fail = f; margin = m; gap = g;
  }
};

// Per-thread FI&FT program of abstract thread g = row*N + ii.  i_dup: N0's duplicate from launch
// indices (replica) or from the abstract id (replay); hist_real: the histogram's true base.
// REAL: the guardian's unguarded variant (R25) — no R16 guards, no R17 watchdog.
template <int KIND, bool REAL = false, class Sink>
__device__ void tpacf_fi_program(const TPParams& p, const TPSmem& S, const FaultRec& f, int32_t row, int32_t ii,
                                 int32_t i_dup, int32_t row_dup, bool mine, uint64_t hist_real, Sink& K) {
  const uint32_t z = p.z;
  const int32_t nr = p.nr, C = p.C, nC = p.nC, nb2 = p.nb + 2;
  const int64_t g = (int64_t)row * p.n + ii;
  const int64_t inst = mine ? f.inst : -1;
  const uint64_t mask = f.mask;
  const int site = f.site;
  const int64_t npts = 3LL * (1 + nr) * p.n, nhist = (int64_t)(1 + 2 * nr) * nb2;
  const uint64_t pts_real = (uint64_t)(uintptr_t)p.pts;
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  uint32_t chk = 0, alarm = 0, fail = 0, margin = 0xffffffffu;
  float gap = __int_as_float(0x7f800000);
  bool applied = false;
  int32_t n = p.n;
  uint64_t ppts = pts_real, phist = hist_real;
  chk ^= (uint32_t)n ^ lohi(ppts) ^ lohi(phist);
  const bool nl = (KIND == TK_NL) && mine;
#define NLF(v, s) do { const bool _n = nl && site == (s); applied |= _n; v = flip_i(v, _n, mask); } while (0)
  int32_t i = ii; NLF(i, 0);
  chk ^= (uint32_t)i;
  alarm |= (i_dup != i) ? AL_DUP : 0u;
  int32_t h = row / nC; NLF(h, 1);
  chk ^= (uint32_t)h; alarm |= (row_dup / nC != h) ? AL_DUP : 0u;
  int32_t c = (int32_t)((uint32_t)row - (uint32_t)h * (uint32_t)nC); NLF(c, 2);
  chk ^= (uint32_t)c; alarm |= ((int32_t)((uint32_t)row - (uint32_t)opq(h, z) * (uint32_t)nC) != c) ? AL_DUP : 0u;
  auto f_aoff = [&](int32_t hh, int32_t i_) { return (int32_t)((uint32_t)(hh <= nr ? hh : 0) * (uint32_t)n + (uint32_t)i_); };
  auto f_boff = [&](int32_t hh) { return (int32_t)((uint32_t)(hh == 0 ? 0 : (hh <= nr ? hh : (int32_t)((uint32_t)hh - (uint32_t)nr))) * (uint32_t)n); };
  auto f_jb = [&](int32_t hh, int32_t i_, int32_t cc) {
    const int32_t cC = (int32_t)((uint32_t)cc * (uint32_t)C), ip = (int32_t)((uint32_t)i_ + 1u);
    return hh <= nr ? (ip > cC ? ip : cC) : cC;
  };
  auto f_je = [&](int32_t cc) { const int32_t e = (int32_t)((uint32_t)(cc + 1) * (uint32_t)C); return e < n ? e : n; };
  auto f_ex = [&](int32_t je_, int32_t jb_) { const int32_t d = (int32_t)((uint32_t)je_ - (uint32_t)jb_); return d > 0 ? d : 0; };
  int32_t aoff = f_aoff(h, i); NLF(aoff, 3);
  chk ^= (uint32_t)aoff; alarm |= (f_aoff(opq(h, z), opq(i, z)) != aoff) ? AL_DUP : 0u;
  int32_t boff = f_boff(h); NLF(boff, 4);
  chk ^= (uint32_t)boff; alarm |= (f_boff(opq(h, z)) != boff) ? AL_DUP : 0u;
  int32_t jb = f_jb(h, i, c); NLF(jb, 5);
  chk ^= (uint32_t)jb; alarm |= (f_jb(opq(h, z), opq(i, z), opq(c, z)) != jb) ? AL_DUP : 0u;
  int32_t je = f_je(c); NLF(je, 6);
  chk ^= (uint32_t)je; alarm |= (f_je(opq(c, z)) != je) ? AL_DUP : 0u;
  int32_t expect = f_ex(je, jb); NLF(expect, 7);
  chk ^= (uint32_t)expect; alarm |= (f_ex(opq(je, z), jb) != expect) ? AL_DUP : 0u;
  int32_t base = (int32_t)((uint32_t)h * (uint32_t)nb2); NLF(base, 8);
  chk ^= (uint32_t)base; alarm |= ((int32_t)((uint32_t)opq(h, z) * (uint32_t)nb2) != base) ? AL_DUP : 0u;
#undef NLF
  float q1[3];
  int32_t acc = 0, cnt = 0, j;
  const float* pe;
  const int32_t row_c = row - (row / nC) * nC;  // uncorrupted launch chunk (watchdog)
  const int32_t g_jb = (row / nC) <= nr ? max(ii + 1, row_c * C) : row_c * C;
  const int32_t g_je = min((row_c + 1) * C, p.n);
  const int64_t golden = g_je > g_jb ? g_je - g_jb : 0;
  const int64_t limit = fi_limit<REAL>(golden);
  constexpr bool real = REAL;
  for (int a = 0; a < 3; ++a) {
    if (!fi_at(real, ppts, pts_real, (int32_t)((uint32_t)aoff * 3u + (uint32_t)a), npts, &pe)) { fail |= FL_CRASH; goto done; }
    float v = __ldg(pe);
    { const bool nn = nl && site == 9 + a; applied |= nn; v = flip_f(v, nn, mask); }
    chk ^= fb(v); alarm |= (fb(__ldg(pe + z)) != fb(v)) ? AL_DUP : 0u;
    q1[a] = v;
  }
  chk ^= (uint32_t)opq(i, z) ^ (uint32_t)opq(h, z) ^ (uint32_t)opq(c, z) ^ (uint32_t)opq(aoff, z) ^ (uint32_t)opq(jb, z);
  j = jb;
  for (int64_t it = 0;; ++it) {
    const bool now = (it == inst);
    if (KIND == TK_J) { applied |= now; j = flip_i(j, now, mask); }
    if (KIND == TK_LIVE && now) {
      applied = true;
      switch (site) {
        case 12: boff = flip_i(boff, true, mask); break;
        case 13: je = flip_i(je, true, mask); break;
        case 14: expect = flip_i(expect, true, mask); break;
        case 15: base = flip_i(base, true, mask); break;
        case 16: q1[0] = flip_f(q1[0], true, mask); break;
        case 17: q1[1] = flip_f(q1[1], true, mask); break;
        case 18: q1[2] = flip_f(q1[2], true, mask); break;
        case 19: n = flip_i(n, true, mask); break;
        case 20: ppts = flip_p(ppts, true, mask); break;
        case 21: phist = flip_p(phist, true, mask); break;
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
      int32_t bin = tp_bin(S.E, dot);
      if (KIND == TK_BIN) { applied |= now; bin = flip_i(bin, now, mask); }
      int32_t hidx = (int32_t)((uint32_t)base + (uint32_t)bin);
      if (KIND == TK_HIDX) { applied |= now; hidx = flip_i(hidx, now, mask); }
      if (K.global_path(mine)) {
        unsigned long long* ph;
        if (!fi_at(real, phist, hist_real, hidx, nhist, &ph)) { fail |= FL_CRASH; goto done; }
        K.hist_p(ph, reinterpret_cast<const unsigned long long*>(hist_real));
      } else {
        K.hist_local(warp, bin, lane);  // fault-free thread: hidx == base + bin (this CTA's row)
      }
      acc = (int32_t)((uint32_t)acc + (uint32_t)bin);
      if (KIND == TK_ACC) { applied |= now; acc = flip_i(acc, now, mask); }
    }
    cnt = count_inc(cnt, p.one);
    if (KIND == TK_CNT) { applied |= now; cnt = flip_i(cnt, now, mask); }
    j = (int32_t)((uint32_t)j + 1u);
  }
  if (cnt != expect) alarm |= AL_COUNT;
  if (cnt != 0 && p.ndet > 0 && p.R.n[0] > 0) {
    const float v = __fdiv_rn((float)acc, (float)cnt);
    if (!in_range<true>(p.R, 0, v, &margin, &gap)) { alarm |= AL_RANGE; K.outlier(0, v); }
  }
  chk ^= (uint32_t)opq(boff, z) ^ (uint32_t)opq(je, z) ^ (uint32_t)opq(base, z);
  chk ^= opqf(q1[0], z) ^ opqf(q1[1], z) ^ opqf(q1[2], z) ^ (uint32_t)opq(expect, z);
  chk ^= ((uint32_t)n + z) ^ (lohi(ppts) + z) ^ (lohi(phist) + z);
  if (chk != 0) alarm |= AL_CHK;
done:
  K.finish(mine, alarm, fail, margin, gap, applied, (uint32_t)g);
}

// The CTA that holds the faulted abstract thread: every thread runs the per-thread program.
template <int KIND, bool REAL>
__device__ __forceinline__ void tpacf_fi_cta(const TPFIParams& q, const TPSmem& S, const FaultRec& f,
                                             unsigned long long* hist, hk_control* cb, int bxi, int byi) {
  {
    const TPParams& p = q.base;
    const int32_t h = byi / p.nC, c = byi - h * p.nC;
    const int32_t sb = (h == 0) ? 0 : (h <= p.nr ? h : h - p.nr);
    tp_stage(p, S, sb, c, true);
    __syncthreads();
    TPReplicaSink K{hist, cb, S.H, p.nb + 2};
#pragma unroll 1
    for (int kpt = 0; kpt < 2; ++kpt) {
      const int32_t ii = bxi * TP_CTA_PTS + kpt * TP_THREADS + threadIdx.x;
      if (ii < p.n) {
        const int32_t idup = (int32_t)((bxi ^ p.z) * TP_CTA_PTS + kpt * TP_THREADS + (threadIdx.x ^ p.z));
        const int64_t g = (int64_t)byi * p.n + ii;
        tpacf_fi_program<KIND, REAL>(p, S, f, (int32_t)byi, ii, idup, (int32_t)((uint32_t)byi ^ p.z),
                                     g == f.thread, (uint64_t)(uintptr_t)hist, K);
      }
    }
    __syncthreads();
    tp_flush(p, S, hist, h * (p.nb + 2));
  }
}

template <int KIND>
__global__ void __launch_bounds__(TP_THREADS, HK_TP_MINB) tpacf_fi_kernel(const TPFIParams q) {
  extern __shared__ __align__(16) unsigned char tp_smem[];
  const TPSmem S = tp_carve(tp_smem, q.base.C);
  const int64_t gx = gridDim.x, ncta = gx * gridDim.y, n = q.base.n;
  int r;
  int64_t cta;
  const bool faulted = fi_order(((int64_t)blockIdx.z * gridDim.y + blockIdx.y) * gx + blockIdx.x, ncta, (int)gridDim.z,
                                [&](int rr) {
                                  const int64_t g = q.faults[rr].thread;
                                  return clamp_cta((g / n) * gx + (g % n) / TP_CTA_PTS, ncta);
                                },
                                &r, &cta);
  const FaultRec f = q.faults[r];
  unsigned long long* hist = q.hist0 + (int64_t)r * q.hist_elems;
  hk_control* cb = q.cb0 + r;
  const int bxi = (int)(cta % gx), byi = (int)(cta / gx);
  if (!faulted) tpacf_body<V_NL | V_L>(q.base, S, hist, cb, bxi, byi);
  else tpacf_fi_cta<KIND, false>(q, S, f, hist, cb, bxi, byi);
}

// Unguarded replicas for the guardian (campaign mode 2, DESIGN R25): every CTA runs the per-thread
// program with REAL = true; the site kind is a runtime switch (one injection per launch).
__global__ void __launch_bounds__(TP_THREADS) tpacf_real_kernel(const TPFIParams q, int kind) {
  extern __shared__ __align__(16) unsigned char tp_smem[];
  const TPSmem S = tp_carve(tp_smem, q.base.C);
  const int r = blockIdx.z;
  const FaultRec f = q.faults[r];
  unsigned long long* hist = q.hist0 + (int64_t)r * q.hist_elems;
  hk_control* cb = q.cb0 + r;
  switch (kind) {
#define K(k) case k: tpacf_fi_cta<k, true>(q, S, f, hist, cb, blockIdx.x, blockIdx.y); break;
    K(TK_NL) K(TK_LIVE) K(TK_J) K(TK_X2) K(TK_Y2) K(TK_Z2) K(TK_DOT) K(TK_BIN) K(TK_HIDX) K(TK_ACC) K(TK_CNT)
#undef K
    default: break;
  }
}

// ============================================================================================
// Replay accelerator: one CUDA thread per injection runs the golden twin (-1) and the faulted
// abstract thread (+1) into deltas of the 3*nb outputs, then applies the 1 % rule (R3/R4).
// ============================================================================================
struct TPReplayParams {
  TPParams base;
  const FaultRec* faults;
  int nrep;
  const unsigned long long* golden;
  hk_outcome* records;
  int64_t first;
  int64_t* counts;
  int64_t* site_counts;
};

template <int KIND>
__device__ __forceinline__ void tpacf_replay_one(const TPReplayParams& q, const FaultRec& f, float* Es) {
  const TPParams& p = q.base;
  TPSmem S{};
  S.E = Es;
  const int32_t row = (int32_t)(f.thread / p.n), ii = (int32_t)(f.thread % p.n);
  int32_t delta[TP_REPLAY_OUT];
  for (int o = 0; o < 3 * p.nb; ++o) delta[o] = 0;
  const uint64_t hist_real = (uint64_t)(uintptr_t)q.golden;
  TPReplaySink twin{p.nr, p.nb, p.nb + 2, -1, delta};
  tpacf_fi_program<KIND>(p, S, f, row, ii, opq(ii, p.z), (int32_t)((uint32_t)row ^ p.z), false, hist_real, twin);
  TPReplaySink K{p.nr, p.nb, p.nb + 2, +1, delta};
  tpacf_fi_program<KIND>(p, S, f, row, ii, opq(ii, p.z), (int32_t)((uint32_t)row ^ p.z), true, hist_real, K);
  bool wrong = false;
  float worst = 0.f;
  if (!K.fail) {
    const int nb = p.nb, nb2 = p.nb + 2, nr = p.nr;
    for (int o = 0; o < 3 * nb; ++o) {
      if (delta[o] == 0) continue;
      const int kind = o / nb, b = 1 + o % nb;
      long long g = 0;
      if (kind == 0) g = (long long)q.golden[b];
      for (int s2 = 1; s2 <= nr; ++s2) {
        const int rr = kind == 1 ? nr + s2 : s2;
        if (kind != 0) g += (long long)q.golden[rr * nb2 + b];
      }
      const long long d = delta[o] < 0 ? -(long long)delta[o] : (long long)delta[o];
      if (100 * d > g) wrong = true;
      const float qv = g > 0 ? (float)(100.0 * (double)d / (double)g) : __int_as_float(0x7f800000);
      worst = fmaxf(worst, qv);
    }
  }
  emit_outcome(HK_TPACF, f, wrong, K.alarm, K.fail, 0u, K.margin, K.gap, worst, q.records, q.first, q.counts,
               q.site_counts);
}

__host__ __device__ __forceinline__ int tpacf_site_kind_d(int site) {
  if (site <= 11) return TK_NL;
  if (site <= 21) return TK_LIVE;
  return TK_J + (site - 22);
}

__global__ void __launch_bounds__(128) tpacf_replay_all_kernel(const TPReplayParams q) {
  __shared__ float Es[32];
  const TPParams& p = q.base;
  if (threadIdx.x < 32) Es[threadIdx.x] = threadIdx.x <= p.nb ? p.edges[threadIdx.x] : __int_as_float(0xff800000);
  __syncthreads();
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= q.nrep) return;
  const FaultRec f = q.faults[r];
  switch (tpacf_site_kind_d(f.site)) {
#define K(k) case k: tpacf_replay_one<k>(q, f, Es); break;
    K(TK_NL) K(TK_LIVE) K(TK_J) K(TK_X2) K(TK_Y2) K(TK_Z2) K(TK_DOT) K(TK_BIN) K(TK_HIDX) K(TK_ACC) K(TK_CNT)
#undef K
    default: break;
  }
}

// ============================================================================================
// Host launchers
// ============================================================================================
static TPParams tp_params(const hk_tpacf_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                          void* lut_ws) {
  TPParams p{};
  p.pts = a.pts;
  p.edges = a.edges;
  p.lut = reinterpret_cast<const uint8_t*>(lut_ws);
  p.lut_ok = reinterpret_cast<const int*>(reinterpret_cast<const char*>(lut_ws) + TP_LUT);
  p.hist = a.hist;
  p.cb = cb;
  p.samples = samples;
  p.R = R;
  p.n = a.n;
  p.nr = a.n_rand;
  p.nb = a.n_bins;
  p.C = a.chunk;
  p.nC = (a.n + a.chunk - 1) / a.chunk;
  p.ndet = ndet;
  p.z = opaque_zero();
  p.one = 1 + (int32_t)opaque_zero();
  p.four = 4 * p.one;
  p.eight = 8 * p.one;
  return p;
}

// workspace: bucket table | ok flag (16 B) | single-run schedule counters next[TP_SCHED_MAX_SM], claimed, exited
size_t tpacf_lut_ws_bytes() { return TP_LUT + 16 + (TP_SCHED_MAX_SM + 2) * sizeof(int); }

cudaError_t tpacf_lut_build(const hk_tpacf_args& a, void* lut_ws, cudaStream_t s) {
  int* ok = reinterpret_cast<int*>(reinterpret_cast<char*>(lut_ws) + TP_LUT);
  cudaError_t e = cudaMemsetAsync(ok, 1, sizeof(int), s);
  if (e != cudaSuccess) return e;
  e = cudaMemsetAsync(reinterpret_cast<char*>(lut_ws) + TP_LUT + 16, 0, (TP_SCHED_MAX_SM + 2) * sizeof(int), s);
  if (e != cudaSuccess) return e;
  tpacf_lut_kernel<<<TP_LUT / 256, 256, 0, s>>>(a.edges, a.n_bins, reinterpret_cast<uint8_t*>(lut_ws), ok);
  count_launch();
  return cudaGetLastError();
}

static double tp_pairs(const TPParams& p) {
  const double n = p.n;
  return (1 + p.nr) * n * (n - 1) / 2 + p.nr * n * n;
}

// Host side of the single-run schedule: exact pair count per (point block, row) work item,
// LPT assignment to the SMs, cached per (shape, SM count, device).
struct TPSchedBuf {
  int2* items = nullptr;
  int* off = nullptr;
  int total = 0;
};
static cudaError_t tp_schedule(const TPParams& p, int nsm, int row0, int row1, TPSchedBuf* out) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  static std::mutex mu;
  static std::map<std::array<int, 7>, TPSchedBuf> cache;
  const std::array<int, 7> key{p.n, p.nr, p.C, nsm, dev, row0, row1};
  std::lock_guard<std::mutex> lk(mu);
  auto f = cache.find(key);
  if (f != cache.end()) { *out = f->second; return cudaSuccess; }
  const int gx = (p.n + TP_CTA_PTS - 1) / TP_CTA_PTS, gy = (1 + 2 * p.nr) * p.nC;
  std::vector<std::pair<double, int2>> w;
  w.reserve((size_t)gx * gy);
  for (int row = std::max(row0, 0); row < std::min(row1, gy); ++row) {  // rows [row0, row1): sharding
    const int h = row / p.nC, c = row - h * p.nC;
    const int64_t cb = (int64_t)c * p.C, ce = std::min<int64_t>(cb + p.C, p.n);
    for (int b = 0; b < gx; ++b) {
      const int64_t i0 = (int64_t)b * TP_CTA_PTS, i1 = std::min<int64_t>(i0 + TP_CTA_PTS, p.n);
      double pairs = 0;
      for (int64_t i = i0; i < i1; ++i) pairs += (double)std::max<int64_t>(0, ce - (h <= p.nr ? std::max(i + 1, cb) : cb));
      // + the per-abstract-thread prologue/epilogue (~64 pair-equivalents) that even empty items run
      w.push_back({pairs + 64.0 * (double)(i1 - i0), make_int2(b, row)});
    }
  }
  std::stable_sort(w.begin(), w.end(), [](const auto& a, const auto& b) { return a.first > b.first; });
  std::vector<std::vector<int2>> lists(nsm);
  std::priority_queue<std::pair<double, int>, std::vector<std::pair<double, int>>, std::greater<>> load;
  for (int m = 0; m < nsm; ++m) load.push({0.0, m});
  for (const auto& it : w) {
    auto top = load.top();
    load.pop();
    lists[top.second].push_back(it.second);
    load.push({top.first + it.first, top.second});
  }
  std::vector<int2> items;
  std::vector<int> off(nsm + 1, 0);
  for (int m = 0; m < nsm; ++m) {
    off[m] = (int)items.size();
    items.insert(items.end(), lists[m].begin(), lists[m].end());
  }
  off[nsm] = (int)items.size();
  TPSchedBuf B;
  B.total = (int)items.size();
  if ((e = cudaMalloc(&B.items, sizeof(int2) * std::max<size_t>(1, items.size()))) != cudaSuccess) return e;
  if ((e = cudaMalloc(&B.off, sizeof(int) * off.size())) != cudaSuccess) return e;
  if (!items.empty() && (e = cudaMemcpy(B.items, items.data(), sizeof(int2) * items.size(), cudaMemcpyHostToDevice)) != cudaSuccess)
    return e;
  if ((e = cudaMemcpy(B.off, off.data(), sizeof(int) * off.size(), cudaMemcpyHostToDevice)) != cudaSuccess) return e;
  cache[key] = B;
  *out = B;
  return cudaSuccess;
}

template <int V>
static cudaError_t launch_tp_v(const TPParams& p, void* lut_ws, cudaStream_t s, int row0, int row1) {
  const size_t smem = tp_smem_bytes(p.C, p.nb + 2);
  cudaError_t e = cudaFuncSetAttribute(tpacf_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (p.n <= 0) return cudaSuccess;
  int dev = 0, nsm = 0, per_sm = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if (nsm > TP_SCHED_MAX_SM) return cudaErrorInvalidValue;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, tpacf_kernel<V>, TP_THREADS, smem)) != cudaSuccess) return e;
  TPSchedBuf B;
  if ((e = tp_schedule(p, nsm, row0, row1, &B)) != cudaSuccess) return e;
  TPSched q;
  q.items = B.items;
  q.off = B.off;
  q.next = reinterpret_cast<int*>(reinterpret_cast<char*>(lut_ws) + TP_LUT + 16);
  q.claimed = q.next + TP_SCHED_MAX_SM;
  q.exited = q.claimed + 1;
  q.nsm = nsm;
  q.total = B.total;
#ifdef HK_TP_STD_CTAS
  per_sm = std::min(per_sm, HK_TP_STD_CTAS);
#endif
  const int grid = nsm * std::max(1, std::min(per_sm, (B.total + nsm - 1) / nsm));
  TimedScope ts(HK_TPACF, 0, tp_pairs(p), s);
  tpacf_kernel<V><<<grid, TP_THREADS, smem, s>>>(p, q);
  count_launch();
  return cudaGetLastError();
}

// rows [row0, row1) of (histogram h, chunk c) work rows, row = h*nC + c (row1 < 0: all): the
// abstract threads of those rows, their counts added into hist (single-run sharding).
cudaError_t tpacf_launch(int vflags, const hk_tpacf_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                         void* lut_ws, cudaStream_t s, int32_t row0, int32_t row1) {
  cudaError_t e = tpacf_lut_build(a, lut_ws, s);
  if (e != cudaSuccess) return e;
  const TPParams p = tp_params(a, R, ndet, cb, samples, lut_ws);
  if (row1 < 0) row1 = (1 + 2 * p.nr) * p.nC;
  switch (vflags) {
    case 0: return launch_tp_v<0>(p, lut_ws, s, row0, row1);
    case V_NL | V_L: return launch_tp_v<V_NL | V_L>(p, lut_ws, s, row0, row1);
    case V_NL: return launch_tp_v<V_NL>(p, lut_ws, s, row0, row1);
    case V_L: return launch_tp_v<V_L>(p, lut_ws, s, row0, row1);
    case V_PROF: return launch_tp_v<V_PROF>(p, lut_ws, s, row0, row1);
  }
  return cudaErrorInvalidValue;
}

int tpacf_site_kind(int site) { return tpacf_site_kind_d(site); }

template <int KIND>
static cudaError_t launch_tp_fi_k(const TPFIParams& q, int nrep, cudaStream_t s) {
  const size_t smem = tp_smem_bytes(q.base.C, q.base.nb + 2);
  cudaError_t e = cudaFuncSetAttribute(tpacf_fi_kernel<KIND>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  dim3 grid((q.base.n + TP_CTA_PTS - 1) / TP_CTA_PTS, (1 + 2 * q.base.nr) * q.base.nC, nrep);
  TimedScope ts(HK_TPACF, 1, tp_pairs(q.base) * nrep, s);
  tpacf_fi_kernel<KIND><<<grid, TP_THREADS, smem, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

cudaError_t tpacf_replay_launch(int kind, const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
                                int nrep, const unsigned long long* golden, hk_outcome* records, int64_t first,
                                int64_t* counts, int64_t* site_counts, cudaStream_t s) {
  if (nrep <= 0) return cudaSuccess;
  if (3 * a.n_bins > TP_REPLAY_OUT) return cudaErrorInvalidValue;
  TPReplayParams q{};
  q.base = tp_params(a, R, ndet, nullptr, nullptr, nullptr);
  q.faults = faults;
  q.nrep = nrep;
  q.golden = golden; q.records = records; q.first = first; q.counts = counts; q.site_counts = site_counts;
  (void)kind;
  TimedScope ts(HK_TPACF, 2, (double)q.base.C * 2 * nrep, s);
  tpacf_replay_all_kernel<<<(nrep + 127) / 128, 128, 0, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

// lut_ws must hold a table built by tpacf_lut_build for a.edges (the campaign builds it once).
cudaError_t tpacf_fi_launch(int kind, const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults, int nrep,
                            unsigned long long* hist0, hk_control* cb0, void* lut_ws, bool real, cudaStream_t s) {
  TPFIParams q{};
  q.base = tp_params(a, R, ndet, nullptr, nullptr, lut_ws);
  q.faults = faults;
  q.hist0 = hist0;
  q.cb0 = cb0;
  q.hist_elems = (int64_t)(1 + 2 * a.n_rand) * (a.n_bins + 2);
  if (real) {
    const size_t smem = tp_smem_bytes(q.base.C, q.base.nb + 2);
    cudaError_t e = cudaFuncSetAttribute(tpacf_real_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    dim3 grid((a.n + TP_CTA_PTS - 1) / TP_CTA_PTS, (1 + 2 * a.n_rand) * q.base.nC, nrep);
    tpacf_real_kernel<<<grid, TP_THREADS, smem, s>>>(q, kind);
    count_launch();
    return cudaGetLastError();
  }
  switch (kind) {
#define K(k) case k: return launch_tp_fi_k<k>(q, nrep, s);
    K(TK_NL) K(TK_LIVE) K(TK_J) K(TK_X2) K(TK_Y2) K(TK_Z2) K(TK_DOT) K(TK_BIN) K(TK_HIDX) K(TK_ACC) K(TK_CNT)
#undef K
  }
  return cudaErrorInvalidValue;
}

}  // namespace hk
