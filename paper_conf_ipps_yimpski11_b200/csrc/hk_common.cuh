// hk_common.cuh — device building blocks shared by the three HAUBERK-instrumented kernels.
//
// Detector helpers follow PAPER.md §V (HAUBERK-NL L986-1053, HAUBERK-L L1275-1313, L1405-1429);
// the injector helpers follow §VII (L2186-2272) with the crash/hang models of DESIGN.md R16/R17.
// Everything here is sm_100a device code; nothing is shared with oracle/.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/hauberk.h"

namespace hk {

// ---------------------------------------------------------------------------------------------
// Variant flags (template parameter V).  BASE = 0; FT = NL | L; PROFILE emits acc/it samples.
// ---------------------------------------------------------------------------------------------
enum : int { V_NL = 1, V_L = 2, V_PROF = 4 };
enum : uint32_t { AL_DUP = 1, AL_CHK = 2, AL_RANGE = 4, AL_COUNT = 8 };
enum : uint32_t { FL_CRASH = 1, FL_HANG = 2 };

constexpr uint64_t VBASE = 0x00007F0000000000ull;  // R16 canonical virtual base of pointer params

// Loop-detector ranges, alpha already applied on the host (R11).  Passed by value (param space).
struct DevRanges {
  int32_t n_det;
  int32_t n[8];
  float lo[8][3];
  float hi[8][3];
};

// One replica's injection, decoded on the host (R14/R15).  `sub` = per-kind selector
// (CP unrolled lane j, or the @live variable id); inst = -1 never fires.
struct FaultRec {
  int64_t index;   // campaign index n
  int64_t thread;  // abstract thread
  int64_t inst;    // dynamic instance
  uint64_t mask;   // XOR mask (32- or 64-bit site)
  int32_t site;
  int32_t sub;
  int32_t real;    // 1: unguarded run for the guardian (DESIGN R25); 0: crash / hang models R16 / R17
  int32_t hang;    // R17 watchdog factor T (<= 0: the paper's 10)
};

// Site catalogue of one benchmark for the device decode (DESIGN R14): enabled sites, per-site
// class/width/kind/sub, thread and instance counts, and the TPACF trip prefix sums.
struct DevCatalog {
  int32_t nen, pad;
  int32_t en[64];
  uint8_t is_nl[64], width[64], kind[64], sub[64];
  int64_t nthr, nk, uniform_trips, total_trips;
  const int64_t* prefix;
};

__device__ __forceinline__ uint32_t fb(float f) { return __float_as_uint(f); }
__device__ __forceinline__ float bf(uint32_t u) { return __uint_as_float(u); }
__device__ __forceinline__ uint32_t lohi(uint64_t p) { return (uint32_t)p ^ (uint32_t)(p >> 32); }
template <class T>
__device__ __forceinline__ uint32_t lohi_ptr(const T* p) { return lohi((uint64_t)(uintptr_t)p); }

// Runtime-opaque identity for duplicated inputs / second checksum XORs: the compiler
// cannot prove `z == 0`, so it can neither CSE a duplicate nor cancel the two XORs of a value.
__device__ __forceinline__ int32_t opq(int32_t v, uint32_t z) { return (int32_t)((uint32_t)v + z); }
__device__ __forceinline__ uint32_t opqf(float v, uint32_t z) { return fb(v) + z; }

// Counter increment the compiler may not strength-reduce out of the loop (it++ of L1286-1300).
__device__ __forceinline__ int32_t count_inc(int32_t it, int32_t one) {
  asm volatile("add.s32 %0, %0, %1;" : "+r"(it) : "r"(one));
  return it;
}

// R8 ordinal of a binary32 value (fits int32: |ord| <= 0x7fffffff).
__device__ __forceinline__ int32_t ordf(float x) {
  uint32_t b = fb(x);
  return (b & 0x80000000u) ? -(int32_t)(b & 0x7fffffffu) : (int32_t)b;
}
__device__ __forceinline__ uint32_t ord_dist(float a, float b) {
  int64_t d = (int64_t)ordf(a) - (int64_t)ordf(b);
  if (d < 0) d = -d;
  return d > 0x7fffffff ? 0x7fffffffu : (uint32_t)d;
}

// HauberkCheckRange (L1302-1313): v in any profiled range?  NaN -> out of range (R10).
template <bool MARGIN>
__device__ __forceinline__ bool in_range(const DevRanges& R, int d, float v, uint32_t* margin, float* gap = nullptr) {
  bool in = false;
#pragma unroll
  for (int r = 0; r < 3; ++r) {
    if (r < R.n[d]) {
      const float lo = R.lo[d][r], hi = R.hi[d][r];
      in |= (lo <= v) & (v <= hi);
      if (MARGIN && v == v) {
        uint32_t a = ord_dist(v, lo), b = ord_dist(v, hi);
        *margin = min(*margin, min(a, b));
        *gap = fminf(*gap, fminf(fabsf(__fsub_rn(v, lo)), fabsf(__fsub_rn(v, hi))));  // R22(a) absolute gap
      }
    }
  }
  return in;
}

// Record an outlier (A11, L1309-1313): the host extends ranges from these ordinals.
__device__ __forceinline__ void record_outlier(hk_control* cb, int d, float v) {
  if (v == v) {
    atomicMin(&cb->outlier_min_ord[d], ordf(v));
    atomicMax(&cb->outlier_max_ord[d], ordf(v));
  }
}

// Deferred reporting (L751-762): fold the per-thread alarm bits of a warp with one vote and at
// most one set of atomics per warp.
__device__ __forceinline__ void fold_alarm(hk_control* cb, uint32_t alarm, uint32_t tid) {
  const unsigned act = __activemask();
  const unsigned who = __ballot_sync(act, alarm != 0u);
  if (who) {
    const uint32_t all = __reduce_or_sync(act, alarm);
    const uint32_t first = __reduce_min_sync(act, alarm ? tid : 0xffffffffu);
    unsigned lane;
    asm("mov.u32 %0, %%laneid;" : "=r"(lane));
    if ((unsigned)(__ffs(who) - 1) == lane) {
      atomicOr(&cb->alarm, all);
      atomicAdd(&cb->n_alarm_warps, 1u);
      atomicMin(&cb->first_thread, first);
    }
  }
}

// ---------------------------------------------------------------------------------------------
// Transcendentals (R20).  FAST = MUFU with .ftz; EXACT = fixed binary32 sequences.
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ float rsqrt_mufu(float x) {
  float y;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float sin_mufu(float x) {
  float y;
  asm("sin.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float cos_mufu(float x) {
  float y;
  asm("cos.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float rsqrt_exact(float x) {
  float y = bf(0x5F375A86u - (fb(x) >> 1));
  const float hx = __fmul_rn(0.5f, x);
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    float t = __fmul_rn(hx, y);
    t = __fmaf_rn(-t, y, 1.5f);
    y = __fmul_rn(y, t);
  }
  return y;
}
// (float)(+-1/n!) computed at compile time in double, rounded once to binary32.
constexpr double fact_d(int n) { return n <= 1 ? 1.0 : n * fact_d(n - 1); }
constexpr float sin_c(int k) { return (float)((k & 1) ? -1.0 / fact_d(2 * k + 1) : 1.0 / fact_d(2 * k + 1)); }
constexpr float cos_c(int k) { return (float)((k & 1) ? -1.0 / fact_d(2 * k) : 1.0 / fact_d(2 * k)); }
template <int K> struct SinC { static constexpr float v = sin_c(K); };
template <int K> struct CosC { static constexpr float v = cos_c(K); };
__device__ __forceinline__ float sin_exact(float a) {
  const float s2 = __fmul_rn(a, a);
  float p = SinC<9>::v;
  p = __fmaf_rn(p, s2, SinC<8>::v); p = __fmaf_rn(p, s2, SinC<7>::v); p = __fmaf_rn(p, s2, SinC<6>::v);
  p = __fmaf_rn(p, s2, SinC<5>::v); p = __fmaf_rn(p, s2, SinC<4>::v); p = __fmaf_rn(p, s2, SinC<3>::v);
  p = __fmaf_rn(p, s2, SinC<2>::v); p = __fmaf_rn(p, s2, SinC<1>::v); p = __fmaf_rn(p, s2, SinC<0>::v);
  return __fmul_rn(a, p);
}
__device__ __forceinline__ float cos_exact(float a) {
  const float s2 = __fmul_rn(a, a);
  float q = CosC<10>::v;
  q = __fmaf_rn(q, s2, CosC<9>::v); q = __fmaf_rn(q, s2, CosC<8>::v); q = __fmaf_rn(q, s2, CosC<7>::v);
  q = __fmaf_rn(q, s2, CosC<6>::v); q = __fmaf_rn(q, s2, CosC<5>::v); q = __fmaf_rn(q, s2, CosC<4>::v);
  q = __fmaf_rn(q, s2, CosC<3>::v); q = __fmaf_rn(q, s2, CosC<2>::v); q = __fmaf_rn(q, s2, CosC<1>::v);
  q = __fmaf_rn(q, s2, CosC<0>::v);
  return q;
}
template <bool EXACT> __device__ __forceinline__ float hk_rsqrt(float x) { return EXACT ? rsqrt_exact(x) : rsqrt_mufu(x); }
template <bool EXACT> __device__ __forceinline__ float hk_sin(float x) { return EXACT ? sin_exact(x) : sin_mufu(x); }
template <bool EXACT> __device__ __forceinline__ float hk_cos(float x) { return EXACT ? cos_exact(x) : cos_mufu(x); }

// ---------------------------------------------------------------------------------------------
// Injector helpers (FI builds only).
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ int32_t flip_i(int32_t v, bool now, uint64_t mask) { return now ? (int32_t)((uint32_t)v ^ (uint32_t)mask) : v; }
__device__ __forceinline__ float flip_f(float v, bool now, uint64_t mask) { return now ? bf(fb(v) ^ (uint32_t)mask) : v; }
__device__ __forceinline__ uint64_t flip_p(uint64_t v, bool now, uint64_t mask) { return now ? v ^ mask : v; }

// R16: element access through a modelled pointer register `preg` whose true value is `preal`.
__device__ __forceinline__ bool guard(uint64_t preg, uint64_t preal, int32_t idx, int64_t esz, int64_t n, int64_t* e) {
  const uint64_t m = preg ^ preal;
  const int64_t delta = (int64_t)((VBASE ^ m) - VBASE);
  if (delta % esz != 0) return false;
  const int64_t ei = (int64_t)idx + delta / esz;
  if (ei < 0 || ei >= n) return false;
  *e = ei;
  return true;
}

// Element address through a modelled pointer register (R16), or — in the guardian's unguarded runs
// (R25) — the corrupted address itself, dereferenced as the uninstrumented program would: the
// hardware decides (illegal or misaligned address kills the context, the guardian sees the crash).
// nullptr = modelled crash.
// Both are `true base + idx * size + delta`: delta = the modelled displacement (VBASE ^ m) - VBASE
// (R16, checked against the buffer) or the real one, preg - preal (unchecked).  false = modelled crash.
template <class T>
__device__ __forceinline__ bool fi_at(bool real, uint64_t preg, uint64_t preal, int32_t idx, int64_t n, T** out) {
  constexpr int64_t esz = (int64_t)sizeof(T);
  const uint64_t m = preg ^ preal;
  const int64_t delta = real ? (int64_t)(preg - preal) : (int64_t)((VBASE ^ m) - VBASE);
  const int64_t off = (int64_t)idx * esz + delta;
  *out = reinterpret_cast<T*>(preal + (uint64_t)off);
  const bool in_buf = ((delta & (esz - 1)) == 0) & (off >= 0) & (off < n * esz);
  return in_buf | real;  // non-short-circuit: one predicate op, no branch around the check
}
// Global-space accesses through fi_at results (the pointer came from an integer, so the compiler
// cannot infer the space; the instrumented program's buffers are global, as are the kernel's).
__device__ __forceinline__ void red_add(float* p, float v) {
  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(p), "f"(v) : "memory");
}
__device__ __forceinline__ void red_add(unsigned long long* p, unsigned long long v) {
  asm volatile("red.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// Launch order of the FI&FT replica kernels.  CTAs are dispatched in (roughly) linear block order:
// the first nrep of them run the faulted CTA of replica 0..nrep-1, whose per-thread FI program is
// several times slower than a fast-path CTA — started first, it overlaps the fast CTAs instead of
// trailing the launch — and the others follow replica by replica in CTA order.  fault_cta(r) in
// [0, ncta) is the CTA that holds replica r's faulted thread.  Returns true for a faulted CTA.
template <class F>
__device__ __forceinline__ bool fi_order(int64_t L, int64_t ncta, int nrep, F fault_cta, int* r, int64_t* cta) {
  if (L < nrep) {
    *r = (int)L;
    *cta = fault_cta((int)L);
    return true;
  }
  const int64_t L2 = L - nrep;
  const int rr = (int)(L2 / (ncta - 1));
  const int64_t k = L2 - (int64_t)rr * (ncta - 1), fc = fault_cta(rr);
  *r = rr;
  *cta = k < fc ? k : k + 1;
  return false;
}
__device__ __forceinline__ int64_t clamp_cta(int64_t c, int64_t ncta) { return c < 0 ? 0 : (c >= ncta ? ncta - 1 : c); }

// R17 watchdog limit T x max(golden trips, 1) (T = 10 unless the campaign sets hang_factor);
// none in unguarded runs (the guardian's timeout observes the hang).
template <bool REAL>
__device__ __forceinline__ int64_t fi_limit(int64_t golden_trips, int32_t hang) {
  const int64_t T = hang > 0 ? hang : 10;
  return REAL ? INT64_MAX : T * (golden_trips > 1 ? golden_trips : 1);
}

__device__ __forceinline__ unsigned lane_id() {
  unsigned l;
  asm("mov.u32 %0, %%laneid;" : "=r"(l));
  return l;
}

// ---------------------------------------------------------------------------------------------
// 1-D bulk async copy (TMA engine, cp.async.bulk) global -> shared with an mbarrier.
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "HK_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra HK_WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// Where a per-thread FI program's effects go.  Replica: atomic adds into the replica's grid and
// the warp-folded control block.  Replay: the (at most U) writes and the thread's verdict bits
// stay in registers for the per-injection classification.
struct ReplicaSinkF {
  float* out[2];
  hk_control* cb;
  __device__ __forceinline__ void store(int buf, int64_t e, float v) { atomicAdd(out[buf] + e, v); }
  __device__ __forceinline__ void store_p(int, float* ptr, const float*, float v) { red_add(ptr, v); }
  __device__ __forceinline__ void outlier(int d, float v) { record_outlier(cb, d, v); }
  __device__ __forceinline__ void finish(bool mine, uint32_t alarm, uint32_t fail, uint32_t margin, float gap,
                                         uint32_t domain, bool applied, uint32_t tid) {
    if (fail) atomicOr(&cb->fail, fail);
    if (mine) {
      cb->fault_applied = applied ? 1u : 0u;
      cb->check_margin = margin;
      cb->check_gap = gap;
      cb->domain = domain;
    }
    fold_alarm(cb, alarm, tid);
  }
};
template <int MAXW>
struct ReplaySinkF {
  int n = 0;
  int buf[MAXW];
  int64_t idx[MAXW];
  float val[MAXW];
  uint32_t alarm = 0, fail = 0, margin = 0xffffffffu, domain = 0;
  float gap = __builtin_huge_valf();
  __device__ __forceinline__ void store(int b, int64_t e, float v) {
    if (n < MAXW) { buf[n] = b; idx[n] = e; val[n] = v; ++n; }
  }
  __device__ __forceinline__ void store_p(int b, float* ptr, const float* base, float v) { store(b, ptr - base, v); }
  __device__ __forceinline__ void outlier(int, float) {}
  __device__ __forceinline__ void finish(bool, uint32_t a, uint32_t f, uint32_t m, float g, uint32_t d, bool, uint32_t) {
    alarm = a; fail = f; margin = m; gap = g; domain = d;
  }
};

// Output-correctness rule shared by the classify epilogue and the replay kernels (R5/R6).
__device__ __forceinline__ void fp_judge(float v, float g, float M, bool* wrong, float* worst) {
  const float err = fabsf(__fsub_rn(v, g));
  const float tol = fmaxf(__fmul_rn(1e-4f, M), __fmul_rn(0.002f, fabsf(g)));
  *wrong |= !(err <= tol);
  float q = __fdiv_rn(err, tol);
  if (q != q) q = __int_as_float(0x7f800000);
  *worst = fmaxf(*worst, q);
}

__device__ __forceinline__ void emit_outcome(int bench, const FaultRec& f, bool wrong, uint32_t alarm, uint32_t fail,
                                             uint32_t domain, uint32_t margin, float gap, float worst, hk_outcome* records,
                                             int64_t first, int64_t* counts, int64_t* site_counts) {
  const int32_t cls = fail ? HK_FAILURE : (!wrong ? (alarm ? HK_DETECTED_MASKED : HK_MASKED) : (alarm ? HK_DETECTED : HK_UNDETECTED));
  if (records) {
    hk_outcome o;
    o.index = f.index; o.bench = bench; o.site = f.site; o.thread = f.thread; o.inst = f.inst; o.mask = f.mask;
    o.cls = cls; o.alarm = alarm; o.fail = fail; o.domain = domain; o.margin = margin; o.worst = worst;
    o.gap = gap; o.pad2 = 0;
    records[f.index - first] = o;
  }
  atomicAdd(reinterpret_cast<unsigned long long*>(counts + bench * 5 + cls), 1ull);
  if (site_counts && f.site < 64)
    atomicAdd(reinterpret_cast<unsigned long long*>(site_counts + ((int64_t)bench * 64 + f.site) * 5 + cls), 1ull);
}

// Initial value of a control block (reset by hk_control_init / the classify epilogue).
__device__ __forceinline__ void control_reset(hk_control* cb, int lane) {
  // lane < 24 writes one 32-bit word each
  uint32_t* w = reinterpret_cast<uint32_t*>(cb);
  if (lane < 24) {
    uint32_t v = 0;
    if (lane == 3) v = 0xffffffffu;                    // first_thread
    else if (lane >= 4 && lane < 12) v = 0x7fffffffu;  // outlier_min_ord
    else if (lane >= 12 && lane < 20) v = 0x80000000u; // outlier_max_ord
    else if (lane == 21) v = 0xffffffffu;              // check_margin
    else if (lane == 23) v = 0x7f800000u;              // check_gap = +inf
    w[lane] = v;
  }
}

}  // namespace hk
