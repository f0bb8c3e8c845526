// Fused MRI-Q + TPACF campaign replicas (replica mode, mixed campaigns; DESIGN "Fused replicas").
//
// One launch runs a batch of Rm MRI-Q replicas (Q-kernel site kinds: every site but PhiMag's) and
// a batch of Rt TPACF replicas.  Each CTA of the 1-D grid takes one role by its slot:
//   * slots [0, Rm): the faulted MRI-Q CTA of replica 0..Rm-1 (per-voxel FI program; the site kind
//     is switched at run time),
//   * slots [Rm, Rm + Rt): the faulted TPACF CTA of replica 0..Rt-1 (fast loop over the other
//     abstract threads, then the faulted one's FI program on its warp),
//   * the rest: the fast CTAs of both, interleaved in proportion to their counts — TPACF in
//     decreasing loop length (rank-major, replica-minor), MRI-Q replica-major.
// Per SM the block scheduler then keeps MRI-Q CTAs (bound by the MUFU sin/cos pipe) and TPACF
// CTAs (bound by issue and shared-memory wavefronts) resident side by side, which two separate
// kernels on two streams do not achieve (the second kernel's CTAs only start as the first one's
// grid drains).  Both roles run exactly the code of their own replica kernels (mriq.cu,
// tpacf.cu), so outcomes are identical to those of the separate launches.
#include "hk_common.cuh"
#include "hk_internal.h"
#include "mriq_dev.cuh"
#include "tpacf_dev.cuh"

#ifndef HK_MIX_MQ_VPT
#define HK_MIX_MQ_VPT 2  // voxels per CUDA thread of the MRI-Q role
#endif
#ifndef HK_MIX_GDIAG
#define HK_MIX_GDIAG true  // TPACF role: the diagonal as grouped loops (at 96 registers the grouped form
                           // cost the main loop its interleaved schedule; at 128 it is 1.4 % faster)
#endif
#ifndef HK_MIX_MINB
#define HK_MIX_MINB 4  // 4 CTAs per SM: 128 registers, no spills (5 CTAs: 96 registers with 12-16 B of spills,
                       // measured 3.7 % slower per mixed step; 6 CTAs: 80 registers, 7 % slower)
#endif

namespace hk {

constexpr int MIX_THREADS = 128;
constexpr int MIX_VPT = HK_MIX_MQ_VPT;
static_assert(MIX_THREADS == TP_THREADS, "the TPACF role needs TP_THREADS threads");

struct MixParams {
  MQFIParams m;    // m.nrep = Rm, m.ncta = MRI-Q CTAs per replica (MIX_THREADS threads each)
  TPFIParams t;
  int32_t rt;      // TPACF replicas
  int32_t tcta;    // TPACF CTAs per replica
  int64_t fm, ft;  // fast slots of each role
  // persistent variant: item counters of the two queues (zeroed before the launch) and the
  // number of the CTAs on each SM that start on the MRI-Q queue
  unsigned long long* queue;
  int32_t mq_per_sm, nsm;
  int32_t smem_used;  // bytes of dynamic shared memory the roles use (the persistent item follows)
};

template <bool EXACT, bool FT>
__device__ __forceinline__ void mix_mq_faulted(const MQParams& p, const FaultRec& f, int bxi) {
  switch (mriq_site_kind_d(f.site)) {
#define K_(k) case k: mq_faulted_cta<k, EXACT, FT, MIX_VPT>(p, f, bxi); break;
    K_(MK_NL) K_(MK_LIVE) K_(MK_K) K_(MK_KX) K_(MK_KY) K_(MK_KZ) K_(MK_PM) K_(MK_T1) K_(MK_T2) K_(MK_T) K_(MK_R) K_(MK_C)
    K_(MK_S) K_(MK_QR) K_(MK_QI) K_(MK_IT)
#undef K_
    default: break;  // PhiMag sites never reach the fused kernel (host)
  }
}

template <bool EXACT, bool FT>
__device__ __forceinline__ void mix_mq_slot(const MixParams& q, unsigned char* smem, int r, int64_t fast) {
  float4(*tile)[MQ_FI_TILE] = reinterpret_cast<float4(*)[MQ_FI_TILE]>(smem);
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + 2 * MQ_FI_TILE * sizeof(float4));
  const int64_t ncta = q.m.ncta, vpc = (int64_t)MIX_VPT * MIX_THREADS;
  const FaultRec f = q.m.faults[r];
  const int64_t fc = clamp_cta(f.thread / vpc, ncta);
  MQParams p = q.m.base;
  p.qr = q.m.out0 + (int64_t)r * q.m.stride;
  p.qi = p.qr + p.numX;
  p.cb = q.m.cb0 + r;
  if (fast < 0) {
    mix_mq_faulted<EXACT, FT>(p, f, (int)fc);
  } else {
    const int bxi = (int)(fast < fc ? fast : fast + 1);
    mriq_body<FT ? (V_NL | V_L) : 0, EXACT, true, MIX_VPT, MQ_FI_UNROLL, MQ_FI_TILE>(p, tile, bar, bxi);
  }
}

template <bool FT, bool LUT>
__device__ __forceinline__ void mix_tp_faulted(const TPFIParams& q, const TPSmem& S, const FaultRec& f, unsigned long long* hist,
                                               hk_control* cb, int h, int blk) {
  const int2 fi = tp_replica_fast<FT, LUT, HK_MIX_GDIAG>(q, S, f, hist, cb, h, blk, true);
  if (fi.x < 0) return;
  TPParams p = q.base;
  p.hist = hist;
  p.cb = cb;
  const int hd = (int)((uint32_t)h ^ p.z);
  const uint64_t hr = (uint64_t)(uintptr_t)hist;
  switch (tpacf_site_kind_d(f.site)) {
#define K_(k) case k: tpacf_fi_warp<k, FT, LUT>(p, S, f, h, fi.x, fi.y, hd, hr, cb); break;
    K_(TK_NL) K_(TK_LIVE) K_(TK_J) K_(TK_X2) K_(TK_Y2) K_(TK_Z2) K_(TK_DOT) K_(TK_BIN) K_(TK_HIDX) K_(TK_ACC) K_(TK_CNT)
#undef K_
    default: break;
  }
}

template <bool FT>
__device__ __forceinline__ void mix_tp_slot(const MixParams& q, unsigned char* smem, int r, int rank) {
  const TPParams& p0 = q.t.base;
  constexpr int CPTS = HK_TP_NP_FI * TP_THREADS;
  const FaultRec f = q.t.faults[r];
  const int fh = (int)(f.thread / p0.n), fb = (int)((f.thread % p0.n) / CPTS);
  int h, blk;
  if (rank < 0) {
    h = fh;
    blk = fb;
  } else {
    tp_cta_of_rank(rank, p0.nr, p0.nblk, &h, &blk);
    if (h == fh && blk == fb) return;  // ran in a faulted slot
  }
  const TPSmem S = tp_carve(smem, p0.nb + 2, HK_TP_NP_FI);
  tp_stage_tables(p0, S);
  cp_async_wait<0>();
  __syncthreads();
  unsigned long long* hist = q.t.hist0 + (int64_t)r * q.t.hist_elems;
  hk_control* cb = q.t.cb0 + r;
  const bool lut = *p0.lut_ok != 0 && tp_dsbase_ok();
  if (rank < 0) {
    if (lut) mix_tp_faulted<FT, true>(q.t, S, f, hist, cb, h, blk);
    else mix_tp_faulted<FT, false>(q.t, S, f, hist, cb, h, blk);
  } else {
    if (lut) tp_replica_fast<FT, true, HK_MIX_GDIAG>(q.t, S, f, hist, cb, h, blk, false);
    else tp_replica_fast<FT, false, HK_MIX_GDIAG>(q.t, S, f, hist, cb, h, blk, false);
  }
}

template <bool EXACT, bool FT>
__global__ void __launch_bounds__(MIX_THREADS, HK_MIX_MINB) mix_fi_kernel(const MixParams q) {
  const int64_t L = blockIdx.x;
  const int rm = q.m.nrep, rt = q.rt;
  if (L < rm) { mix_mq_slot<EXACT, FT>(q, hk_tp_dsmem, (int)L, -1); return; }
  if (L < rm + rt) { mix_tp_slot<FT>(q, hk_tp_dsmem, (int)(L - rm), -1); return; }
  const int64_t s = L - rm - rt, tot = q.fm + q.ft;
  const int64_t tb = s * q.ft / tot, tb1 = (s + 1) * q.ft / tot;  // TPACF slots among the first s (s + 1)
  if (tb1 > tb) {
    mix_tp_slot<FT>(q, hk_tp_dsmem, (int)(tb % rt), (int)(tb / rt));
  } else {
    const int64_t k = s - tb, per = q.m.ncta - 1;
    mix_mq_slot<EXACT, FT>(q, hk_tp_dsmem, (int)(k / per), k % per);
  }
}

// Persistent variant (HK_MIX_PERSIST=k, experiment): one wave of HK_MIX_MINB CTAs per SM; CTA c
// starts on the MRI-Q queue if c / nsm < k (the block scheduler fills the SMs breadth first, so
// every SM holds k MRI-Q and HK_MIX_MINB - k TPACF CTAs) and takes the other queue once its own
// is drained.  Items in the same order as the slots above (faulted CTAs first).
// Per-role item bodies of the persistent variant, not inlined: each gets its own register
// allocation (inlined into the item loop, both roles' state stayed live and spilled 1.6 KB).
template <bool EXACT, bool FT>
__device__ __noinline__ void mix_mq_item(const MixParams& q, long long it) {
  const int rm = q.m.nrep;
  if (it < rm) {
    mix_mq_slot<EXACT, FT>(q, hk_tp_dsmem, (int)it, -1);
  } else {
    const long long k = it - rm, per = q.m.ncta - 1;
    mix_mq_slot<EXACT, FT>(q, hk_tp_dsmem, (int)(k / per), k % per);
  }
}
template <bool FT>
__device__ __noinline__ void mix_tp_item(const MixParams& q, long long it) {
  const int rt = q.rt;
  if (it < rt) mix_tp_slot<FT>(q, hk_tp_dsmem, (int)it, -1);
  else mix_tp_slot<FT>(q, hk_tp_dsmem, (int)((it - rt) % rt), (int)((it - rt) / rt));
}

template <bool EXACT, bool FT>
__global__ void __launch_bounds__(MIX_THREADS, HK_MIX_MINB) mix_persist_kernel(const MixParams q) {
  // the claimed item lives past the roles' shared memory (no static shared memory: tp_dsbase_ok)
  long long* s_item = reinterpret_cast<long long*>(hk_tp_dsmem + q.smem_used);
  int* s_role = reinterpret_cast<int*>(s_item + 1);
  const long long nq[2] = {(long long)q.m.nrep + q.fm, (long long)q.rt + q.ft};
  int role = (int)(blockIdx.x / q.nsm) < q.mq_per_sm ? 0 : 1;
  for (;;) {
    __syncthreads();  // the previous item is done with shared memory
    if (threadIdx.x == 0) {
      long long it = -1;
      for (int tries = 0; tries < 2 && it < 0; ++tries) {
        const long long v = (long long)atomicAdd(q.queue + role, 1ull);
        if (v < nq[role]) it = v;
        else role ^= 1;
      }
      *s_item = it;
      *s_role = role;
      if (it >= 0 && role == 0) fence_proxy_async();  // earlier generic writes before the bulk copies
    }
    __syncthreads();
    const long long it = *s_item;
    role = *s_role;
    if (it < 0) return;
    if (role == 0) {
      mix_mq_item<EXACT, FT>(q, it);
      __syncthreads();
      if (threadIdx.x == 0) {  // the k-space barriers are re-initialised by the next MRI-Q item
        uint64_t* bar = reinterpret_cast<uint64_t*>(hk_tp_dsmem + 2 * MQ_FI_TILE * sizeof(float4));
        asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(&bar[0])) : "memory");
        asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(&bar[1])) : "memory");
      }
    } else {
      mix_tp_item<FT>(q, it);
    }
  }
}

size_t mix_smem_bytes(const hk_tpacf_args& t) {
  return std::max(tp_smem_bytes(t.n_bins + 2, HK_TP_NP_FI), 2 * MQ_FI_TILE * sizeof(float4) + 16);
}

template <bool EXACT, bool FT>
static cudaError_t launch_mix(const MixParams& q, size_t smem, int64_t grid, cudaStream_t s) {
  if (q.queue) {
    cudaError_t e = cudaFuncSetAttribute(mix_persist_kernel<EXACT, FT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem + 16);
    if (e != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(q.queue, 0, 2 * sizeof(unsigned long long), s)) != cudaSuccess) return e;
    mix_persist_kernel<EXACT, FT><<<(unsigned)(q.nsm * HK_MIX_MINB), MIX_THREADS, smem + 16, s>>>(q);
    count_launch();
    return cudaGetLastError();
  }
  cudaError_t e = cudaFuncSetAttribute(mix_fi_kernel<EXACT, FT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  mix_fi_kernel<EXACT, FT><<<(unsigned)grid, MIX_THREADS, smem, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

bool mix_supported(const hk_mriq_args& m, const hk_tpacf_args& t) {
  const int64_t vpc = (int64_t)MIX_VPT * MIX_THREADS;
  return (m.n_vox + vpc - 1) / vpc >= 2 && t.n > 0 && t.n_bins + 2 <= 32;
}

cudaError_t mix_fi_launch(bool ft, const hk_mriq_args& ma, const DevRanges& mR, int mndet, const FaultRec* mfaults, int rm,
                          float* mout0, int64_t mstride, hk_control* mcb0, const hk_tpacf_args& ta, const DevRanges& tR, int tndet,
                          const FaultRec* tfaults, int rt, unsigned long long* thist0, hk_control* tcb0, void* tlut, cudaStream_t s) {
  if (rm <= 0 || rt <= 0 || !mix_supported(ma, ta)) return cudaErrorInvalidValue;
  MixParams q{};
  q.m = mriq_fi_params(ma, mR, mndet, mfaults, rm, mout0, mstride, mcb0, MIX_THREADS, MIX_VPT);
  q.t = tpacf_fi_params(ta, tR, tndet, tfaults, thist0, tcb0, tlut);
  q.rt = rt;
  q.tcta = (1 + 2 * ta.n_rand) * q.t.base.nblk;
  q.fm = (int64_t)rm * (q.m.ncta - 1);
  q.ft = (int64_t)rt * q.tcta;
  const int64_t grid = rm + rt + q.fm + q.ft;
  const char* pv = getenv("HK_MIX_PERSIST");  // read per launch (experiments, tests)
  const int persist = pv ? atoi(pv) : 0;
  if (persist > 0) {
    static unsigned long long* queue = nullptr;  // experiment only: one per process
    if (!queue && cudaMalloc((void**)&queue, 2 * sizeof(unsigned long long)) != cudaSuccess) return cudaErrorMemoryAllocation;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    q.queue = queue;
    q.mq_per_sm = std::min(persist, HK_MIX_MINB);
    q.nsm = sms;
  }
  const size_t smem = mix_smem_bytes(ta);
  q.smem_used = (int32_t)((smem + 15) / 16 * 16);
  // timing class 3: the same launches under both benchmarks, each with its own work
  const double n = ta.n;
  TimedScope tt(HK_TPACF, 3, ((1 + ta.n_rand) * n * (n - 1) / 2 + ta.n_rand * n * n) * rt, s);
  TimedScope tm(HK_MRIQ, 3, (double)ma.n_vox * (double)ma.n_k * rm, s);
  if (ma.exact) return ft ? launch_mix<true, true>(q, smem, grid, s) : launch_mix<true, false>(q, smem, grid, s);
  return ft ? launch_mix<false, true>(q, smem, grid, s) : launch_mix<false, false>(q, smem, grid, s);
}

}  // namespace hk
