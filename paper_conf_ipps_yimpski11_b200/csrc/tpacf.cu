// tpacf.cu — two-point angular correlation histograms (K3) with HAUBERK detectors, sm_100a.
//
// Abstract program: DESIGN.md §3.4 / SURVEY §8.1.3 (benchmark: Parboil TPACF; the paper cites its
// 1 % output rule, L80-84, its shared-memory footprint, L2428-2431, and its retry-until-written
// histogram loop that could hang, L2643-2649 — not reproduced: B200 shared-memory atomics need no
// retry).  One abstract thread per (histogram h, point i) loops over EVERY partner j in [jb, N);
// the loop detector is acc += bin, cnt++ (the "two addition instructions", L679-680), checked once
// after the whole loop.  How the kernels tile that loop is not part of the program:
//  * acc, cnt and the histogram are integer sums, so any split of a thread's partner range into
//    pieces, added exactly, gives the same values as the one sequential loop;
//  * the single run (tpacf_kernel) cuts each point block's partner range into pieces of equal
//    pair counts that fill one wave of CTAs, adds the per-piece (acc, cnt) partials with global
//    atomics, and the last piece of a point block (a per-(h, block) completion counter) runs
//    CheckEqual / CheckRange for its points;
//  * the campaign replicas (tpacf_fi_kernel) give each CTA whole loops (all partners of its
//    points, streamed through a two-stage shared-memory ring), and the faulted abstract thread runs
//    its sequential per-thread FI program after the CTA's fast loop.
// B200 shape: 128 threads, NP abstract threads per CUDA thread (points i0 + t + 128k) sharing
// every partner load (broadcast LDS.128); bin = byte table of 4 * bmin indexed by the top 11 bits
// of u = fl(1 - dot), then one edge load and one compare; lane-private shared histograms
// [warp][word][bin][lane] (bank = lane) with two points packed in the 16-bit halves of a counter,
// one ATOMS per pair.  Shared-memory wavefronts bind this loop (ncu: LDS.64 and LDS.128 cost two
// wavefronts each even as broadcasts, 32-bit LDS / ATOMS one), so the table stays byte-wide and
// NP = 4 amortises the partner loads over four points.
#include <algorithm>
#include <vector>

#include "tpacf_dev.cuh"

namespace hk {

// One thread per bucket q.  Buckets in u-value order: ord(q) = 1024 + q for u >= +0 (q < 1024),
// 2047 - q for u <= -0 (bit order reversed).  Because fl(1 - .) is monotone non-increasing, every
// dot of bucket q is below edge e iff bucket(fl(1 - e)) comes before q (then dot < e for all of
// them), and above it iff that bucket comes after q; so bmin(q) = bin(dmax(q)) is the number of
// edges whose u-bucket precedes q, and bin = bmin + (dot < edge[bmin]) holds exactly when no two
// edges share a bucket (checked; the edges are strictly decreasing, so their bucket ordinals are
// non-decreasing).  Exponent-0xff buckets: +inf u (dot = -inf) follows the same rule (every finite
// edge precedes it); NaN u (dot NaN) has bin 0; -inf u (dot = +inf) precedes every bucket.
// Block 0 also writes the validity flag, and the grid zeroes up to two word ranges for the run that
// follows (its histogram and its partial-sum workspace: no separate memsets).
__device__ __forceinline__ int tp_bucket_ord(uint32_t q) { return q < 1024u ? 1024 + (int)q : 2047 - (int)q; }
__global__ void __launch_bounds__(256) tpacf_lut_kernel(const float* __restrict__ edges, int nb, uint8_t* __restrict__ lut, int* ok,
                                                         uint32_t* z0, int64_t n0, uint32_t* z1, int64_t n1) {
  __shared__ int eo[32];
  __shared__ int bad;
  const int q = blockIdx.x * blockDim.x + threadIdx.x;
  for (int64_t k = q; k < n0; k += TP_LUT) z0[k] = 0u;
  for (int64_t k = q; k < n1; k += TP_LUT) z1[k] = 0u;
  if (threadIdx.x == 0) bad = 0;
  __syncthreads();
  if (threadIdx.x <= nb && threadIdx.x < 32) {
    const float e = edges[threadIdx.x];
    const float u = __fsub_rn(1.0f, e);
    eo[threadIdx.x] = tp_bucket_ord(fb(u) >> 21);
    if (u != u) atomicExch(&bad, 1);  // a NaN edge: no table
  }
  __syncthreads();
  if (threadIdx.x < nb && threadIdx.x < 31 && eo[threadIdx.x] >= eo[threadIdx.x + 1]) atomicExch(&bad, 1);
  __syncthreads();
  if (blockIdx.x == 0 && threadIdx.x == 0) *ok = bad ? 0 : 1;
  if (q >= TP_LUT) return;
  const uint32_t uq = (uint32_t)q;
  const uint32_t ex = (uq >> 2) & 0xffu;
  int bmin = 0;
  if (ex == 0xffu && (uq & 0x400u) == 0 && (uq & 0x3u) != 0) {
    bmin = 0;  // positive NaN buckets (0x7fa00000 .. 0x7fffffff): dot NaN -> bin 0
  } else if (ex == 0xffu && (uq & 0x400u) != 0) {
    bmin = 0;  // -inf / negative-NaN buckets: dot = +inf or NaN -> bin 0
  } else {
    const int o = tp_bucket_ord(uq);
    for (int k = 0; k <= nb && k < 32; ++k) bmin += eo[k] < o ? 1 : 0;
  }
  lut[q] = (uint8_t)(4 * bmin);  // byte offset of E[bmin] (E padded with -inf beyond nb)
}
#ifdef HK_TP_SR_TRACE
__device__ unsigned long long g_tp_trace[4096][4];  // debug builds: (smid, start ns, end ns, piece)
extern "C" __attribute__((visibility("default"))) int hk_debug_trace(void* out) {
  return (int)cudaMemcpyFromSymbol(out, g_tp_trace, sizeof(g_tp_trace));
}
#endif
template <int V>
__global__ void __launch_bounds__(TP_SR_T, V == 0 ? HK_TP_MINB_SR : (V == V_NL ? HK_TP_MINB_SR_NL : HK_TP_MINB_SR_FT)) tpacf_kernel(const TPParams p, const TPSR q) {
#ifdef HK_TP_SR_TRACE
  unsigned long long t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
#endif
  // the piece descriptor lives past the carve (no static shared memory: tp_dsbase_ok)
  const TPSmem S = tp_carve(hk_tp_dsmem, p.nb + 2, HK_TP_NP_SR, TP_SR_T);
  int3& s_pc = *reinterpret_cast<int3*>(hk_tp_dsmem + tp_smem_bytes(p.nb + 2, HK_TP_NP_SR, TP_SR_T));
  tp_stage_tables(p, S);
  if (threadIdx.x < 32) {
    const int3 pc = tp_sr_locate(p, q, (int)blockIdx.x);
    if (threadIdx.x == 0) s_pc = pc;
  }
  cp_async_wait<0>();
  __syncthreads();
  const int3 pc = s_pc;
  if (pc.x < 0) return;
  if (*p.lut_ok && tp_dsbase_ok()) tp_sr_piece<V, true>(p, S, q, pc);
  else tp_sr_piece<V, false>(p, S, q, pc);
#ifdef HK_TP_SR_TRACE
  __syncthreads();
  if (threadIdx.x == 0 && blockIdx.x < 4096) {
    unsigned long long t1;
    uint32_t sm;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    g_tp_trace[blockIdx.x][0] = sm;
    g_tp_trace[blockIdx.x][1] = t0;
    g_tp_trace[blockIdx.x][2] = t1;
    g_tp_trace[blockIdx.x][3] = ((unsigned long long)pc.x << 32) | ((unsigned)pc.y << 16) | (unsigned)pc.z;
  }
#endif
}

// ============================================================================================
template <int KIND, bool FT>
__global__ void __launch_bounds__(TP_THREADS, HK_TP_MINB) tpacf_fi_kernel(const TPFIParams q) {
  const TPParams& p0 = q.base;
  constexpr int CPTS = HK_TP_NP_FI * TP_THREADS;
  const TPSmem S = tp_carve(hk_tp_dsmem, p0.nb + 2, HK_TP_NP_FI);
  // launch slot (x = replica, y = 0: its faulted CTA, y = 1 + rank: CTA of that rank)
  const int r = (int)blockIdx.x;
  int h, blk;
  bool faulted;
  if (blockIdx.y == 0) {
    const int64_t g = q.faults[r].thread;
    h = (int)(g / p0.n);
    blk = (int)((g % p0.n) / CPTS);
    faulted = true;
  } else {
    tp_cta_of_rank((int)blockIdx.y - 1, p0.nr, p0.nblk, &h, &blk);
    const int64_t g = q.faults[r].thread;
    if (h == (int)(g / p0.n) && blk == (int)((g % p0.n) / CPTS)) return;  // ran in the first slots
    faulted = false;
  }
  const FaultRec f = q.faults[r];
  tp_stage_tables(p0, S);
  cp_async_wait<0>();
  __syncthreads();
  unsigned long long* hist = q.hist0 + (int64_t)r * q.hist_elems;
  hk_control* cb = q.cb0 + r;
  if (*p0.lut_ok && tp_dsbase_ok()) tp_replica_cta<KIND, FT, true>(q, S, f, hist, cb, h, blk, faulted);
  else tp_replica_cta<KIND, FT, false>(q, S, f, hist, cb, h, blk, faulted);
}

// Unguarded replicas for the guardian (campaign mode 2, DESIGN R25): one CUDA thread per abstract
// thread runs the per-thread program with REAL = true; the site kind is a runtime switch (one
// injection per launch; slow and simple — a guardian child runs a handful of injections).
__global__ void __launch_bounds__(128) tpacf_real_kernel(const TPFIParams q, int kind) {
  __shared__ float Es[32];
  const TPParams& p = q.base;
  if (threadIdx.x < 32) Es[threadIdx.x] = threadIdx.x <= p.nb ? p.edges[threadIdx.x] : __int_as_float(0xff800000);
  __syncthreads();
  const int r = blockIdx.y;
  const FaultRec f = q.faults[r];
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g >= (int64_t)(1 + 2 * p.nr) * p.n) return;
  unsigned long long* hist = q.hist0 + (int64_t)r * q.hist_elems;
  TPReplicaSink K{q.cb0 + r};
  const int32_t h = (int32_t)(g / p.n), ii = (int32_t)(g % p.n);
  switch (kind) {
#define K_(k) case k: tpacf_fi_program<k, true, true>(p, Es, f, h, ii, opq(ii, p.z), (int32_t)((uint32_t)h ^ p.z), g == f.thread, (uint64_t)(uintptr_t)hist, K); break;
    K_(TK_NL) K_(TK_LIVE) K_(TK_J) K_(TK_X2) K_(TK_Y2) K_(TK_Z2) K_(TK_DOT) K_(TK_BIN) K_(TK_HIDX) K_(TK_ACC) K_(TK_CNT)
#undef K_
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

template <int KIND, bool FT>
__device__ __forceinline__ void tpacf_replay_one(const TPReplayParams& q, const FaultRec& f, const float* Es) {
  const TPParams& p = q.base;
  const int32_t h = (int32_t)(f.thread / p.n), ii = (int32_t)(f.thread % p.n);
  int32_t delta[TP_REPLAY_OUT];
  for (int o = 0; o < 3 * p.nb; ++o) delta[o] = 0;
  const uint64_t hist_real = (uint64_t)(uintptr_t)q.golden;
  TPReplaySink twin{p.nr, p.nb, p.nb + 2, -1, delta};
  tpacf_fi_program<KIND, FT>(p, Es, f, h, ii, opq(ii, p.z), (int32_t)((uint32_t)h ^ p.z), false, hist_real, twin);
  TPReplaySink K{p.nr, p.nb, p.nb + 2, +1, delta};
  tpacf_fi_program<KIND, FT>(p, Es, f, h, ii, opq(ii, p.z), (int32_t)((uint32_t)h ^ p.z), true, hist_real, K);
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

template <bool FT>
__global__ void __launch_bounds__(128) tpacf_replay_all_kernel(const TPReplayParams q) {
  __shared__ float Es[32];
  const TPParams& p = q.base;
  if (threadIdx.x < 32) Es[threadIdx.x] = threadIdx.x <= p.nb ? p.edges[threadIdx.x] : __int_as_float(0xff800000);
  __syncthreads();
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= q.nrep) return;
  const FaultRec f = q.faults[r];
  switch (tpacf_site_kind_d(f.site)) {
#define K_(k) case k: tpacf_replay_one<k, FT>(q, f, Es); break;
    K_(TK_NL) K_(TK_LIVE) K_(TK_J) K_(TK_X2) K_(TK_Y2) K_(TK_Z2) K_(TK_DOT) K_(TK_BIN) K_(TK_HIDX) K_(TK_ACC) K_(TK_CNT)
#undef K_
    default: break;
  }
}

// ============================================================================================
// Host launchers
// ============================================================================================
static int tp_nblk(int n, int np, int T = TP_THREADS) { return (n + np * T - 1) / (np * T); }

static TPParams tp_params(const hk_tpacf_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                          void* ws) {
  TPParams p{};
  p.pts = a.pts;
  p.edges = a.edges;
  p.lut = reinterpret_cast<const uint8_t*>(ws);
  p.lut_ok = reinterpret_cast<const int*>(reinterpret_cast<const char*>(ws) + TP_LUT);
  p.hist = a.hist;
  p.cb = cb;
  p.samples = samples;
  p.R = R;
  p.n = a.n;
  p.nr = a.n_rand;
  p.nb = a.n_bins;
  p.ndet = ndet;
  p.nblk = tp_nblk(a.n, HK_TP_NP_SR, TP_SR_T);
  p.g0 = 0;
  p.g1 = (1 + 2 * a.n_rand) * a.n;
  p.z = opaque_zero();
  p.one = 1 + (int32_t)opaque_zero();
  p.four = 4 * p.one;
  p.eight = 8 * p.one;
  return p;
}

// Workspace (tpacf_ws_bytes): table [TP_LUT] u8 | ok flag (16 B) | row_done [nrows] (padded to 16 B) |
// accg [nh * N] | cntg [nh * N]  (nrows = nh * blocks of 128 * HK_TP_NP_SR points)
static size_t tp_ws_head() { return (size_t)TP_LUT + 16; }
static int tp_nrows(const hk_tpacf_args& a) { return (1 + 2 * a.n_rand) * tp_nblk(a.n, HK_TP_NP_SR, TP_SR_T); }
static size_t tp_rows_bytes(const hk_tpacf_args& a) { return ((size_t)tp_nrows(a) * sizeof(int) + 15) / 16 * 16; }
size_t tpacf_ws_bytes(const hk_tpacf_args& a) {
  const size_t nt = (size_t)(1 + 2 * a.n_rand) * (size_t)a.n;
  return tp_ws_head() + tp_rows_bytes(a) + nt * 8;
}

cudaError_t tpacf_lut_build(const hk_tpacf_args& a, void* ws, cudaStream_t s, uint32_t* z0, int64_t n0, uint32_t* z1,
                            int64_t n1) {
  int* ok = reinterpret_cast<int*>(reinterpret_cast<char*>(ws) + TP_LUT);
  tpacf_lut_kernel<<<TP_LUT / 256, 256, 0, s>>>(a.edges, a.n_bins, reinterpret_cast<uint8_t*>(ws), ok, z0, n0, z1, n1);
  count_launch();
  return cudaGetLastError();
}

static double tp_pairs(const hk_tpacf_args& a) {
  const double n = a.n;
  return (1 + a.n_rand) * n * (n - 1) / 2 + a.n_rand * n * n;
}

// hauberk_release_caches: the TPACF kernels keep no per-shape device state between calls (the
// single run's pieces are recomputed per call), so there is nothing to free.
void tpacf_release_caches() {}

template <int V>
static cudaError_t launch_tp_v(const hk_tpacf_args& a, TPParams p, void* ws, cudaStream_t s) {
  const size_t smem = tp_smem_bytes(p.nb + 2, HK_TP_NP_SR, TP_SR_T) + 16;  // + the piece descriptor
  cudaError_t e = cudaFuncSetAttribute(tpacf_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (p.g1 <= p.g0) return cudaSuccess;
  int dev = 0, nsm = 0, per_sm = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, tpacf_kernel<V>, TP_SR_T, smem)) != cudaSuccess) return e;
  char* w = reinterpret_cast<char*>(ws);
  TPSR q;
  q.nrows = tp_nrows(a);
  q.row_done = reinterpret_cast<int*>(w + tp_ws_head());
  const size_t nt = (size_t)(1 + 2 * p.nr) * (size_t)p.n;
  p.accg = reinterpret_cast<int32_t*>(w + tp_ws_head() + tp_rows_bytes(a));
  p.cntg = p.accg + nt;
  // pieces: one wave of nsm * per_sm CTAs holding equal pair-slot counts
  int64_t total = 0;
  for (int r = 0; r < q.nrows; ++r) {
    int h, blk, jlo;
    total += tp_sr_row(p.n, p.nr, p.nblk, p.g0, p.g1, r, &h, &blk, &jlo);
  }
  if (total <= 0) return cudaSuccess;
  {  // HK_TP_SR_SLOTS: pieces per wave-slot x 100 (experiments; default 100 = one wave)
    const char* v = getenv("HK_TP_SR_SLOTS");
    const int pct = v && atoi(v) > 0 ? atoi(v) : 100;
    q.slots = std::max(1, (int)((int64_t)nsm * std::max(1, per_sm) * pct / 100));
  }
  q.total = total;
  int64_t grid = 0, wcum = 0;
  for (int r = 0; r < q.nrows; ++r) {
    int h, blk, jlo;
    const int64_t wr = tp_sr_row(p.n, p.nr, p.nblk, p.g0, p.g1, r, &h, &blk, &jlo);
    grid += tp_sr_pieces(wr, wcum, p.n - jlo, q.slots, total);
    wcum += wr;
  }
  // (the histogram and, for CNT, the workspace's counters and partial sums were zeroed by the table
  // kernel: tpacf_launch)
  TimedScope ts(HK_TPACF, 0, tp_pairs(a) * (double)(p.g1 - p.g0) / (double)((1 + 2 * p.nr) * p.n), s);
  tpacf_kernel<V><<<(unsigned)grid, TP_SR_T, smem, s>>>(p, q);
  count_launch();
  return cudaGetLastError();
}

// Abstract threads [g0, g1) (g1 < 0: all) of one run, their counts added into hist (sharding).
cudaError_t tpacf_launch(int vflags, const hk_tpacf_args& a, const DevRanges& R, int ndet, hk_control* cb, float* samples,
                         void* ws, cudaStream_t s, int32_t g0, int32_t g1) {
  // the table kernel also zeroes the histogram and (detector variants) the partial-sum workspace
  const bool cnt = (vflags & (V_L | V_PROF)) != 0;
  uint32_t* ws_tail = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ws) + tp_ws_head());
  const int64_t ws_words = cnt ? (int64_t)((tpacf_ws_bytes(a) - tp_ws_head()) / 4) : 0;
  const int64_t hist_words = 2 * (int64_t)(1 + 2 * a.n_rand) * (a.n_bins + 2);
  cudaError_t e = tpacf_lut_build(a, ws, s, reinterpret_cast<uint32_t*>(a.hist), hist_words, ws_tail, ws_words);
  if (e != cudaSuccess) return e;
  TPParams p = tp_params(a, R, ndet, cb, samples, ws);
  p.g0 = g0;
  if (g1 >= 0) p.g1 = g1;
  switch (vflags) {
    case 0: return launch_tp_v<0>(a, p, ws, s);
    case V_NL | V_L: return launch_tp_v<V_NL | V_L>(a, p, ws, s);
    case V_NL: return launch_tp_v<V_NL>(a, p, ws, s);
    case V_L: return launch_tp_v<V_L>(a, p, ws, s);
    case V_PROF: return launch_tp_v<V_PROF>(a, p, ws, s);
  }
  return cudaErrorInvalidValue;
}

int tpacf_site_kind(int site) { return tpacf_site_kind_d(site); }

template <int KIND, bool FT>
static cudaError_t launch_tp_fi_k(const TPFIParams& q, int nrep, cudaStream_t s) {
  const size_t smem = tp_smem_bytes(q.base.nb + 2, HK_TP_NP_FI);
  cudaError_t e = cudaFuncSetAttribute(tpacf_fi_kernel<KIND, FT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int ncta = (1 + 2 * q.base.nr) * q.base.nblk;
  dim3 grid(nrep, 1 + ncta);  // dispatch order: the nrep faulted CTAs, then rank 0..ncta-1 x nrep replicas
  const hk_tpacf_args a{q.base.pts, q.base.edges, q.base.n, q.base.nr, q.base.nb, nullptr};
  TimedScope ts(HK_TPACF, 1, tp_pairs(a) * nrep, s);
  tpacf_fi_kernel<KIND, FT><<<grid, TP_THREADS, smem, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

cudaError_t tpacf_replay_launch(int kind, bool ft, const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
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
  TimedScope ts(HK_TPACF, 2, (double)a.n * 2 * nrep, s);
  if (ft) tpacf_replay_all_kernel<true><<<(nrep + 127) / 128, 128, 0, s>>>(q);
  else tpacf_replay_all_kernel<false><<<(nrep + 127) / 128, 128, 0, s>>>(q);
  count_launch();
  return cudaGetLastError();
}

TPFIParams tpacf_fi_params(const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults, unsigned long long* hist0,
                           hk_control* cb0, void* ws) {
  TPFIParams q{};
  q.base = tp_params(a, R, ndet, nullptr, nullptr, ws);
  q.base.nblk = tp_nblk(a.n, HK_TP_NP_FI);
  q.faults = faults;
  q.hist0 = hist0;
  q.cb0 = cb0;
  q.hist_elems = (int64_t)(1 + 2 * a.n_rand) * (a.n_bins + 2);
  return q;
}

// ws must hold a table built by tpacf_lut_build for a.edges (the campaign builds it once).
cudaError_t tpacf_fi_launch(int kind, bool ft, const hk_tpacf_args& a, const DevRanges& R, int ndet, const FaultRec* faults,
                            int nrep, unsigned long long* hist0, hk_control* cb0, void* ws, bool real, cudaStream_t s) {
  TPFIParams q = tpacf_fi_params(a, R, ndet, faults, hist0, cb0, ws);
  if (real) {
    dim3 grid((unsigned)(((int64_t)(1 + 2 * a.n_rand) * a.n + 127) / 128), nrep);
    tpacf_real_kernel<<<grid, 128, 0, s>>>(q, kind);
    count_launch();
    return cudaGetLastError();
  }
  if (ft) {
    switch (kind) {
#define K_(k) case k: return launch_tp_fi_k<k, true>(q, nrep, s);
      K_(TK_NL) K_(TK_LIVE) K_(TK_J) K_(TK_X2) K_(TK_Y2) K_(TK_Z2) K_(TK_DOT) K_(TK_BIN) K_(TK_HIDX) K_(TK_ACC) K_(TK_CNT)
#undef K_
    }
  } else {
    switch (kind) {
#define K_(k) case k: return launch_tp_fi_k<k, false>(q, nrep, s);
      K_(TK_NL) K_(TK_LIVE) K_(TK_J) K_(TK_X2) K_(TK_Y2) K_(TK_Z2) K_(TK_DOT) K_(TK_BIN) K_(TK_HIDX) K_(TK_ACC) K_(TK_CNT)
#undef K_
    }
  }
  return cudaErrorInvalidValue;
}

}  // namespace hk
