// host.cpp — the C ABI of libhauberk (include/hauberk.h): argument validation, control blocks,
// the value-range profiler (DESIGN R8/R9), the injection decode (R14/R15) and
// the replica-mode campaign driver.  Host C++; every per-element
// step of the path runs in the CUDA kernels of cp.cu / mriq.cu / tpacf.cu / classify.cu.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "hk_internal.h"

namespace hk {

static std::atomic<uint64_t> g_launches{0};
static volatile uint32_t g_zero = 0;
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
uint32_t opaque_zero() { return g_zero; }

static thread_local std::string g_err;

// ---- optional per-kernel event timing
struct TimedRec { cudaEvent_t a, b; int bench, cls; double work; };
static std::atomic<int> g_timing{0};
static std::vector<TimedRec> g_timed;
TimedScope::TimedScope(int bench_, int cls_, double work_, cudaStream_t s_) : bench(bench_), cls(cls_), work(work_), s(s_) {
  if (!g_timing.load()) return;
  cudaEvent_t e;
  if (cudaEventCreate(&e) == cudaSuccess && cudaEventRecord(e, s) == cudaSuccess) start = (void*)e;
}
TimedScope::~TimedScope() {
  if (!start) return;
  cudaEvent_t e;
  if (cudaEventCreate(&e) == cudaSuccess && cudaEventRecord(e, s) == cudaSuccess)
    g_timed.push_back(TimedRec{(cudaEvent_t)start, e, bench, cls, work});
}

static hk_status cuda_fail(cudaError_t e, const char* where) {
  g_err = std::string(where) + ": " + cudaGetErrorString(e);
  return e == cudaErrorMemoryAllocation ? HK_ERR_OOM : HK_ERR_CUDA;
}
static hk_status invalid(const char* why) {
  g_err = why;
  return HK_ERR_INVALID;
}
// Stream-ordered allocations of the library come from a private memory pool per device (release
// threshold: keep freed memory for the next call) so the caller's default pool keeps its own
// settings (the library no longer changes the default pool).
static cudaError_t lib_malloc(void** p, size_t bytes, cudaStream_t s) {
  static std::mutex mu;
  static cudaMemPool_t pools[64] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaMallocAsync(p, bytes, s);
  {
    std::lock_guard<std::mutex> lk(mu);
    if (!pools[dev]) {
      cudaMemPoolProps props{};
      props.allocType = cudaMemAllocationTypePinned;
      props.handleTypes = cudaMemHandleTypeNone;
      props.location.type = cudaMemLocationTypeDevice;
      props.location.id = dev;
      if ((e = cudaMemPoolCreate(&pools[dev], &props)) != cudaSuccess) return e;
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  return cudaMallocFromPoolAsync(p, bytes, pools[dev], s);
}

#define HK_CUDA(call, where)                       \
  do {                                             \
    cudaError_t _e = (call);                       \
    if (_e != cudaSuccess) return cuda_fail(_e, where); \
  } while (0)

// ---------------------------------------------------------------------------------------------
// Ranges: hk_ranges (host) -> DevRanges with alpha applied (R11)
// ---------------------------------------------------------------------------------------------
static DevRanges dev_ranges(const hk_ranges* r) {
  DevRanges d{};
  if (!r) return d;
  d.n_det = r->n_det;
  const float a = r->alpha > 0.f ? r->alpha : 1.f;
  for (int k = 0; k < 8 && k < r->n_det; ++k) {
    d.n[k] = std::max(0, std::min(3, r->det[k].n));
    for (int q = 0; q < d.n[k]; ++q) {
      const float lo = r->det[k].lo[q], hi = r->det[k].hi[q];
      d.lo[k][q] = lo > 0.f ? lo / a : lo * a;
      d.hi[k][q] = hi > 0.f ? hi * a : hi / a;
    }
  }
  return d;
}

static int vflags_of(int variant) {
  switch (variant) {
    case HK_BASE: return 0;
    case HK_FT: return V_NL | V_L;
    case HK_FT_NL: return V_NL;
    case HK_FT_L: return V_L;
    case HK_PROFILE: return V_PROF;
  }
  return -1;
}

// ---------------------------------------------------------------------------------------------
// Validation and per-benchmark geometry
// ---------------------------------------------------------------------------------------------
static bool cp_ok(const hk_cp_args* a) {
  if (!a || !a->atoms_ws || !a->grid || (a->n_atoms > 0 && !a->atoms)) return false;
  if (a->n_atoms < 0 || a->nx <= 0 || a->ny <= 0 || a->bx <= 0 || a->by <= 0) return false;
  if (!(a->unroll == 1 || a->unroll == 2 || a->unroll == 4 || a->unroll == 8)) return false;
  if (a->bx * a->by > 256 || a->nx % (a->bx * a->unroll) != 0 || a->ny % a->by != 0) return false;
  if ((a->bx * a->by) % 32 != 0) return false;
  if (((uintptr_t)a->atoms | (uintptr_t)a->atoms_ws) & 15u) return false;
  return true;
}
static bool mriq_ok(const hk_mriq_args* a) {
  if (!a || a->n_vox < 0 || a->n_k < 0 || !a->qr || !a->qi) return false;
  if (a->n_vox > 0 && (!a->x || !a->y || !a->z)) return false;
  if (a->n_k > 0 && (!a->kx || !a->ky || !a->kz || !a->phi_r || !a->phi_i || !a->kv_ws)) return false;
  if ((uintptr_t)a->kv_ws & 15u) return false;
  return true;
}
static bool tpacf_ok(const hk_tpacf_args* a) {
  if (!a || !a->pts || !a->edges || !a->hist) return false;
  if (a->n <= 0 || a->n_rand < 1 || a->n_bins < 1 || a->n_bins > 30) return false;
  if ((int64_t)(1 + 2 * a->n_rand) * a->n > INT32_MAX / 2) return false;  // abstract thread ids are int32
  return true;
}
static bool tpacf_edges_ok(const hk_tpacf_args* a, cudaStream_t s) {
  std::vector<float> e(a->n_bins + 1);
  if (cudaMemcpyAsync(e.data(), a->edges, sizeof(float) * e.size(), cudaMemcpyDeviceToHost, s) != cudaSuccess) return false;
  if (cudaStreamSynchronize(s) != cudaSuccess) return false;
  for (int k = 0; k < a->n_bins; ++k)
    if (!(e[k] > e[k + 1])) return false;
  return true;
}

static int64_t cp_threads(const hk_cp_args* a) { return (int64_t)(a->nx / a->unroll) * a->ny; }
// TPACF abstract thread g = h*N + i loops over j in [jb, N): jb = i + 1 on the self-correlation
// rows h <= n_rand (DD, RR_s), 0 on the DR rows.
static int64_t tp_threads(const hk_tpacf_args* a) { return (int64_t)(1 + 2 * a->n_rand) * a->n; }
static int64_t tp_trips(const hk_tpacf_args* a, int64_t g) {
  const int64_t h = g / a->n, i = g % a->n;
  return h <= a->n_rand ? (int64_t)a->n - (i + 1) : (int64_t)a->n;
}
static int64_t bench_threads(int b, const void* args) {
  if (b == HK_CP) return cp_threads((const hk_cp_args*)args);
  if (b == HK_MRIQ) return ((const hk_mriq_args*)args)->n_vox;
  return tp_threads((const hk_tpacf_args*)args);
}

// ---------------------------------------------------------------------------------------------
// Runs
// ---------------------------------------------------------------------------------------------
static hk_status run_common_checks(int variant, const hk_ranges* ranges, hk_control* d_cb, float* d_samples) {
  if (vflags_of(variant) < 0) return invalid("unknown variant");
  if ((variant == HK_FT || variant == HK_FT_L) && (!ranges || ranges->n_det <= 0)) {
    g_err = "FT variant needs profiled ranges";
    return HK_ERR_NO_RANGES;
  }
  if (variant != HK_BASE && !d_cb) return invalid("control block required");
  if (variant == HK_PROFILE && !d_samples) return invalid("PROFILE needs d_samples");
  if (ranges && (ranges->n_det < 0 || ranges->n_det > 8)) return invalid("n_det out of range");
  return HK_OK;
}

static hk_status run_bench(int b, const void* args, int variant, const hk_ranges* ranges, hk_control* d_cb,
                           float* d_samples, cudaStream_t s) {
  const int vf = vflags_of(variant);
  const DevRanges R = dev_ranges(ranges);
  int ndet = ranges ? ranges->n_det : 1;
  if (d_cb) HK_CUDA(control_init_launch(d_cb, 1, s), "control init");
  if (b == HK_CP) {
    const hk_cp_args* a = (const hk_cp_args*)args;
    ndet = std::min(ndet, a->unroll);
    // no zeroing: a whole run stores every grid point once, which equals R18's "+=" on a zeroed grid
    HK_CUDA(cp_launch(vf, *a, R, ndet, d_cb, d_samples, s), "cp kernel");
  } else if (b == HK_MRIQ) {
    const hk_mriq_args* a = (const hk_mriq_args*)args;
    ndet = std::min(ndet, 2);
    // no zeroing: a whole run stores every voxel's Qr, Qi once (R18's "+=" on zeroed outputs)
    HK_CUDA(mriq_launch(vf, *a, R, ndet, d_cb, d_samples, s), "mriq kernels");
  } else {
    const hk_tpacf_args* a = (const hk_tpacf_args*)args;
    ndet = std::min(ndet, 1);
    void* ws = nullptr;  // (tpacf_launch zeroes the histogram in its table kernel)
    HK_CUDA(lib_malloc(&ws, tpacf_ws_bytes(*a), s), "alloc tpacf workspace");
    cudaError_t e = tpacf_launch(vf, *a, R, ndet, d_cb, d_samples, ws, s);
    cudaFreeAsync(ws, s);
    HK_CUDA(e, "tpacf kernel");
  }
  return HK_OK;
}

// ---------------------------------------------------------------------------------------------
// Value-range profiler (L1489-1508; R8 value-space size, R9 threshold walk)
// ---------------------------------------------------------------------------------------------
static int64_t ord_of(float x) {
  uint32_t b;
  std::memcpy(&b, &x, 4);
  return (b & 0x80000000u) ? -(int64_t)(b & 0x7fffffffu) : (int64_t)b;
}
static float threshold(int k) {
  char buf[16];
  std::snprintf(buf, sizeof buf, "1e%d", k);
  return std::strtof(buf, nullptr);
}
struct Classes {
  int n = 0;
  float lo[3], hi[3];
  int64_t cost = 0;
};
static Classes classes_at(const std::vector<float>& v, float T) {
  bool have[3] = {false, false, false};
  float mn[3] = {0, 0, 0}, mx[3] = {0, 0, 0};
  for (float x : v) {
    const int c = x < -T ? 0 : (x > T ? 2 : 1);
    if (!have[c]) { have[c] = true; mn[c] = mx[c] = x; }
    else { mn[c] = std::min(mn[c], x); mx[c] = std::max(mx[c], x); }
  }
  Classes r;
  for (int c = 0; c < 3; ++c)
    if (have[c]) {
      r.lo[r.n] = mn[c]; r.hi[r.n] = mx[c]; r.n++;
      r.cost += ord_of(mx[c]) - ord_of(mn[c]) + 1;
    }
  return r;
}
static hk_range_set profile_search(const std::vector<float>& v, int t0) {
  hk_range_set out{};
  out.t_exp10 = t0;
  if (v.empty()) return out;
  int k = t0;
  const int64_t INF = INT64_MAX;
  for (;;) {
    const int64_t c0 = classes_at(v, threshold(k)).cost;
    const int64_t cm = k - 1 >= -38 ? classes_at(v, threshold(k - 1)).cost : INF;
    const int64_t cp = k + 1 <= 38 ? classes_at(v, threshold(k + 1)).cost : INF;
    if (!(cp < c0 || cm < c0)) break;
    k = (cp <= cm) ? k + 1 : k - 1;
  }
  const Classes r = classes_at(v, threshold(k));
  out.n = r.n;
  for (int q = 0; q < r.n; ++q) { out.lo[q] = r.lo[q]; out.hi[q] = r.hi[q]; }
  out.t_exp10 = k;
  return out;
}

// ---------------------------------------------------------------------------------------------
// Site catalogue and decode (R14, R15)
// ---------------------------------------------------------------------------------------------
static int num_sites(int b, int unroll) { return b == HK_CP ? 22 + 4 * unroll : (b == HK_MRIQ ? 36 : 30); }
static bool site_is_nl(int b, int s) {
  return b == HK_CP ? s <= 5 : (b == HK_MRIQ ? (s <= 3 || s >= MRIQ_PHIMAG_SITE0) : s <= 10);
}
static int site_width(int b, int s) {
  if (b == HK_CP) return (s == 12 || s == 13) ? 64 : 32;
  if (b == HK_MRIQ) return (s >= 9 && s <= 14) ? 64 : 32;
  return (s == 19 || s == 20) ? 64 : 32;
}
// Sites that exist only because of HAUBERK (absent from the FI-only binary, row a7): the loop
// detector's counter (CP, MRI-Q `it`), TPACF's expected trip count (@def 6, @live 13), acc and cnt.
static bool site_is_detector(int b, int unroll, int s) {
  if (b == HK_CP) return s == num_sites(b, unroll) - 1;
  if (b == HK_MRIQ) return s == 28;
  return s == 6 || s == 13 || s == 28 || s == 29;
}
static uint64_t splitmix(uint64_t seed, uint64_t m) {
  uint64_t z = seed + (m + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static uint64_t below(uint64_t r, uint64_t m) { return (uint64_t)(((unsigned __int128)r * m) >> 64); }

struct Catalog {
  int bench = -1, unroll = 1;
  std::vector<int> enabled;
  int64_t nthr = 0, uniform_trips = 0, total_trips = 0;
  int64_t nk = 0;  // MRI-Q: PhiMag threads (sites 29-35)
  int64_t nl_threads(int s) const { return (bench == HK_MRIQ && s >= MRIQ_PHIMAG_SITE0) ? nk : nthr; }
  std::vector<int64_t> prefix;  // TPACF: prefix[g] = trips of threads < g
};

static bool build_catalog(Catalog& K, int b, const void* args, uint64_t mask, int variant) {
  K.bench = b;
  if (b == HK_CP) {
    const hk_cp_args* a = (const hk_cp_args*)args;
    K.unroll = a->unroll;
    K.nthr = cp_threads(a);
    K.uniform_trips = a->n_atoms;
    K.total_trips = K.nthr * K.uniform_trips;
  } else if (b == HK_MRIQ) {
    const hk_mriq_args* a = (const hk_mriq_args*)args;
    K.nthr = a->n_vox;
    K.nk = a->n_k;
    K.uniform_trips = a->n_k;
    K.total_trips = K.nthr * K.uniform_trips;
  } else {
    const hk_tpacf_args* a = (const hk_tpacf_args*)args;
    K.nthr = tp_threads(a);
    K.prefix.resize(K.nthr + 1);
    K.prefix[0] = 0;
    for (int64_t g = 0; g < K.nthr; ++g) K.prefix[g + 1] = K.prefix[g] + tp_trips(a, g);
    K.total_trips = K.prefix[K.nthr];
  }
  for (int s = 0; s < num_sites(b, K.unroll) && s < 64; ++s) {
    if (!((mask >> s) & 1ull)) continue;
    if (variant == HK_FI_ONLY && site_is_detector(b, K.unroll, s)) continue;
    const int64_t D = site_is_nl(b, s) ? K.nl_threads(s) : K.total_trips;
    if (D > 0) K.enabled.push_back(s);
  }
  return !K.enabled.empty();
}

static hk_fault decode_one(const Catalog& K, uint64_t seed, int64_t n, int nbits) {
  hk_fault f{};
  f.hang = 0;
  const uint64_t r1 = splitmix(seed, 8 * (uint64_t)n + 1);
  const uint64_t r2 = splitmix(seed, 8 * (uint64_t)n + 2);
  const uint64_t r3 = splitmix(seed, 8 * (uint64_t)n + 3);
  const int s = K.enabled[below(r1, K.enabled.size())];
  f.site = s;
  if (site_is_nl(K.bench, s)) {
    f.thread = (int64_t)below(r2, (uint64_t)K.nl_threads(s));
    f.inst = 0;
  } else {
    const int64_t u = (int64_t)below(r2, (uint64_t)K.total_trips);
    if (K.prefix.empty()) {
      f.thread = u / K.uniform_trips;
      f.inst = u % K.uniform_trips;
    } else {
      // first g with prefix[g + 1] > u
      const int64_t g = (int64_t)(std::upper_bound(K.prefix.begin(), K.prefix.end(), u) - K.prefix.begin()) - 1;
      f.thread = g;
      f.inst = u - K.prefix[g];
    }
  }
  const int w = site_width(K.bench, s);
  if (nbits <= 1) {
    f.mask = 1ull << below(r3, (uint64_t)w);
    return f;
  }
  // NEXT f1 (Fig. 14): k distinct bits, partial Fisher-Yates over [0, w);
  // step 0 uses r_3, step t >= 1 output 16n + t of the stream seed ^ 0xD1B54A32D192ED03.
  const int k = std::min(nbits, w);
  int perm[64];
  for (int b = 0; b < w; ++b) perm[b] = b;
  uint64_t mask = 0;
  for (int t = 0; t < k; ++t) {
    const uint64_t r = t == 0 ? r3 : splitmix(seed ^ 0xD1B54A32D192ED03ull, 16 * (uint64_t)n + (uint64_t)t);
    const int j = t + (int)below(r, (uint64_t)(w - t));
    std::swap(perm[t], perm[j]);
    mask |= 1ull << perm[t];
  }
  f.mask = mask;
  return f;
}

static bool args_ok(int b, const void* a) {
  if (!a) return false;
  return b == HK_CP ? cp_ok((const hk_cp_args*)a) : (b == HK_MRIQ ? mriq_ok((const hk_mriq_args*)a) : tpacf_ok((const hk_tpacf_args*)a));
}

// ---------------------------------------------------------------------------------------------
// Campaign workspace per benchmark
// ---------------------------------------------------------------------------------------------
struct BenchWS {
  bool used = false;
  const void* args = nullptr;
  DevRanges R{};
  int ndet = 1;
  int64_t out_elems = 0;   // floats (CP/MRI-Q) or u64 (TPACF) per replica
  void* golden = nullptr;
  float* dM = nullptr;
  void* rep_out = nullptr;
  hk_control* rep_cb = nullptr;
  hk_control* gold_cb = nullptr;
  void* lut = nullptr;  // TPACF bucket table
  float4* kv_rep = nullptr;  // MRI-Q PhiMag-site replicas: per-replica k-space
  int batch = 0;
};

static int default_batch(int b, const void* args) {
  {  // HK_BATCH_<b>: replicas per launch override (experiments)
    char name[16];
    snprintf(name, sizeof name, "HK_BATCH_%d", b);
    const char* v = getenv(name);
    if (v && atoi(v) > 0) return atoi(v);
  }
  if (b == HK_CP) {
    const hk_cp_args* a = (const hk_cp_args*)args;
    const int64_t ctas = (int64_t)(a->nx / (a->bx * a->unroll)) * (a->ny / a->by);
    return (int)std::max<int64_t>(64, std::min<int64_t>(4096, (148 * 8 * 4) / std::max<int64_t>(ctas, 1)));
  }
  if (b == HK_MRIQ) return 256;
  return 64;
}

}  // namespace hk

using namespace hk;

extern "C" {

const char* hauberk_strerror(hk_status s) {
  switch (s) {
    case HK_OK: return "ok";
    case HK_ERR_INVALID: return "invalid argument";
    case HK_ERR_CUDA: return "CUDA error";
    case HK_ERR_NO_RANGES: return "FT variant without profiled ranges";
    case HK_ERR_OOM: return "out of device memory";
    case HK_ERR_UNSUPPORTED: return "unsupported shape or variant";
    case HK_ERR_PROFILE_NAN: return "profile sample is NaN/Inf";
    case HK_ERR_GOLDEN_ALARM: return "fault-free golden run raised an alarm";
  }
  return "unknown status";
}
const char* hauberk_last_error(void) { return g_err.c_str(); }
int32_t hauberk_version(void) { return HK_ABI_VERSION; }
uint64_t hauberk_launch_count(void) { return g_launches.load(); }

void hauberk_timing_enable(int32_t on) {
  g_timing.store(on ? 1 : 0);
  if (!on) {
    for (auto& r : g_timed) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
    g_timed.clear();
  }
}
hk_status hauberk_timing_read(int32_t bench, int32_t cls, double* ms, int64_t* launches, double* work) {
  if (!ms || !launches || !work) return invalid("timing_read: null output");
  *ms = 0; *launches = 0; *work = 0;
  std::vector<TimedRec> keep;
  for (auto& r : g_timed) {
    if (r.bench != bench || r.cls != cls) { keep.push_back(r); continue; }
    cudaError_t e = cudaEventSynchronize(r.b);
    if (e != cudaSuccess) return cuda_fail(e, "timing event");
    float t = 0.f;
    cudaEventElapsedTime(&t, r.a, r.b);
    *ms += t; *launches += 1; *work += r.work;
    cudaEventDestroy(r.a); cudaEventDestroy(r.b);
  }
  g_timed.swap(keep);
  return HK_OK;
}
int32_t hauberk_num_sites(int32_t bench, int32_t unroll) {
  if (bench < 0 || bench > 2) return 0;
  return num_sites(bench, unroll);
}
int32_t hauberk_detector_site(int32_t bench, int32_t unroll, int32_t site) {
  if (bench < 0 || bench > 2 || site < 0 || site >= num_sites(bench, unroll)) return -1;
  return site_is_detector(bench, unroll, site) ? 1 : 0;
}

hk_status hauberk_summarize(const int64_t counts[5], hk_summary* out) {
  if (!counts || !out) return invalid("summarize: null argument");
  int64_t tot = 0;
  for (int c = 0; c < 5; ++c) {
    if (counts[c] < 0) return invalid("summarize: negative count");
    tot += counts[c];
  }
  out->total = tot;
  if (tot == 0) {
    out->coverage = out->sdc = out->detected = out->failure = NAN;
    return invalid("summarize: empty campaign");
  }
  out->sdc = (double)counts[HK_UNDETECTED] / (double)tot;
  out->coverage = 1.0 - out->sdc;
  out->detected = (double)(counts[HK_DETECTED] + counts[HK_DETECTED_MASKED]) / (double)tot;
  out->failure = (double)counts[HK_FAILURE] / (double)tot;
  return HK_OK;
}

hk_status hauberk_extend_ranges(hk_range_set* set, const float* values, int32_t n, int32_t* added) {
  if (!set || n < 0 || (n > 0 && !values) || set->n < 0 || set->n > 3 || set->t_exp10 < -38 || set->t_exp10 > 38)
    return invalid("extend_ranges: bad arguments");
  const float T = threshold(set->t_exp10);
  auto cls = [&](float x) { return x < -T ? 0 : (x > T ? 2 : 1); };
  bool have[3] = {false, false, false};
  float lo[3] = {0, 0, 0}, hi[3] = {0, 0, 0};
  for (int r = 0; r < set->n; ++r) {
    const int c = cls(set->lo[r]);
    have[c] = true; lo[c] = set->lo[r]; hi[c] = set->hi[r];
  }
  int32_t add = 0;
  for (int32_t k = 0; k < n; ++k) {
    const float x = values[k];
    if (!std::isfinite(x)) continue;
    const int c = cls(x);
    if (!have[c]) { have[c] = true; lo[c] = hi[c] = x; ++add; }
    else { lo[c] = std::min(lo[c], x); hi[c] = std::max(hi[c], x); }
  }
  int r = 0;
  for (int c = 0; c < 3; ++c)
    if (have[c]) { set->lo[r] = lo[c]; set->hi[r] = hi[c]; ++r; }
  set->n = r;
  if (added) *added = add;
  return HK_OK;
}

static float ord_to_float(int32_t o) {
  const uint32_t b = o >= 0 ? (uint32_t)o : (0x80000000u | (uint32_t)(-(int64_t)o));
  float f;
  std::memcpy(&f, &b, 4);
  return f;
}
hk_status hauberk_outliers(const hk_control* cb, int32_t d, float out[2], int32_t* n) {
  if (!cb || !out || !n || d < 0 || d >= 8) return invalid("outliers: bad arguments");
  const int32_t lo = cb->outlier_min_ord[d], hi = cb->outlier_max_ord[d];
  *n = 0;
  if (lo > hi) return HK_OK;  // initial values 0x7fffffff / 0x80000000: nothing recorded
  out[(*n)++] = ord_to_float(lo);
  if (hi != lo) out[(*n)++] = ord_to_float(hi);
  return HK_OK;
}

float hauberk_alpha_update(float alpha, double fp_ratio, double hi, double lo) {
  if (fp_ratio > hi) return alpha * 10.0f;
  if (fp_ratio < lo && alpha >= 10.0f) return alpha / 10.0f;
  return alpha;
}

int32_t hauberk_diagnose(uint32_t alarm1, uint32_t fail1, uint32_t alarm2, uint32_t fail2, int32_t identical) {
  if (fail1) return HK_DIAG_FAILURE;
  if (!alarm1) return HK_DIAG_OK;
  if (fail2) return HK_DIAG_FAILURE;
  if (!alarm2) return HK_DIAG_TRANSIENT;
  return identical ? HK_DIAG_FALSE_ALARM : HK_DIAG_PERSISTENT;
}

void hauberk_release_caches(void) { tpacf_release_caches(); }

hk_status hauberk_run_cp(const hk_cp_args* args, int32_t variant, const hk_ranges* ranges, hk_control* d_cb,
                         float* d_samples, void* stream) {
  if (!cp_ok(args)) return invalid("hk_cp_args invalid (shape, alignment or null pointer)");
  hk_status st = run_common_checks(variant, ranges, d_cb, d_samples);
  if (st != HK_OK) return st;
  return run_bench(HK_CP, args, variant, ranges, d_cb, d_samples, (cudaStream_t)stream);
}

hk_status hauberk_run_mriq(const hk_mriq_args* args, int32_t variant, const hk_ranges* ranges, hk_control* d_cb,
                           float* d_samples, void* stream) {
  if (!mriq_ok(args)) return invalid("hk_mriq_args invalid");
  hk_status st = run_common_checks(variant, ranges, d_cb, d_samples);
  if (st != HK_OK) return st;
  return run_bench(HK_MRIQ, args, variant, ranges, d_cb, d_samples, (cudaStream_t)stream);
}

hk_status hauberk_run_tpacf(const hk_tpacf_args* args, int32_t variant, const hk_ranges* ranges, hk_control* d_cb,
                            float* d_samples, void* stream) {
  if (!tpacf_ok(args)) return invalid("hk_tpacf_args invalid");
  hk_status st = run_common_checks(variant, ranges, d_cb, d_samples);
  if (st != HK_OK) return st;
  return run_bench(HK_TPACF, args, variant, ranges, d_cb, d_samples, (cudaStream_t)stream);
}

hk_status hauberk_compare(const void* d_a, const void* d_b, int64_t n_words, hk_control* d_cb, void* stream) {
  if (!d_a || !d_b || !d_cb || n_words < 0) return invalid("compare: bad arguments");
  if (((uintptr_t)d_a | (uintptr_t)d_b) & 15u) return invalid("compare: buffers must be 16-byte aligned");
  cudaStream_t s = (cudaStream_t)stream;
  HK_CUDA(control_init_launch(d_cb, 1, s), "control init");
  if (n_words == 0) return HK_OK;
  HK_CUDA(compare_launch(d_a, d_b, n_words, d_cb, s), "compare");
  return HK_OK;
}

hk_status hauberk_part_units(int32_t bench, const void* args, int64_t* units, int64_t* granule) {
  if (bench < 0 || bench > 2 || !units || !granule || !args_ok(bench, args)) return invalid("part_units: bad bench/args");
  if (bench == HK_CP) {
    const hk_cp_args* a = (const hk_cp_args*)args;
    *units = a->ny; *granule = a->by;
  } else if (bench == HK_MRIQ) {
    *units = ((const hk_mriq_args*)args)->n_vox; *granule = 1;
  } else {
    const hk_tpacf_args* a = (const hk_tpacf_args*)args;
    *units = tp_threads(a); *granule = 1;  // abstract threads g = h*n + i
  }
  return HK_OK;
}

hk_status hauberk_run_part(int32_t bench, const void* args, int32_t variant, const hk_ranges* ranges, hk_control* d_cb,
                           int64_t begin, int64_t end, void* stream) {
  if (bench < 0 || bench > 2 || !args_ok(bench, args)) return invalid("run_part: bad bench/args");
  if (variant == HK_PROFILE) return invalid("run_part: PROFILE runs over the whole input (hauberk_profile_ranges)");
  hk_status st = run_common_checks(variant, ranges, d_cb, nullptr);
  if (st != HK_OK) return st;
  int64_t units = 0, granule = 1;
  hauberk_part_units(bench, args, &units, &granule);
  if (begin < 0 || end < begin || end > units || begin % granule != 0 || (end % granule != 0 && end != units))
    return invalid("run_part: [begin, end) outside the partition units or not aligned to the granule");
  cudaStream_t s = (cudaStream_t)stream;
  const int vf = vflags_of(variant);
  const DevRanges R = dev_ranges(ranges);
  int ndet = ranges ? ranges->n_det : 1;
  if (d_cb) HK_CUDA(control_init_launch(d_cb, 1, s), "control init");
  if (bench == HK_CP) {
    const hk_cp_args* a = (const hk_cp_args*)args;
    ndet = std::min(ndet, a->unroll);
    HK_CUDA(cudaMemsetAsync(a->grid + (size_t)begin * a->nx, 0, sizeof(float) * (size_t)(end - begin) * a->nx, s), "memset rows");
    HK_CUDA(cp_launch_rows(vf, *a, R, ndet, d_cb, nullptr, (int32_t)begin, (int32_t)end, s), "cp kernel");
  } else if (bench == HK_MRIQ) {
    hk_mriq_args a = *(const hk_mriq_args*)args;  // the voxel slice: independent abstract threads
    a.x += begin; a.y += begin; a.z += begin; a.qr += begin; a.qi += begin;
    a.n_vox = (int32_t)(end - begin);
    ndet = std::min(ndet, 2);
    if (a.n_vox == 0) return HK_OK;
    HK_CUDA(cudaMemsetAsync(a.qr, 0, sizeof(float) * (size_t)a.n_vox, s), "memset qr");
    HK_CUDA(cudaMemsetAsync(a.qi, 0, sizeof(float) * (size_t)a.n_vox, s), "memset qi");
    HK_CUDA(mriq_launch(vf, a, R, ndet, d_cb, nullptr, s), "mriq kernels");
  } else {
    const hk_tpacf_args* a = (const hk_tpacf_args*)args;
    ndet = std::min(ndet, 1);
    if (end == begin) {  // an empty part: a zeroed histogram (otherwise tpacf_launch zeroes it)
      HK_CUDA(cudaMemsetAsync(a->hist, 0, sizeof(unsigned long long) * (size_t)(1 + 2 * a->n_rand) * (a->n_bins + 2), s),
              "memset hist");
      return HK_OK;
    }
    void* ws = nullptr;
    HK_CUDA(lib_malloc(&ws, tpacf_ws_bytes(*a), s), "alloc tpacf workspace");
    cudaError_t e = tpacf_launch(vf, *a, R, ndet, d_cb, nullptr, ws, s, (int32_t)begin, (int32_t)end);
    cudaFreeAsync(ws, s);
    HK_CUDA(e, "tpacf kernel");
  }
  return HK_OK;
}

hk_status hauberk_profile_ranges(int32_t bench, const void* args, const hk_profile_opts* opts, hk_ranges* out,
                                 void* stream) {
  if (bench < 0 || bench > 2 || !out || !args_ok(bench, args)) return invalid("profile: bad bench/args");
  cudaStream_t s = (cudaStream_t)stream;
  const int maxvar = opts ? opts->maxvar : 1;
  const int t0 = opts ? opts->t0_exp10 : -5;
  const float alpha = opts ? opts->alpha : 1.f;
  const int cap = bench == HK_CP ? ((const hk_cp_args*)args)->unroll : (bench == HK_MRIQ ? 2 : 1);
  if (maxvar < 1 || maxvar > cap || t0 < -38 || t0 > 38 || !(alpha >= 1.f)) return invalid("profile: bad options");
  if (bench == HK_TPACF && !tpacf_edges_ok((const hk_tpacf_args*)args, s)) return invalid("edges must strictly decrease");
  const int64_t T = bench_threads(bench, args);
  float* d_samples = nullptr;
  hk_control* d_cb = nullptr;
  HK_CUDA(lib_malloc((void**)&d_samples, sizeof(float) * std::max<int64_t>(1, T * maxvar), s), "alloc samples");
  HK_CUDA(lib_malloc((void**)&d_cb, sizeof(hk_control), s), "alloc cb");
  hk_ranges pr{};
  pr.n_det = maxvar;
  pr.alpha = 1.f;
  hk_status st = run_bench(bench, args, HK_PROFILE, &pr, d_cb, d_samples, s);
  std::vector<float> h((size_t)(T * maxvar));
  if (st == HK_OK && T > 0) {
    cudaError_t e = cudaMemcpyAsync(h.data(), d_samples, sizeof(float) * h.size(), cudaMemcpyDeviceToHost, s);
    if (e != cudaSuccess) st = cuda_fail(e, "copy samples");
  }
  cudaFreeAsync(d_samples, s);
  cudaFreeAsync(d_cb, s);
  cudaError_t e = cudaStreamSynchronize(s);
  if (st != HK_OK) return st;
  if (e != cudaSuccess) return cuda_fail(e, "profile run");
  std::memset(out, 0, sizeof(*out));
  out->n_det = maxvar;
  out->alpha = alpha;
  std::vector<unsigned char> valid((size_t)T, 1);
  if (bench == HK_TPACF)
    for (int64_t g = 0; g < T; ++g) valid[g] = tp_trips((const hk_tpacf_args*)args, g) > 0;
  else if ((bench == HK_CP && ((const hk_cp_args*)args)->n_atoms == 0) || (bench == HK_MRIQ && ((const hk_mriq_args*)args)->n_k == 0))
    std::fill(valid.begin(), valid.end(), 0);
  for (int d = 0; d < maxvar; ++d) {
    std::vector<float> v;
    v.reserve((size_t)T);
    for (int64_t t = 0; t < T; ++t) {
      if (!valid[t]) continue;
      const float x = h[(size_t)(d * T + t)];
      if (!std::isfinite(x)) { g_err = "profile sample NaN/Inf"; return HK_ERR_PROFILE_NAN; }
      v.push_back(x);
    }
    out->det[d] = profile_search(v, t0);
  }
  return HK_OK;
}

hk_status hauberk_profile_search(const float* samples, int64_t n, int32_t t0_exp10, hk_range_set* out) {
  if (!out || n < 0 || (n > 0 && !samples) || t0_exp10 < -38 || t0_exp10 > 38) return invalid("profile_search: bad arguments");
  std::vector<float> v;
  v.reserve((size_t)n);
  for (int64_t i = 0; i < n; ++i) {
    if (!std::isfinite(samples[i])) { g_err = "profile sample NaN/Inf"; return HK_ERR_PROFILE_NAN; }
    v.push_back(samples[i]);
  }
  *out = profile_search(v, t0_exp10);
  return HK_OK;
}

hk_status hauberk_decode(int32_t bench_mode, const void* const args[3], const uint64_t site_mask[3], uint64_t seed,
                         int32_t nbits, int32_t variant, int64_t first, int64_t count, int32_t* bench_out, hk_fault* out) {
  if (!args || !site_mask || !bench_out || !out || count < 0 || first < 0 || bench_mode < -1 || bench_mode > 2 ||
      variant < 0 || variant > 1)
    return invalid("decode: bad arguments");
  Catalog K[3];
  bool have[3] = {false, false, false};
  for (int64_t q = 0; q < count; ++q) {
    const int64_t n = first + q;
    const int b = bench_mode >= 0 ? bench_mode : (int)(n % 3);
    if (!have[b]) {
      if (!args_ok(b, args[b])) return invalid("decode: args of a used benchmark are invalid");
      if (!build_catalog(K[b], b, args[b], site_mask[b], variant)) return invalid("decode: empty site catalogue");
      have[b] = true;
    }
    bench_out[q] = b;
    out[q] = decode_one(K[b], seed, n, nbits);
  }
  return HK_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------------------------
// Campaign session: golden runs, catalogues and replica workspaces prepared once; each
// hauberk_campaign_run enqueues one slice of injections without synchronising.
// ---------------------------------------------------------------------------------------------
#ifndef HK_CONCURRENT_DEFAULT
#define HK_CONCURRENT_DEFAULT 1
#endif
struct hk_campaign_session {
  DevCatalog dcat[3]{};
  int64_t* d_prefix = nullptr;  // TPACF trip prefix sums on the device (replay decode)
  void* d_decode = nullptr;
  size_t decode_cap = 0;
  int bench_mode = -1;
  hk_campaign cfg{};
  hk_cp_args cp{};
  hk_mriq_args mq{};
  hk_tpacf_args tp{};
  BenchWS W[3];
  Catalog K[3];
  FaultRec* d_faults = nullptr;
  size_t d_cap = 0;
  FaultRec* h_faults = nullptr;  // pinned staging
  size_t h_cap = 0;
  cudaEvent_t uploaded = nullptr;
  cudaStream_t stream = nullptr;
  // replica mode, mixed campaigns: one forked stream per benchmark so the XU-bound MRI-Q
  // replicas and the issue-bound TPACF replicas can share SMs (joined back into `stream`)
  bool concurrent = false;
  // replica mode, mixed campaigns: MRI-Q (Q-kernel sites) and TPACF replicas share fused launches
  // (mix.cu) so both kinds of CTA are resident on every SM (HK_FUSED=0: separate launches)
  bool fused = false;
  cudaStream_t sub[3]{};
  cudaEvent_t fork = nullptr, join[3]{};
};

static void session_free(hk_campaign_session* S) {
  if (!S) return;
  if (S->stream) cudaStreamSynchronize(S->stream);
  for (int b = 0; b < 3; ++b) {
    BenchWS& w = S->W[b];
    if (w.golden) cudaFree(w.golden);
    if (w.dM) cudaFree(w.dM);
    if (w.rep_out) cudaFree(w.rep_out);
    if (w.rep_cb) cudaFree(w.rep_cb);
    if (w.gold_cb) cudaFree(w.gold_cb);
    if (w.lut) cudaFree(w.lut);
    if (w.kv_rep) cudaFree(w.kv_rep);
  }
  if (S->d_faults) cudaFree(S->d_faults);
  if (S->h_faults) cudaFreeHost(S->h_faults);
  if (S->d_prefix) cudaFree(S->d_prefix);
  if (S->d_decode) cudaFree(S->d_decode);
  if (S->uploaded) cudaEventDestroy(S->uploaded);
  for (int b = 0; b < 3; ++b) {
    if (S->sub[b]) cudaStreamDestroy(S->sub[b]);
    if (S->join[b]) cudaEventDestroy(S->join[b]);
  }
  if (S->fork) cudaEventDestroy(S->fork);
  delete S;
}

static hk_status session_create(int32_t bench_mode, const void* const args[3], const hk_ranges* const ranges[3],
                                const hk_campaign* C, cudaStream_t s, hk_campaign_session** out) {
  if (!args || !ranges || !C || !out || bench_mode < -1 || bench_mode > 2) return invalid("campaign: bad arguments");
  if (C->mode < 0 || C->mode > 2) return invalid("campaign: mode must be 0 (replica), 1 (replay) or 2 (unguarded replica)");
  if (C->nbits < 0 || C->nbits > 64) return invalid("campaign: nbits out of range");
  if (C->variant != HK_FIFT && C->variant != HK_FI_ONLY) return invalid("campaign: variant must be HK_FIFT or HK_FI_ONLY");
  if (C->hang_factor < 0) return invalid("campaign: hang_factor must be >= 0 (0 = the paper's 10)");
  const bool ft = C->variant == HK_FIFT;
  hk_campaign_session* S = new hk_campaign_session();
  S->bench_mode = bench_mode;
  S->cfg = *C;
  S->stream = s;
  {
    const char* env = getenv("HK_CONCURRENT");
    S->concurrent = env ? atoi(env) != 0 : HK_CONCURRENT_DEFAULT;
    const char* fe = getenv("HK_FUSED");
    S->fused = (fe ? atoi(fe) != 0 : true) && C->mode == 0 && bench_mode == -1 && args[HK_MRIQ] && args[HK_TPACF];
  }
  hk_status st = HK_OK;
  cudaError_t e;
  for (int b = 0; b < 3 && st == HK_OK; ++b) {
    const bool want = bench_mode == b || (bench_mode == -1 && args[b] != nullptr);
    if (!want) continue;
    if (!args_ok(b, args[b])) { st = invalid("campaign: args of a used benchmark are invalid"); break; }
    if (ft && (!ranges[b] || ranges[b]->n_det <= 0)) { g_err = "campaign: ranges missing"; st = HK_ERR_NO_RANGES; break; }
    if (b == HK_CP && ((const hk_cp_args*)args[b])->unroll != 4 && ((const hk_cp_args*)args[b])->unroll != 8) {
      g_err = "campaign kernels are built for CP unroll 4 and 8"; st = HK_ERR_UNSUPPORTED; break;
    }
    if (b == HK_TPACF && !tpacf_edges_ok((const hk_tpacf_args*)args[b], s)) { st = invalid("edges must strictly decrease"); break; }
    const void* own = b == HK_CP ? (const void*)&S->cp : (b == HK_MRIQ ? (const void*)&S->mq : (const void*)&S->tp);
    if (b == HK_CP) S->cp = *(const hk_cp_args*)args[b];
    else if (b == HK_MRIQ) S->mq = *(const hk_mriq_args*)args[b];
    else S->tp = *(const hk_tpacf_args*)args[b];
    if (!build_catalog(S->K[b], b, own, C->site_mask[b], C->variant)) { st = invalid("campaign: empty site catalogue"); break; }
    BenchWS& w = S->W[b];
    w.used = true;
    w.args = own;
    w.R = dev_ranges(ft ? ranges[b] : nullptr);  // the FI-only binary has no detectors
    w.ndet = ft ? ranges[b]->n_det : 0;
    w.batch = C->mode == 1 ? 1 : (C->batch > 0 ? C->batch : default_batch(b, own));
    if (b == HK_TPACF && S->fused) {
      S->fused = S->W[HK_MRIQ].used && mix_supported(S->mq, S->tp);
      // a fused launch pairs as many TPACF replicas as MRI-Q ones (the TPACF workspace is small)
      if (S->fused && C->batch <= 0 && !getenv("HK_BATCH_2")) w.batch = std::max(w.batch, S->W[HK_MRIQ].batch);
    }
    if (C->mode == 1 && b == HK_TPACF && 3 * S->tp.n_bins > 96) { g_err = "replay supports n_bins <= 32"; st = HK_ERR_UNSUPPORTED; break; }
    const bool phimag_sites = b == HK_MRIQ && (C->site_mask[b] >> MRIQ_PHIMAG_SITE0) != 0;
    if (C->mode == 1 && phimag_sites) {
      g_err = "PhiMag sites reach every voxel: replica mode only (clear site_mask bits 29-35 for replay)";
      st = HK_ERR_UNSUPPORTED;
      break;
    }
    size_t esz = sizeof(float);
    if (b == HK_CP) w.out_elems = (int64_t)S->cp.nx * S->cp.ny;
    else if (b == HK_MRIQ) w.out_elems = 2LL * S->mq.n_vox;
    else { w.out_elems = (int64_t)(1 + 2 * S->tp.n_rand) * (S->tp.n_bins + 2); esz = 8; }
    const int64_t stride = (w.out_elems + 3) / 4 * 4;  // keep replicas 16-byte aligned
    w.out_elems = stride;
    if ((e = cudaMalloc(&w.golden, esz * stride)) != cudaSuccess ||
        (e = cudaMalloc((void**)&w.dM, sizeof(float))) != cudaSuccess ||
        (e = cudaMalloc((void**)&w.gold_cb, sizeof(hk_control))) != cudaSuccess ||
        (e = cudaMalloc(&w.rep_out, esz * stride * w.batch)) != cudaSuccess ||
        (e = cudaMalloc((void**)&w.rep_cb, sizeof(hk_control) * w.batch)) != cudaSuccess ||
        (b == HK_MRIQ && (C->site_mask[b] >> MRIQ_PHIMAG_SITE0) != 0 &&
         (e = cudaMalloc((void**)&w.kv_rep, sizeof(float4) * (size_t)std::max(1, S->mq.n_k) * w.batch)) != cudaSuccess)) {
      st = cuda_fail(e, "campaign workspace");
      break;
    }
    if ((e = cudaMemsetAsync(w.golden, 0, esz * stride, s)) != cudaSuccess ||
        (e = cudaMemsetAsync(w.rep_out, 0, esz * stride * w.batch, s)) != cudaSuccess ||
        (e = control_init_launch(w.rep_cb, w.batch, s)) != cudaSuccess) {
      st = cuda_fail(e, "campaign init");
      break;
    }
    // golden = this library's own fault-free output of the same binary (R7): FT, or BASE for FI-only
    const int gv = ft ? HK_FT : HK_BASE;
    const hk_ranges* gr = ft ? ranges[b] : nullptr;
    if (b == HK_CP) {
      hk_cp_args a = S->cp;
      a.grid = (float*)w.golden;
      st = run_bench(b, &a, gv, gr, w.gold_cb, nullptr, s);
      if (st == HK_OK && (e = max_abs_launch((float*)w.golden, (int64_t)a.nx * a.ny, w.dM, s)) != cudaSuccess) st = cuda_fail(e, "max");
    } else if (b == HK_MRIQ) {
      hk_mriq_args a = S->mq;
      a.qr = (float*)w.golden;
      a.qi = a.qr + a.n_vox;
      st = run_bench(b, &a, gv, gr, w.gold_cb, nullptr, s);
      if (st == HK_OK && (e = max_abs_launch((float*)w.golden, 2LL * a.n_vox, w.dM, s)) != cudaSuccess) st = cuda_fail(e, "max");
    } else {
      hk_tpacf_args a = S->tp;
      a.hist = (unsigned long long*)w.golden;
      st = run_bench(b, &a, gv, gr, w.gold_cb, nullptr, s);
      if (st == HK_OK && (e = cudaMalloc(&w.lut, tpacf_ws_bytes(a))) != cudaSuccess) st = cuda_fail(e, "alloc table");
      if (st == HK_OK && (e = tpacf_lut_build(a, w.lut, s)) != cudaSuccess) st = cuda_fail(e, "table");
    }
  }
  if (st == HK_OK && !(S->W[0].used || S->W[1].used || S->W[2].used)) st = invalid("campaign: no benchmark");
  if (st == HK_OK) {
    hk_control hc[3];
    for (int b = 0; b < 3; ++b)
      if (S->W[b].used) cudaMemcpyAsync(&hc[b], S->W[b].gold_cb, sizeof(hk_control), cudaMemcpyDeviceToHost, s);
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) st = cuda_fail(e, "golden runs");
    for (int b = 0; b < 3 && st == HK_OK; ++b)
      if (S->W[b].used && (hc[b].alarm != 0 || hc[b].fail != 0)) {
        g_err = "golden run alarm (ranges were not profiled on this input)";
        st = HK_ERR_GOLDEN_ALARM;
      }
  }
  if (st == HK_OK && (e = cudaEventCreateWithFlags(&S->uploaded, cudaEventDisableTiming)) != cudaSuccess)
    st = cuda_fail(e, "event");
  // device catalogues for the replay path's on-device decode
  for (int b = 0; b < 3 && st == HK_OK; ++b) {
    if (!S->W[b].used) continue;
    const Catalog& K = S->K[b];
    DevCatalog& D = S->dcat[b];
    D.nen = (int)K.enabled.size();
    for (int q = 0; q < D.nen; ++q) D.en[q] = K.enabled[q];
    const int U = b == HK_CP ? S->cp.unroll : 1;
    for (int site = 0; site < 64 && site < num_sites(b, U); ++site) {
      int sub = 0, kind = 0;
      if (b == HK_CP) kind = cp_site_kind(site, U, &sub);
      else if (b == HK_MRIQ) kind = mriq_site_kind(site);
      else kind = tpacf_site_kind(site);
      D.is_nl[site] = site_is_nl(b, site) ? 1 : 0;
      D.width[site] = (uint8_t)site_width(b, site);
      D.kind[site] = (uint8_t)kind;
      D.sub[site] = (uint8_t)sub;
    }
    D.nthr = K.nthr; D.nk = K.nk; D.uniform_trips = K.uniform_trips; D.total_trips = K.total_trips;
    D.prefix = nullptr;
    if (!K.prefix.empty()) {
      if ((e = cudaMalloc((void**)&S->d_prefix, sizeof(int64_t) * K.prefix.size())) != cudaSuccess ||
          (e = cudaMemcpy(S->d_prefix, K.prefix.data(), sizeof(int64_t) * K.prefix.size(), cudaMemcpyHostToDevice)) != cudaSuccess)
        st = cuda_fail(e, "prefix");
      D.prefix = S->d_prefix;
    }
  }
  if (st != HK_OK) { session_free(S); return st; }
  *out = S;
  return HK_OK;
}

static hk_status session_run(hk_campaign_session* S, int64_t first, int64_t count, hk_outcome* d_records,
                             int64_t* d_counts, int64_t* d_site_counts) {
  if (!S || !d_counts || first < 0 || count < 0) return invalid("campaign_run: bad arguments");
  if (count == 0) return HK_OK;
  cudaStream_t s = S->stream;
  cudaError_t e;
  if (S->cfg.mode == 1) {
    // ---- replay: decode and sort on the device, then one launch per benchmark (no host round trip)
    int64_t per[3] = {0, 0, 0};
    if (S->bench_mode >= 0) per[S->bench_mode] = count;
    else
      for (int b = 0; b < 3; ++b) {
        const int64_t off = (b - first % 3 + 3) % 3;
        per[b] = count > off ? (count - off + 2) / 3 : 0;
      }
    for (int b = 0; b < 3; ++b)
      if (per[b] && !S->W[b].used) return invalid("campaign_run: index hits a benchmark the session was not created with");
    const size_t need = decode_ws_bytes(count);
    if (S->decode_cap < need) {
      if (S->d_decode) cudaFreeAsync(S->d_decode, s);
      S->d_decode = nullptr;
      S->decode_cap = 0;
      if ((e = lib_malloc(&S->d_decode, need, s)) != cudaSuccess) return cuda_fail(e, "decode workspace");
      S->decode_cap = need;
    }
    FaultRec* sorted = nullptr;
    if ((e = decode_sort_launch(S->dcat, S->cfg.seed, first, count, S->bench_mode, S->cfg.nbits, S->cfg.hang_factor,
                                S->d_decode, &sorted, s)) != cudaSuccess)
      return cuda_fail(e, "device decode");
    int64_t off = 0;
    for (int b = 0; b < 3; ++b) {
      if (!per[b]) continue;
      BenchWS& w = S->W[b];
      const FaultRec* fr = sorted + off;
      const int nrep = (int)per[b];
      const bool ft = S->cfg.variant == HK_FIFT;
      if (b == HK_CP) e = cp_replay_launch(0, ft, S->cp, w.R, std::min(w.ndet, S->cp.unroll), fr, nrep, (const float*)w.golden,
                                           w.dM, d_records, first, d_counts, d_site_counts, s);
      else if (b == HK_MRIQ) e = mriq_replay_launch(0, ft, S->mq, w.R, std::min(w.ndet, 2), fr, nrep, (const float*)w.golden,
                                                    w.dM, d_records, first, d_counts, d_site_counts, s);
      else e = tpacf_replay_launch(0, ft, S->tp, w.R, std::min(w.ndet, 1), fr, nrep, (const unsigned long long*)w.golden,
                                   d_records, first, d_counts, d_site_counts, s);
      if (e != cudaSuccess) return cuda_fail(e, "replay");
      off += per[b];
    }
    return HK_OK;
  }
  // ---- replica: decode on the host, group by (bench, kind)
  struct Item { int b, kind; FaultRec f; };
  std::vector<Item> items((size_t)count);
  for (int64_t q = 0; q < count; ++q) {
    const int64_t n = first + q;
    const int b = S->bench_mode >= 0 ? S->bench_mode : (int)(n % 3);
    if (!S->W[b].used) return invalid("campaign_run: index hits a benchmark the session was not created with");
    const hk_fault hf = decode_one(S->K[b], S->cfg.seed, n, S->cfg.nbits);
    Item it{};
    it.b = b;
    it.f.index = n; it.f.thread = hf.thread; it.f.inst = hf.inst; it.f.mask = hf.mask; it.f.site = hf.site;
    int sub = 0;
    if (b == HK_CP) it.kind = cp_site_kind(hf.site, S->cp.unroll, &sub);
    else if (b == HK_MRIQ) it.kind = mriq_site_kind(hf.site);
    else it.kind = tpacf_site_kind(hf.site);
    it.f.sub = sub;
    it.f.real = S->cfg.mode == 2 ? 1 : 0;  // R25: guardian child processes only
    it.f.hang = S->cfg.hang_factor;
    items[(size_t)q] = it;
  }
  const auto by_kind = [](const Item& x, const Item& y) { return x.b != y.b ? x.b < y.b : x.kind < y.kind; };
  std::stable_sort(items.begin(), items.end(), by_kind);
  // ---- fused MRI-Q + TPACF chunks first (MRI-Q slice, then TPACF slice), then the rest by kind
  struct Chunk { size_t m_off; int rm; size_t t_off; int rt; };
  std::vector<Chunk> chunks;
  size_t rest_off = 0;
  if (S->fused && S->cfg.mode == 0) {
    std::vector<Item> M, T, order, rest;
    for (const Item& it : items) {
      if (it.b == HK_MRIQ && it.f.site < MRIQ_PHIMAG_SITE0) M.push_back(it);
      else if (it.b == HK_TPACF) T.push_back(it);
      else rest.push_back(it);
    }
    if (!M.empty() && !T.empty()) {
      const int64_t nm = (int64_t)M.size(), nt = (int64_t)T.size();
      const int64_t bm = S->W[HK_MRIQ].batch, bt = S->W[HK_TPACF].batch;
      const int64_t k = std::max((nm + bm - 1) / bm, (nt + bt - 1) / bt);
      order.reserve(items.size());
      for (int64_t j = 0; j < k; ++j) {
        const int64_t m0 = nm * j / k, m1 = nm * (j + 1) / k, t0 = nt * j / k, t1 = nt * (j + 1) / k;
        if (m1 > m0 && t1 > t0) {
          chunks.push_back(Chunk{order.size(), (int)(m1 - m0), order.size() + (size_t)(m1 - m0), (int)(t1 - t0)});
          order.insert(order.end(), M.begin() + m0, M.begin() + m1);
          order.insert(order.end(), T.begin() + t0, T.begin() + t1);
        } else {
          rest.insert(rest.end(), M.begin() + m0, M.begin() + m1);
          rest.insert(rest.end(), T.begin() + t0, T.begin() + t1);
        }
      }
      std::stable_sort(rest.begin(), rest.end(), by_kind);
      rest_off = order.size();
      order.insert(order.end(), rest.begin(), rest.end());
      items.swap(order);
    }
  }
  // ---- upload through the pinned staging buffer (wait until the previous upload consumed it)
  if ((e = cudaEventSynchronize(S->uploaded)) != cudaSuccess) return cuda_fail(e, "staging");
  if (S->h_cap < items.size()) {
    if (S->h_faults) cudaFreeHost(S->h_faults);
    S->h_faults = nullptr;
    S->h_cap = 0;
    if ((e = cudaMallocHost((void**)&S->h_faults, sizeof(FaultRec) * items.size())) != cudaSuccess) return cuda_fail(e, "pinned");
    S->h_cap = items.size();
  }
  if (S->d_cap < items.size()) {
    if (S->d_faults) cudaFreeAsync(S->d_faults, s);
    S->d_faults = nullptr;
    S->d_cap = 0;
    if ((e = lib_malloc((void**)&S->d_faults, sizeof(FaultRec) * items.size(), s)) != cudaSuccess) return cuda_fail(e, "faults");
    S->d_cap = items.size();
  }
  for (size_t q = 0; q < items.size(); ++q) S->h_faults[q] = items[q].f;
  if ((e = cudaMemcpyAsync(S->d_faults, S->h_faults, sizeof(FaultRec) * items.size(), cudaMemcpyHostToDevice, s)) != cudaSuccess)
    return cuda_fail(e, "upload faults");
  cudaEventRecord(S->uploaded, s);

  // ---- batches: FI&FT replicas, then the classify epilogue (which also recycles the workspace)
  const bool real = S->cfg.mode == 2;  // R25: unguarded replicas (guardian child processes only)
  const bool ft = S->cfg.variant == HK_FIFT;
  const cudaStream_t s0 = s;
  bool touched[3] = {false, false, false};
  for (const Item& it : items) touched[it.b] = true;
  const bool conc = S->concurrent && (int)touched[0] + (int)touched[1] + (int)touched[2] > 1;
  if (conc) {
    if (!S->fork && (e = cudaEventCreateWithFlags(&S->fork, cudaEventDisableTiming)) != cudaSuccess) return cuda_fail(e, "event");
    for (int b = 0; b < 3; ++b) {
      if (!touched[b]) continue;
      if (!S->sub[b]) {
        // HK_CONC_PRIO=b: benchmark b's stream gets the highest priority (experiments)
        const char* pe = getenv("HK_CONC_PRIO");
        int lo = 0, hi = 0;
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        const int prio = (pe && atoi(pe) == b) ? hi : lo;
        if ((e = cudaStreamCreateWithPriority(&S->sub[b], cudaStreamNonBlocking, prio)) != cudaSuccess)
          return cuda_fail(e, "stream");
      }
      if (!S->join[b] && (e = cudaEventCreateWithFlags(&S->join[b], cudaEventDisableTiming)) != cudaSuccess)
        return cuda_fail(e, "event");
    }
    if ((e = cudaEventRecord(S->fork, s0)) != cudaSuccess) return cuda_fail(e, "fork");
    for (int b = 0; b < 3; ++b)
      if (touched[b] && (e = cudaStreamWaitEvent(S->sub[b], S->fork, 0)) != cudaSuccess) return cuda_fail(e, "fork");
  }
  // fused launches and any MRI-Q / TPACF launch of the rest share one stream (one workspace each)
  const auto stream_of = [&](int b) { return conc ? S->sub[!chunks.empty() && b == HK_TPACF ? HK_MRIQ : b] : s0; };
  for (const Chunk& c : chunks) {
    s = stream_of(HK_MRIQ);
    BenchWS& wm = S->W[HK_MRIQ];
    BenchWS& wt = S->W[HK_TPACF];
    const FaultRec* fm = S->d_faults + c.m_off;
    const FaultRec* ftp = S->d_faults + c.t_off;
    if ((e = mix_fi_launch(ft, S->mq, wm.R, std::min(wm.ndet, 2), fm, c.rm, (float*)wm.rep_out, wm.out_elems, wm.rep_cb, S->tp, wt.R,
                           std::min(wt.ndet, 1), ftp, c.rt, (unsigned long long*)wt.rep_out, wt.rep_cb, wt.lut, s)) != cudaSuccess)
      return cuda_fail(e, "fused FI");
    if ((e = classify_fp_launch(HK_MRIQ, (float*)wm.rep_out, wm.out_elems, (const float*)wm.golden, wm.dM, wm.rep_cb, fm, c.rm,
                                d_records, first, d_counts, d_site_counts, s)) != cudaSuccess ||
        (e = classify_tpacf_launch((unsigned long long*)wt.rep_out, S->tp.n_rand, S->tp.n_bins, (const unsigned long long*)wt.golden,
                                   wt.rep_cb, ftp, c.rt, d_records, first, d_counts, d_site_counts, s)) != cudaSuccess)
      return cuda_fail(e, "classify");
  }
  size_t q = rest_off;
  while (q < items.size()) {
    const int b = items[q].b, kind = items[q].kind;
    s = stream_of(b);
    size_t end = q;
    while (end < items.size() && items[end].b == b && items[end].kind == kind && (int)(end - q) < S->W[b].batch) ++end;
    const int nrep = (int)(end - q);
    BenchWS& w = S->W[b];
    const FaultRec* fr = S->d_faults + q;
    if (b == HK_CP) {
      if ((e = cp_fi_launch(kind, ft, S->cp, w.R, std::min(w.ndet, S->cp.unroll), fr, nrep, (float*)w.rep_out, w.out_elems, w.rep_cb,
                            real, s)) != cudaSuccess)
        return cuda_fail(e, "cp FI");
      if ((e = classify_fp_launch(b, (float*)w.rep_out, w.out_elems, (const float*)w.golden, w.dM, w.rep_cb, fr, nrep,
                                  d_records, first, d_counts, d_site_counts, s)) != cudaSuccess)
        return cuda_fail(e, "classify");
    } else if (b == HK_MRIQ) {
      if ((e = mriq_fi_launch(kind, ft, S->mq, w.R, std::min(w.ndet, 2), fr, nrep, (float*)w.rep_out, w.out_elems, w.rep_cb,
                              w.kv_rep, real, s)) != cudaSuccess)
        return cuda_fail(e, "mriq FI");
      if ((e = classify_fp_launch(b, (float*)w.rep_out, w.out_elems, (const float*)w.golden, w.dM, w.rep_cb, fr, nrep,
                                  d_records, first, d_counts, d_site_counts, s)) != cudaSuccess)
        return cuda_fail(e, "classify");
    } else {
      if ((e = tpacf_fi_launch(kind, ft, S->tp, w.R, std::min(w.ndet, 1), fr, nrep, (unsigned long long*)w.rep_out, w.rep_cb,
                               w.lut, real, s)) != cudaSuccess)
        return cuda_fail(e, "tpacf FI");
      if ((e = classify_tpacf_launch((unsigned long long*)w.rep_out, S->tp.n_rand, S->tp.n_bins,
                                     (const unsigned long long*)w.golden, w.rep_cb, fr, nrep, d_records, first, d_counts,
                                     d_site_counts, s)) != cudaSuccess)
        return cuda_fail(e, "classify");
    }
    q = end;
  }
  if (conc)
    for (int b = 0; b < 3; ++b) {
      if (!touched[b]) continue;
      if ((e = cudaEventRecord(S->join[b], S->sub[b])) != cudaSuccess || (e = cudaStreamWaitEvent(s0, S->join[b], 0)) != cudaSuccess)
        return cuda_fail(e, "join");
    }
  return HK_OK;
}

extern "C" {

hk_status hauberk_campaign_create(int32_t bench_mode, const void* const args[3], const hk_ranges* const ranges[3],
                                  const hk_campaign* campaign, hk_campaign_session** out, void* stream) {
  return session_create(bench_mode, args, ranges, campaign, (cudaStream_t)stream, out);
}

hk_status hauberk_campaign_run(hk_campaign_session* session, int64_t first, int64_t count, hk_outcome* d_records,
                               int64_t* d_counts, int64_t* d_site_counts) {
  return session_run(session, first, count, d_records, d_counts, d_site_counts);
}

void hauberk_campaign_destroy(hk_campaign_session* session) { session_free(session); }

size_t hauberk_campaign_workspace_bytes(int32_t bench, const void* args, const hk_campaign* C) {
  if (bench < 0 || bench > 2 || !C || !args_ok(bench, args) || C->mode < 0 || C->mode > 2) return 0;
  const int batch = C->mode == 1 ? 1 : (C->batch > 0 ? C->batch : default_batch(bench, args));
  size_t esz = sizeof(float);
  int64_t elems = 0;
  if (bench == HK_CP) elems = (int64_t)((const hk_cp_args*)args)->nx * ((const hk_cp_args*)args)->ny;
  else if (bench == HK_MRIQ) elems = 2LL * ((const hk_mriq_args*)args)->n_vox;
  else {
    const hk_tpacf_args* a = (const hk_tpacf_args*)args;
    elems = (int64_t)(1 + 2 * a->n_rand) * (a->n_bins + 2);
    esz = 8;
  }
  const size_t stride = (size_t)((elems + 3) / 4 * 4);
  size_t bytes = esz * stride * (1 + (size_t)batch) + sizeof(float) + sizeof(hk_control) * (1 + (size_t)batch);
  if (bench == HK_TPACF) bytes += tpacf_ws_bytes(*(const hk_tpacf_args*)args);
  if (bench == HK_MRIQ && (C->site_mask[HK_MRIQ] >> MRIQ_PHIMAG_SITE0) != 0)
    bytes += sizeof(float4) * (size_t)std::max(1, ((const hk_mriq_args*)args)->n_k) * batch;
  return bytes;
}

hk_status hauberk_inject_campaign(int32_t bench_mode, const void* const args[3], const hk_ranges* const ranges[3],
                                  const hk_campaign* C, hk_outcome* d_records, int64_t* d_counts, int64_t* d_site_counts,
                                  void* stream) {
  if (!args || !ranges || !C || !d_counts || bench_mode < -1 || bench_mode > 2) return invalid("campaign: bad arguments");
  if (C->count < 0 || C->first < 0) return invalid("campaign: bad index range");
  if (C->count == 0) return HK_OK;
  // prepare only the benchmarks this index range touches
  const void* used_args[3] = {nullptr, nullptr, nullptr};
  for (int b = 0; b < 3; ++b) {
    const bool used = bench_mode == b || (bench_mode == -1 && C->count > (b - C->first % 3 + 3) % 3);
    if (used) {
      if (!args[b]) return invalid("campaign: args of a used benchmark are missing");
      used_args[b] = args[b];
    }
  }
  hk_campaign_session* S = nullptr;
  hk_status st = session_create(bench_mode, used_args, ranges, C, (cudaStream_t)stream, &S);
  if (st != HK_OK) return st;
  st = session_run(S, C->first, C->count, d_records, d_counts, d_site_counts);
  session_free(S);
  return st;
}

}  // extern "C"
