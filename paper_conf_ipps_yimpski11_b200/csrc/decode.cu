// decode.cu — injection decode on the device (DESIGN R14/R15) and a counting sort by
// (benchmark, site kind), feeding the replay accelerator without a host round trip.
//
// The rule is the one host.cpp's decode_one and the oracle's cat_decode implement: SplitMix64
// outputs 8n+1..8n+3 pick the site (over the enabled catalogue), the (thread, instance) pair (over
// the site's dynamic instances in thread-major order) and the bit; multi-bit masks extend the
// single-bit draw by a partial Fisher-Yates shuffle fed by the stream seed ^ 0xD1B54A32D192ED03.
#include "hk_internal.h"

namespace hk {

__device__ __forceinline__ uint64_t d_splitmix(uint64_t seed, uint64_t m) {
  uint64_t z = seed + (m + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t d_below(uint64_t r, uint64_t m) { return __umul64hi(r, m); }

struct DecodeParams {
  DevCatalog cat[3];
  uint64_t seed;
  int64_t first, count;
  int32_t bench_mode, nbits, hang;
  FaultRec* tmp;
  uint8_t* key;       // bench * 32 + kind
  uint32_t* hist;     // [96]
};

__global__ void decode_kernel(const DecodeParams P) {
  const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (q >= P.count) return;
  const int64_t n = P.first + q;
  const int b = P.bench_mode >= 0 ? P.bench_mode : (int)(n % 3);
  const DevCatalog& K = P.cat[b];
  const uint64_t r1 = d_splitmix(P.seed, 8 * (uint64_t)n + 1);
  const uint64_t r2 = d_splitmix(P.seed, 8 * (uint64_t)n + 2);
  const uint64_t r3 = d_splitmix(P.seed, 8 * (uint64_t)n + 3);
  const int s = K.en[d_below(r1, (uint64_t)K.nen)];
  FaultRec f;
  f.index = n;
  f.site = s;
  f.sub = K.sub[s];
  f.real = 0;
  f.hang = P.hang;
  if (K.is_nl[s]) {
    const int64_t nt = (b == HK_MRIQ && s >= MRIQ_PHIMAG_SITE0) ? K.nk : K.nthr;
    f.thread = (int64_t)d_below(r2, (uint64_t)nt);
    f.inst = 0;
  } else {
    const int64_t u = (int64_t)d_below(r2, (uint64_t)K.total_trips);
    if (!K.prefix) {
      f.thread = u / K.uniform_trips;
      f.inst = u % K.uniform_trips;
    } else {  // largest g with prefix[g] <= u (prefix[0] = 0 <= u < prefix[nthr])
      int64_t lo = 0, hi = K.nthr;
      while (hi - lo > 1) {
        const int64_t mid = lo + (hi - lo) / 2;
        if (K.prefix[mid] <= u) lo = mid;
        else hi = mid;
      }
      f.thread = lo;
      f.inst = u - K.prefix[lo];
    }
  }
  const int w = K.width[s];
  if (P.nbits <= 1) {
    f.mask = 1ull << d_below(r3, (uint64_t)w);
  } else {
    const int k = min(P.nbits, w);
    uint8_t perm[64];
    for (int i = 0; i < w; ++i) perm[i] = (uint8_t)i;
    uint64_t mask = 0;
    for (int t = 0; t < k; ++t) {
      const uint64_t r = t == 0 ? r3 : d_splitmix(P.seed ^ 0xD1B54A32D192ED03ull, 16 * (uint64_t)n + (uint64_t)t);
      const int j = t + (int)d_below(r, (uint64_t)(w - t));
      const uint8_t tmp = perm[t];
      perm[t] = perm[j];
      perm[j] = tmp;
      mask |= 1ull << perm[t];
    }
    f.mask = mask;
  }
  const uint8_t key = (uint8_t)(b * 32 + K.kind[s]);
  P.tmp[q] = f;
  P.key[q] = key;
  atomicAdd(P.hist + key, 1u);
}

__global__ void decode_offsets_kernel(const uint32_t* hist, uint32_t* cursor) {
  if (threadIdx.x == 0) {
    uint32_t acc = 0;
    for (int k = 0; k < 96; ++k) { cursor[k] = acc; acc += hist[k]; }
  }
}

__global__ void decode_scatter_kernel(const FaultRec* tmp, const uint8_t* key, uint32_t* cursor, FaultRec* sorted,
                                      int64_t count) {
  const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (q >= count) return;
  const uint32_t pos = atomicAdd(cursor + key[q], 1u);
  sorted[pos] = tmp[q];
}

// ws: workspace of decode_ws_bytes(count); the sorted records start at ws (count FaultRec).
size_t decode_ws_bytes(int64_t count) {
  const size_t c = (size_t)count;
  return sizeof(FaultRec) * c * 2 + c + 16 + 2 * 96 * sizeof(uint32_t) + 64;
}

cudaError_t decode_sort_launch(const DevCatalog cat[3], uint64_t seed, int64_t first, int64_t count, int32_t bench_mode,
                               int32_t nbits, int32_t hang, void* ws, FaultRec** sorted_out, cudaStream_t s) {
  char* p = reinterpret_cast<char*>(ws);
  FaultRec* sorted = reinterpret_cast<FaultRec*>(p);
  FaultRec* tmp = sorted + count;
  uint8_t* key = reinterpret_cast<uint8_t*>(tmp + count);
  uint32_t* hist = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(key) + ((count + 15) / 16) * 16);
  uint32_t* cursor = hist + 96;
  cudaError_t e = cudaMemsetAsync(hist, 0, 96 * sizeof(uint32_t), s);
  if (e != cudaSuccess) return e;
  DecodeParams P{};
  for (int b = 0; b < 3; ++b) P.cat[b] = cat[b];
  P.seed = seed; P.first = first; P.count = count; P.bench_mode = bench_mode; P.nbits = nbits; P.hang = hang;
  P.tmp = tmp; P.key = key; P.hist = hist;
  const unsigned g = (unsigned)((count + 255) / 256);
  decode_kernel<<<g, 256, 0, s>>>(P);
  count_launch();
  decode_offsets_kernel<<<1, 32, 0, s>>>(hist, cursor);
  count_launch();
  decode_scatter_kernel<<<g, 256, 0, s>>>(tmp, key, cursor, sorted, count);
  count_launch();
  *sorted_out = sorted;
  return cudaGetLastError();
}

}  // namespace hk
