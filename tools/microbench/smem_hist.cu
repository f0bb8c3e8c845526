// Lane-private shared-memory histogram increments: RMW (LDS+IADD+STS) vs red.shared.add (ATOMS/RED).
#include <cstdio>
#include <cuda_runtime.h>
template <int MODE>
__global__ void k(unsigned* out, int iters, unsigned seed) {
  __shared__ unsigned H[8][32][32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 8 * 32 * 32; i += blockDim.x) (&H[0][0][0])[i] = 0;
  __syncthreads();
  unsigned x = seed ^ (threadIdx.x * 2654435761u);
  unsigned* Hw = &H[warp][0][lane];
#pragma unroll 4
  for (int i = 0; i < iters; ++i) {
    x = x * 1664525u + 1013904223u;
    const unsigned bin = (x >> 27) % 22;
    if (MODE == 0) Hw[bin * 32] += 1u;
    else atomicAdd(&Hw[bin * 32], 1u);
  }
  __syncthreads();
  unsigned s = 0;
  for (int b = 0; b < 22; ++b) s += H[warp][b][lane];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int MODE> void run(const char* name) {
  int blocks = 148 * 4, threads = 256, iters = 4096;
  unsigned* out; cudaMalloc(&out, blocks * threads * 4);
  k<MODE><<<blocks, threads>>>(out, iters, 1); cudaDeviceSynchronize();
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a); k<MODE><<<blocks, threads>>>(out, iters, 2); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  double warp_updates = (double)blocks * threads / 32 * iters;
  printf("{\"mode\":\"%s\",\"ms\":%.4f,\"warp_updates_per_sm_per_ns\":%.4f}\n", name, ms, warp_updates / 148 / (ms * 1e6));
}
int main() { run<0>("rmw"); run<1>("red_shared"); run<0>("rmw"); run<1>("red_shared"); return 0; }
