// Exhaustive error of the FAST path's MUFU sin / cos (sin.approx.ftz.f32 / cos.approx.ftz.f32, DESIGN
// R20) over every binary32 input in [-pi_f, pi_f] (the domain the MRI-Q FAST kernels reach: |r| <= 0.5,
// ang = r * 2pi_f), against double-precision sin / cos.  Prints the maximum absolute error of each
// and its log2 — the measured counterpart of the documented 2^-20.9 that R21 / R22 assume.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o mufu_err mufu_err.cu && ./mufu_err
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>

__device__ unsigned long long g_max[2];  // bit patterns of the max errors (non-negative doubles order as u64)

__global__ void mufu_err_kernel(uint32_t hi_bits) {
  // every non-negative bit pattern 0 .. hi_bits, both signs
  const uint64_t n = (uint64_t)hi_bits + 1;
  double ms = 0.0, mc = 0.0;
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < 2 * n; k += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t b = (uint32_t)(k % n) | (k >= n ? 0x80000000u : 0u);
    const float x = __uint_as_float(b);
    float s, c;
    asm("sin.approx.ftz.f32 %0, %1;" : "=f"(s) : "f"(x));
    asm("cos.approx.ftz.f32 %0, %1;" : "=f"(c) : "f"(x));
    // ftz: a denormal input is read as +-0
    const double xd = (fabsf(x) < 1.17549435e-38f) ? 0.0 : (double)x;
    ms = fmax(ms, fabs((double)s - sin(xd)));
    mc = fmax(mc, fabs((double)c - cos(xd)));
  }
  for (int o = 16; o; o >>= 1) {
    ms = fmax(ms, __shfl_xor_sync(0xffffffffu, ms, o));
    mc = fmax(mc, __shfl_xor_sync(0xffffffffu, mc, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMax(&g_max[0], (unsigned long long)__double_as_longlong(ms));
    atomicMax(&g_max[1], (unsigned long long)__double_as_longlong(mc));
  }
}

int main() {
  const float pi_f = 3.14159274f;  // fl(pi), the largest |ang| of the FAST domain
  uint32_t hb;
  memcpy(&hb, &pi_f, 4);
  unsigned long long z[2] = {0, 0};
  cudaMemcpyToSymbol(g_max, z, sizeof z);
  mufu_err_kernel<<<148 * 16, 256>>>(hb);
  if (cudaDeviceSynchronize() != cudaSuccess) { printf("kernel failed\n"); return 1; }
  unsigned long long r[2];
  cudaMemcpyFromSymbol(r, g_max, sizeof r);
  double e[2];
  memcpy(&e[0], &r[0], 8);
  memcpy(&e[1], &r[1], 8);
  printf("{\"domain\": \"all binary32 x with |x| <= fl(pi) (%llu inputs)\", \"sin_max_abs_err\": %.6e, \"sin_log2\": %.3f, "
         "\"cos_max_abs_err\": %.6e, \"cos_log2\": %.3f, \"documented\": \"2^-20.9 = %.6e\"}\n",
         2ull * ((unsigned long long)hb + 1), e[0], log2(e[0]), e[1], log2(e[1]), exp2(-20.9));
  return 0;
}
