// Does a MUFU warp instruction with only some lanes active occupy the XU pipe for fewer cycles?
// (Decides whether partially filled warps can rebalance the MRI-Q single run.)
// Each warp runs 8 independent sin.approx chains; ACTIVE lanes per warp execute them.
#include <cstdio>
#include <cuda_runtime.h>
#define N_IT 32768
template <int ACTIVE>
__global__ void k(float* out, float seed, long long* cyc) {
  float a0 = seed + threadIdx.x * 1e-3f, a1 = a0 + 1.f, a2 = a0 + 2.f, a3 = a0 + 3.f;
  float a4 = a0 + 4.f, a5 = a0 + 5.f, a6 = a0 + 6.f, a7 = a0 + 7.f;
  const int on = (threadIdx.x & 31) < ACTIVE ? 1 : 0;
  long long t0 = clock64();
#pragma unroll 1
  for (int i = 0; i < N_IT; ++i) {
#define S(x) asm volatile("{ .reg .pred p; setp.ne.s32 p, %1, 0; @p sin.approx.ftz.f32 %0, %0; }" : "+f"(x) : "r"(on))
    S(a0); S(a1); S(a2); S(a3); S(a4); S(a5); S(a6); S(a7);
  }
  __syncwarp();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  out[blockIdx.x * blockDim.x + threadIdx.x] = a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7;
}
template <int A> void run(int sms) {
  const int blocks = sms * 2, threads = 1024;
  float* out; long long* cyc;
  cudaMalloc(&out, blocks * threads * 4); cudaMalloc(&cyc, blocks * 8);
  k<A><<<blocks, threads>>>(out, 0.5f, cyc); cudaDeviceSynchronize();
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0); k<A><<<blocks, threads>>>(out, 0.5f, cyc); cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  long long h[2048]; cudaMemcpy(h, cyc, blocks * 8, cudaMemcpyDeviceToHost);
  double avg = 0; for (int i = 0; i < blocks; ++i) avg += h[i]; avg /= blocks;
  // 64 warps per SM (2 CTAs x 32 warps), 16 per SMSP, N_IT*8 MUFU instructions each
  const double warp_instr_per_smsp = 16.0 * N_IT * 8;
  printf("{\"active_lanes\":%d,\"ms\":%.3f,\"cycles_per_warp_mufu_per_smsp\":%.3f}\n", A, ms, avg / warp_instr_per_smsp);
  cudaFree(out); cudaFree(cyc);
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  run<32>(sms); run<28>(sms); run<24>(sms); run<16>(sms); run<8>(sms); run<4>(sms); run<1>(sms); run<32>(sms);
  return 0;
}
