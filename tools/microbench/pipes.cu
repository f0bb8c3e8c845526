// Pipe-throughput microbenchmark for the planning peaks:
// MUFU.RSQ, MUFU.SIN/COS, FFMA, IADD/LOP3 per SM per clock on the box's B200.
#include <cstdio>
#include <cuda_runtime.h>
#define N_IT 65536
template <int OP>
__global__ void k(float* out, float seed, long long* cyc) {
  float a0 = seed + threadIdx.x * 1e-3f, a1 = a0 + 1.f, a2 = a0 + 2.f, a3 = a0 + 3.f;
  float a4 = a0 + 4.f, a5 = a0 + 5.f, a6 = a0 + 6.f, a7 = a0 + 7.f;
  unsigned u0 = threadIdx.x, u1 = u0 + 1, u2 = u0 + 2, u3 = u0 + 3, u4 = u0+4, u5=u0+5, u6=u0+6, u7=u0+7;
  long long t0 = clock64();
  for (int i = 0; i < N_IT; ++i) {
#define R(x) asm volatile("rsqrt.approx.ftz.f32 %0, %0;" : "+f"(x))
#define S(x) asm volatile("sin.approx.ftz.f32 %0, %0;" : "+f"(x))
#define F(x) asm volatile("fma.rn.f32 %0, %0, %0, %0;" : "+f"(x))
#define I(x) asm volatile("add.u32 %0, %0, %1;" : "+r"(x) : "r"(x))
#define E(x) asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(x))
#define N(x) asm volatile("cvt.rni.f32.f32 %0, %0;" : "+f"(x))
    if (OP == 0) { R(a0); R(a1); R(a2); R(a3); R(a4); R(a5); R(a6); R(a7); }
    if (OP == 1) { S(a0); S(a1); S(a2); S(a3); S(a4); S(a5); S(a6); S(a7); }
    if (OP == 2) { F(a0); F(a1); F(a2); F(a3); F(a4); F(a5); F(a6); F(a7); }
    if (OP == 3) { I(u0); I(u1); I(u2); I(u3); I(u4); I(u5); I(u6); I(u7); }
    if (OP == 4) { E(a0); E(a1); E(a2); E(a3); E(a4); E(a5); E(a6); E(a7); }
    if (OP == 5) { R(a0); F(a1); F(a2); F(a3); R(a4); F(a5); F(a6); F(a7); }
    if (OP == 6) { R(a0); R(a1); I(u2); I(u3); R(a4); R(a5); I(u6); I(u7); }
    if (OP == 7) { N(a0); N(a1); N(a2); N(a3); N(a4); N(a5); N(a6); N(a7); }
    if (OP == 8) { S(a0); N(a1); N(a2); N(a3); S(a4); N(a5); N(a6); N(a7); }
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  out[blockIdx.x * blockDim.x + threadIdx.x] = a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 + (float)(u0 ^ u1 ^ u2 ^ u3 ^ u4 ^ u5 ^ u6 ^ u7);
}
template <int OP> void run(const char* name, int sms) {
  int blocks = sms * 2, threads = 1024;
  float* out; long long* cyc; cudaMalloc(&out, blocks * threads * 4); cudaMalloc(&cyc, blocks * 8);
  k<OP><<<blocks, threads>>>(out, 0.5f, cyc); cudaDeviceSynchronize();
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0); k<OP><<<blocks, threads>>>(out, 0.5f, cyc); cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  long long h[1024]; cudaMemcpy(h, cyc, blocks * 8, cudaMemcpyDeviceToHost);
  double avg = 0; for (int i = 0; i < blocks; ++i) avg += h[i]; avg /= blocks;
  double ops = (double)blocks * threads * N_IT * 8;
  // per-SM lanes per clock: two CTAs of 1024 threads co-resident per SM
  double per_sm_clk = (2.0 * threads * N_IT * 8) / avg;
  printf("{\"op\":\"%s\",\"ms\":%.4f,\"ops_per_s\":%.4e,\"lanes_per_sm_per_clk\":%.2f,\"cycles\":%.0f}\n", name, ms, ops / (ms * 1e-3), per_sm_clk, avg);
  cudaFree(out); cudaFree(cyc);
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("{\"sms\":%d,\"clock_khz\":%d}\n", sms, clk);
  run<0>("rsqrt", sms); run<1>("sin", sms); run<2>("ffma", sms); run<3>("iadd", sms); run<4>("ex2", sms);
  run<0>("rsqrt", sms); run<1>("sin", sms); run<2>("ffma", sms); run<5>("mix_2rsq_6ffma", sms); run<6>("mix_4rsq_4iadd", sms);
  run<7>("frnd", sms); run<8>("mix_2sin_6frnd", sms);
  return 0;
}
