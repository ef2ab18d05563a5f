// Microbenchmark: MUFU ex2.approx throughput per SM per clock on this GPU (and FFMA for scale).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_ex2(float* out, int iters, float seed) {
  float a[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) a[i] = seed * (threadIdx.x + i) * 1e-3f - 3.f;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      float y;
      asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(a[i]));
      a[i] = y - 3.f;
    }
  }
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_ffma(float* out, int iters, float seed) {
  float a[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) a[i] = seed * (threadIdx.x + i);
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], 0.999f, 0.001f);
  }
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
  int sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  float* out;
  cudaMalloc(&out, sizeof(float) * sms * 8 * 1024);
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  const int iters = 4096;
  for (int warps : {4, 8, 16, 32}) {
    for (int which = 0; which < 2; ++which) {
      auto run = [&]() {
        if (which == 0) k_ex2<<<sms * 2, warps * 16>>>(out, iters, 1.f);
        else k_ffma<<<sms * 2, warps * 16>>>(out, iters, 1.f);
      };
      run(); cudaDeviceSynchronize();
      cudaEventRecord(a); run(); cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b);
      double ops = double(sms) * 2 * warps * 16 * iters * 16;
      double per_sm_clk = ops / (ms * 1e-3) / sms / (clk * 1e3);
      printf("%s warps/SM=%d: %.1f ops/clk/SM (at the %d MHz nominal clock)\n", which ? "ffma" : "ex2 ",
             warps, per_sm_clk, clk / 1000);
    }
  }
  return 0;
}
