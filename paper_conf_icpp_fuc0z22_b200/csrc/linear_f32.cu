// linear_f32.cu -- fp32 SIMT linear layer C = epi(A . W^T + bias) (+ R): the fp32 parity
// path (toy config, 1e-4 bar).  TF32 tensor cores would miss 1e-4, so this stays on the
// FFMA pipe: 64x64 output tile per 256-thread CTA, 4x4 outputs per thread, K staged through
// shared memory in steps of 16.  Eq. (3) and the FFN linears.
#include <cmath>

#include "kernels.h"
#include "../../include/tcb_ops.h"

namespace tcb {
namespace k {
namespace {

constexpr int TM = 64, TN = 64, TK = 16;

__device__ __forceinline__ float apply_epi(float acc, int epi) {
  if (epi == TCB_EPI_BIAS_GELU) return 0.5f * acc * (1.f + erff(acc * 0.70710678118654752f));
  if (epi == TCB_EPI_BIAS_RELU) return fmaxf(acc, 0.f);
  return acc;
}

__global__ void __launch_bounds__(256)
linear_f32_kernel(int64_t M, int N, int K, const float* __restrict__ A,
                  const float* __restrict__ W, const float* __restrict__ bias,
                  const float* __restrict__ R, int epi, float* __restrict__ C) {
  __shared__ float sA[TK][TM + 4];
  __shared__ float sW[TK][TN + 4];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int64_t m0 = static_cast<int64_t>(blockIdx.y) * TM;
  const int n0 = blockIdx.x * TN;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += TK) {
    for (int i = threadIdx.x; i < TM * TK; i += 256) {
      const int r = i / TK, c = i % TK;
      const int64_t gm = m0 + r;
      const int gk = k0 + c;
      sA[c][r] = (gm < M && gk < K) ? A[gm * K + gk] : 0.f;
      const int gn = n0 + r;
      sW[c][r] = (gn < N && gk < K) ? W[static_cast<int64_t>(gn) * K + gk] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < TK; ++kk) {
      float a[4], w[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { a[i] = sA[kk][ty * 4 + i]; w[i] = sW[kk][tx * 4 + i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], w[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int64_t gm = m0 + ty * 4 + i;
    if (gm >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int gn = n0 + tx * 4 + j;
      if (gn >= N) continue;
      float v = apply_epi(acc[i][j] + bias[gn], epi);
      if (epi == TCB_EPI_BIAS_RESIDUAL) v += R[gm * N + gn];
      C[gm * N + gn] = v;
    }
  }
}

}  // namespace

cudaError_t launch_linear_f32(int64_t M, int N, int K, const float* A, const float* W,
                              const float* bias, const float* R, int epi, float* C,
                              cudaStream_t s) {
  if (M == 0) return cudaSuccess;
  dim3 grid((N + TN - 1) / TN, static_cast<unsigned>((M + TM - 1) / TM));
  linear_f32_kernel<<<grid, 256, 0, s>>>(M, N, K, A, W, bias, R, epi, C);
  return cudaGetLastError();
}

}  // namespace k
}  // namespace tcb
