// attention.cu -- segment-masked self-attention over packed rows, fp32 parity path (C1 toy).
//
// Eq. (5)-(6): Att_CB(Q,K,V) = softmax(QK^T/sqrt(d) + M) V with M = 0 on the
// diagonal blocks Q_i K_i^T and -inf elsewhere.  Only the diagonal blocks are useful
// (Eq. (7)), so a query only ever visits the keys of its own request
// (the entries M leaves finite; masked pairs contribute exactly 0, R11).  One warp per
// (query slot, head), online softmax in fp32 -- the 1e-4 bar of R21 (TF32 tensor cores would
// miss it).  The bf16 path is the tcgen05 kernel of attention_tc.cu.
#include <cmath>
#include <cstdio>

#include "kernels.h"

namespace tcb {
namespace k {
namespace {

// fp32 path: one warp per (query slot, head); keys restricted to the query's own request
// (the only entries M leaves finite); online softmax in fp32.
__global__ void __launch_bounds__(128)
attn_f32_kernel(const float* __restrict__ qkv, const int32_t* __restrict__ seg_ids,
                const int4* __restrict__ segtab, float* __restrict__ O, int64_t num_slots,
                int d_model, int dh, float scale) {
  const int lane = threadIdx.x & 31;
  const int64_t slot = static_cast<int64_t>(blockIdx.x) * 4 + (threadIdx.x >> 5);
  const int h = blockIdx.y;
  if (slot >= num_slots) return;
  const int64_t ld = 3 * static_cast<int64_t>(d_model);
  float* o = O + slot * d_model + h * dh;
  const int seg = __ldg(&seg_ids[slot]);
  if (seg < 0) {
    for (int c = lane; c < dh; c += 32) o[c] = 0.f;
    return;
  }
  const int4 rec = __ldg(&segtab[1 + seg]);
  const float* q = qkv + slot * ld + h * dh;
  const float q0 = lane < dh ? q[lane] : 0.f;
  const float q1 = lane + 32 < dh ? q[lane + 32] : 0.f;
  float m = -INFINITY, l = 0.f, a0 = 0.f, a1 = 0.f;
  for (int j = rec.x; j < rec.x + rec.y; ++j) {
    const float* kr = qkv + static_cast<int64_t>(j) * ld + d_model + h * dh;
    float dot = (lane < dh ? q0 * kr[lane] : 0.f) + (lane + 32 < dh ? q1 * kr[lane + 32] : 0.f);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) dot += __shfl_xor_sync(0xffffffffu, dot, off);
    const float s = dot * scale;
    const float nm = fmaxf(m, s);
    const float alpha = expf(m - nm);
    const float p = expf(s - nm);
    l = l * alpha + p;
    const float* vr = kr + d_model;
    a0 = a0 * alpha + (lane < dh ? p * vr[lane] : 0.f);
    a1 = a1 * alpha + (lane + 32 < dh ? p * vr[lane + 32] : 0.f);
    m = nm;
  }
  if (lane < dh) o[lane] = a0 / l;
  if (lane + 32 < dh) o[lane + 32] = a1 / l;
}

}  // namespace

cudaError_t launch_attention_f32(int64_t num_slots, int d_model, int num_heads,
                                 const float* qkv, const int32_t* seg_ids, const int4* segtab,
                                 float* O, cudaStream_t s) {
  if (num_slots == 0) return cudaSuccess;
  const int dh = d_model / num_heads;
  dim3 grid(static_cast<unsigned>((num_slots + 3) / 4), num_heads);
  attn_f32_kernel<<<grid, 128, 0, s>>>(qkv, seg_ids, segtab, O, num_slots, d_model, dh,
                                       1.f / sqrtf(static_cast<float>(dh)));
  return cudaGetLastError();
}

}  // namespace k
}  // namespace tcb
