// attention.cu -- segment-masked self-attention over packed rows (sm_100a).
//
// Eq. (5)-(6): Att_CB(Q,K,V) = softmax(QK^T/sqrt(d) + M) V with M = 0 on the
// diagonal blocks Q_i K_i^T and -inf elsewhere.  Only the diagonal blocks are useful
// (Eq. (7)), and the paper notes that computing the masked blocks
// anyway wastes memory and compute (§4.2).  This kernel therefore never
// materialises M or the score matrix: a CTA owns 64 query slots of one head; each of its 4
// warps owns 16 query rows and evaluates only the 16-key sub-blocks that intersect the key
// interval of its own rows' requests, so cross-request tiles are skipped outright.  Inside a
// visited sub-block, pairs from different requests get exactly -inf before the softmax
// (R11), i.e. probability 0.  Softmax is the online (running max / running sum) form in the
// exp2 domain (R23), fp32 throughout; P is rounded to bf16 only as the A operand of P.V.
//
// The contraction is tiny per sub-block (16x16x64 and 16x64x16) and the kernel is HBM /
// MUFU bound for the paper's request lengths, so it uses warp-level
// mma.sync.m16n8k16 (bf16 in, fp32 accumulate) with K/V staged in swizzled shared memory by
// cp.async (double-buffered 64-key chunks).  The fp32 variant below is the 1e-4 parity path.
#include <cuda_bf16.h>

#include <cmath>

#include "kernels.h"

namespace tcb {
namespace k {
namespace {

constexpr int QB = 64;      // query slots per CTA
constexpr int KC = 64;      // keys per staged chunk
constexpr int DH = 64;      // head dim of the bf16 path
constexpr int kThreads = 128;

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// [rows][64] bf16 tile, 16-byte chunk c of row r stored at chunk (c ^ (r & 7)).
__device__ __forceinline__ int swz(int row, int chunk) { return row * 64 + ((chunk ^ (row & 7)) << 3); }

__device__ __forceinline__ void cp_async16(void* dst, const void* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "r"(valid ? 16 : 0)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2,
                                        uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& r0, uint32_t& r1,
                                          uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void mma_bf16(float (&c)[4], const uint32_t (&a)[4], uint32_t b0,
                                         uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, "
      "{%8,%9}, {%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t pack_bf16(float lo, float hi) {
  __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&h);
}

__global__ void __launch_bounds__(kThreads)
attn_bf16_kernel(const __nv_bfloat16* __restrict__ qkv, const int32_t* __restrict__ seg_ids,
                 const int4* __restrict__ segtab, __nv_bfloat16* __restrict__ O,
                 int64_t num_slots, int d_model, float scale_log2) {
  __shared__ alignas(128) __nv_bfloat16 sQ[QB * DH];
  __shared__ alignas(128) __nv_bfloat16 sK[2][KC * DH];
  __shared__ alignas(128) __nv_bfloat16 sV[2][KC * DH];
  __shared__ alignas(16) int sSegK[2][KC];
  __shared__ int sLo[4], sHi[4];

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int h = blockIdx.y;
  const int64_t q0 = static_cast<int64_t>(blockIdx.x) * QB;
  const int64_t ld = 3 * static_cast<int64_t>(d_model);

  // --- 1. segments of this warp's 16 query rows and their key interval ------------------
  const int g = lane >> 2, t4 = lane & 3;
  const int64_t rowA = q0 + warp * 16 + g, rowB = rowA + 8;
  const int segA = rowA < num_slots ? __ldg(&seg_ids[rowA]) : -1;
  const int segB = rowB < num_slots ? __ldg(&seg_ids[rowB]) : -1;
  int lo = INT_MAX, hi = -1;
  if (segA >= 0) { const int4 r = __ldg(&segtab[1 + segA]); lo = min(lo, r.x); hi = max(hi, r.x + r.y); }
  if (segB >= 0) { const int4 r = __ldg(&segtab[1 + segB]); lo = min(lo, r.x); hi = max(hi, r.x + r.y); }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
  }
  const int wlo = lo, whi = hi;  // empty if whi < 0
  if (lane == 0) { sLo[warp] = wlo; sHi[warp] = whi; }

  // --- 2. stage Q (64 rows x 64 dims of head h) -----------------------------------------
  for (int i = threadIdx.x; i < QB * 8; i += kThreads) {
    const int r = i >> 3, c = i & 7;
    const int64_t row = q0 + r;
    const bool ok = row < num_slots;
    cp_async16(&sQ[swz(r, c)], qkv + (ok ? row : 0) * ld + h * DH + c * 8, ok);
  }
  cp_async_commit();
  __syncthreads();
  int clo = INT_MAX, chi = -1;
#pragma unroll
  for (int w = 0; w < 4; ++w) {
    if (sHi[w] >= 0) { clo = min(clo, sLo[w]); chi = max(chi, sHi[w]); }
  }

  auto load_chunk = [&](int buf, int kbase) {
    for (int i = threadIdx.x; i < KC * 8; i += kThreads) {
      const int r = i >> 3, c = i & 7;
      const int64_t key = static_cast<int64_t>(kbase) + r;
      const bool ok = key < chi;
      const __nv_bfloat16* src = qkv + (ok ? key : 0) * ld + d_model + h * DH + c * 8;
      cp_async16(&sK[buf][swz(r, c)], src, ok);
      cp_async16(&sV[buf][swz(r, c)], src + d_model, ok);
    }
    if (threadIdx.x < KC) {
      const int64_t key = static_cast<int64_t>(kbase) + threadIdx.x;
      sSegK[buf][threadIdx.x] = key < chi ? __ldg(&seg_ids[key]) : -2;
    }
  };

  float acc[8][4];
#pragma unroll
  for (int j = 0; j < 8; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
  float mA = -INFINITY, mB = -INFINITY, lA = 0.f, lB = 0.f;

  if (chi >= 0) {
    const int nchunks = (chi - clo + KC - 1) / KC;
    load_chunk(0, clo);
    cp_async_commit();
    // Q fragments (A operand, 16 rows x 64 dims = 4 k-steps)
    cp_async_wait<1>();
    __syncthreads();
    uint32_t qf[4][4];
#pragma unroll
    for (int ks = 0; ks < 4; ++ks) {
      const int r = warp * 16 + (lane & 15);
      const int c = 2 * ks + (lane >> 4);
      ldsm_x4(smem_u32(&sQ[swz(r, c)]), qf[ks][0], qf[ks][1], qf[ks][2], qf[ks][3]);
    }
    for (int ch = 0; ch < nchunks; ++ch) {
      const int buf = ch & 1;
      const int kbase = clo + ch * KC;
      if (ch + 1 < nchunks) load_chunk(buf ^ 1, kbase + KC);
      cp_async_commit();
      cp_async_wait<1>();
      __syncthreads();
      // sub-blocks [sb_lo, sb_hi) of this chunk intersect the warp's key interval; the
      // others are cross-request (or beyond the row) and are skipped outright
      const int lim = min(whi, chi);
      const int sb_lo = wlo > kbase ? (wlo - kbase) >> 4 : 0;
      const int sb_hi = lim > kbase ? min(KC / 16, (lim - kbase + 15) >> 4) : 0;
      if (whi >= 0 && sb_lo < sb_hi) {
        // S = Q K^T for 16 queries x up to 64 keys
        float s[KC / 16][2][4];
#pragma unroll
        for (int sb = 0; sb < KC / 16; ++sb) {
#pragma unroll
          for (int j = 0; j < 2; ++j) s[sb][j][0] = s[sb][j][1] = s[sb][j][2] = s[sb][j][3] = 0.f;
          if (sb < sb_lo || sb >= sb_hi) continue;   // warp-uniform
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            const int mi = lane >> 3;
            const int r = sb * 16 + (mi >> 1) * 8 + (lane & 7);
            const int c = 2 * ks + (mi & 1);
            uint32_t k0, k1, k2, k3;
            ldsm_x4(smem_u32(&sK[buf][swz(r, c)]), k0, k1, k2, k3);
            mma_bf16(s[sb][0], qf[ks], k0, k1);
            mma_bf16(s[sb][1], qf[ks], k2, k3);
          }
        }
        // mask M of Eq. (6) (pairs of different requests -> -inf) + scale to log2 domain
        float bmA = -INFINITY, bmB = -INFINITY;
#pragma unroll
        for (int sb = 0; sb < KC / 16; ++sb) {
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            const int kl = sb * 16 + j * 8 + 2 * t4;
            const int2 sk = *reinterpret_cast<const int2*>(&sSegK[buf][kl]);
            const bool live = sb >= sb_lo && sb < sb_hi;
            s[sb][j][0] = (live && sk.x == segA) ? s[sb][j][0] * scale_log2 : -INFINITY;
            s[sb][j][1] = (live && sk.y == segA) ? s[sb][j][1] * scale_log2 : -INFINITY;
            s[sb][j][2] = (live && sk.x == segB) ? s[sb][j][2] * scale_log2 : -INFINITY;
            s[sb][j][3] = (live && sk.y == segB) ? s[sb][j][3] * scale_log2 : -INFINITY;
            bmA = fmaxf(bmA, fmaxf(s[sb][j][0], s[sb][j][1]));
            bmB = fmaxf(bmB, fmaxf(s[sb][j][2], s[sb][j][3]));
          }
        }
        bmA = fmaxf(bmA, __shfl_xor_sync(0xffffffffu, bmA, 1));
        bmA = fmaxf(bmA, __shfl_xor_sync(0xffffffffu, bmA, 2));
        bmB = fmaxf(bmB, __shfl_xor_sync(0xffffffffu, bmB, 1));
        bmB = fmaxf(bmB, __shfl_xor_sync(0xffffffffu, bmB, 2));
        const float nmA = fmaxf(mA, bmA), nmB = fmaxf(mB, bmB);
        const float uA = nmA == -INFINITY ? 0.f : nmA;
        const float uB = nmB == -INFINITY ? 0.f : nmB;
        if (nmA != mA || nmB != mB) {          // rescale only when a running max moved
          const float aA = exp2f(mA - uA), aB = exp2f(mB - uB);
          lA *= aA;
          lB *= aB;
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            acc[j][0] *= aA; acc[j][1] *= aA;
            acc[j][2] *= aB; acc[j][3] *= aB;
          }
          mA = nmA;
          mB = nmB;
        }
#pragma unroll
        for (int sb = 0; sb < KC / 16; ++sb) {
          if (sb < sb_lo || sb >= sb_hi) continue;   // warp-uniform
          float p[2][4];
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            p[j][0] = exp2f(s[sb][j][0] - uA);
            p[j][1] = exp2f(s[sb][j][1] - uA);
            p[j][2] = exp2f(s[sb][j][2] - uB);
            p[j][3] = exp2f(s[sb][j][3] - uB);
            lA += p[j][0] + p[j][1];
            lB += p[j][2] + p[j][3];
          }
          const uint32_t pa[4] = {pack_bf16(p[0][0], p[0][1]), pack_bf16(p[0][2], p[0][3]),
                                  pack_bf16(p[1][0], p[1][1]), pack_bf16(p[1][2], p[1][3])};
          // O += P V  (16 keys x 64 dims)
#pragma unroll
          for (int jj = 0; jj < 4; ++jj) {
            const int mi = lane >> 3;
            const int r = sb * 16 + (mi & 1) * 8 + (lane & 7);
            const int c = 2 * jj + (mi >> 1);
            uint32_t v0, v1, v2, v3;
            ldsm_x4_t(smem_u32(&sV[buf][swz(r, c)]), v0, v1, v2, v3);
            mma_bf16(acc[2 * jj], pa, v0, v1);
            mma_bf16(acc[2 * jj + 1], pa, v2, v3);
          }
        }
      }
      __syncthreads();
    }
  }
  cp_async_wait<0>();
  // --- 3. normalise and store (pad / empty rows -> 0) ------------------------------------
  lA += __shfl_xor_sync(0xffffffffu, lA, 1);
  lA += __shfl_xor_sync(0xffffffffu, lA, 2);
  lB += __shfl_xor_sync(0xffffffffu, lB, 1);
  lB += __shfl_xor_sync(0xffffffffu, lB, 2);
  const float iA = (segA >= 0 && lA > 0.f) ? 1.f / lA : 0.f;
  const float iB = (segB >= 0 && lB > 0.f) ? 1.f / lB : 0.f;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const int col = h * DH + j * 8 + 2 * t4;
    if (rowA < num_slots)
      *reinterpret_cast<uint32_t*>(O + rowA * d_model + col) = pack_bf16(acc[j][0] * iA, acc[j][1] * iA);
    if (rowB < num_slots)
      *reinterpret_cast<uint32_t*>(O + rowB * d_model + col) = pack_bf16(acc[j][2] * iB, acc[j][3] * iB);
  }
}

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

cudaError_t launch_attention_bf16(int64_t num_slots, int d_model, int num_heads,
                                  const void* qkv, const int32_t* seg_ids, const int4* segtab,
                                  void* O, cudaStream_t s) {
  if (num_slots == 0) return cudaSuccess;
  dim3 grid(static_cast<unsigned>((num_slots + QB - 1) / QB), num_heads);
  const float scale_log2 = 1.4426950408889634f / sqrtf(static_cast<float>(DH));
  attn_bf16_kernel<<<grid, kThreads, 0, s>>>(static_cast<const __nv_bfloat16*>(qkv), seg_ids,
                                             segtab, static_cast<__nv_bfloat16*>(O), num_slots,
                                             d_model, scale_log2);
  return cudaGetLastError();
}

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
