// elementwise.cu -- HBM-bound kernels of the ConcatBatching path (sm_100a):
//   pack_embed : gather token embeddings, add the separate positional encoding (positions
//                restart at each request, §4.1.1, Eq. (1)-(2) P:329-333), write
//                the per-slot segment metadata; optional BERT type-0 + LayerNorm (R5).
//   layernorm  : warp-per-row two-pass LayerNorm (post-LN encoder, R10).
//   unpack     : scatter the rows back per request (Concat of Eq. (8)).
//   pe_table   : the sinusoidal table PE[pos, dim] (Eq. (1)-(2); R1 variant flag).
// One warp owns one slot / row; each lane moves 16-byte vectors so a warp touches whole
// 512-byte spans (coalesced); rows are kept in registers between the reduction passes.
#include <cuda_bf16.h>

#include <cmath>
#include <type_traits>

#include "kernels.h"

namespace tcb {
namespace k {
namespace {

constexpr int kWarpsPerBlock = 8;

template <typename T> struct Vec;
template <> struct Vec<float> {
  static constexpr int N = 4;
  __device__ static void load(const float* p, float* v) {
    float4 x = *reinterpret_cast<const float4*>(p);
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
  }
  __device__ static void store(float* p, const float* v) {
    *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
  }
};
template <> struct Vec<__nv_bfloat16> {
  static constexpr int N = 8;
  __device__ static void load(const __nv_bfloat16* p, float* v) {
    uint4 x = *reinterpret_cast<const uint4*>(p);
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&x);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      float2 f = __bfloat1622float2(h[i]);
      v[2 * i] = f.x; v[2 * i + 1] = f.y;
    }
  }
  __device__ static void store(__nv_bfloat16* p, const float* v) {
    uint4 x;
    __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&x);
#pragma unroll
    for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
    *reinterpret_cast<uint4*>(p) = x;
  }
};

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// One CTA per (batch row, 64-slot chunk of it).  The row's segment records (row_first[] of
// the device segment table gives them in O(1)) are staged in shared memory; each warp then
// owns slots j = chunk*64 + warp, +8, ... and finds its segment by a binary search in smem.
#ifndef TCB_ROW_CHUNK
#define TCB_ROW_CHUNK 16
#endif
constexpr int kRowChunk = TCB_ROW_CHUNK;   // slots per CTA (64 measured slower: fewer CTAs in flight)
static_assert(kRowChunk <= kWarpsPerBlock * 32, "one metadata thread per slot of a chunk");
template <typename T, int NV>
__global__ void __launch_bounds__(kWarpsPerBlock * 32) pack_embed_kernel(EmbedArgs a) {
  constexpr int V = Vec<T>::N;
  extern __shared__ int4 row_recs[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int row = blockIdx.x;
  pdl_wait();
  pdl_trigger();
  const int S = a.segtab[0].x;
  const int* row_first = reinterpret_cast<const int*>(a.segtab + 1 + S);
  const int f = __ldg(&row_first[row]);
  const int nseg = __ldg(&row_first[row + 1]) - f;
  for (int i = threadIdx.x; i < nseg; i += blockDim.x) row_recs[i] = __ldg(&a.segtab[1 + f + i]);
  // per-column vectors shared by every slot (BERT type-0 embedding, embedding LN) -> smem
  float* s_type = reinterpret_cast<float*>(row_recs + a.row_len);
  float* s_g = s_type + a.d;
  float* s_b = s_g + a.d;
  if (a.type_emb || a.ln_g) {
    for (int i = threadIdx.x; i < a.d; i += blockDim.x) {
      if (a.type_emb) s_type[i] = __ldg(&a.type_emb[i]);
      if (a.ln_g) { s_g[i] = __ldg(&a.ln_g[i]); s_b[i] = __ldg(&a.ln_b[i]); }
    }
  }
  __syncthreads();
  const int d = a.d;
  const int nvec = d / V;
  const int64_t row0 = static_cast<int64_t>(row) * a.row_len;
  const int jc0 = static_cast<int>(blockIdx.y) * kRowChunk;
  const int j_end = min(a.row_len, jc0 + kRowChunk);
  // one thread per slot of the chunk resolves (segment, position, token id) -- every id load
  // of the chunk in flight together -- and writes the slot metadata coalesced; the warps then
  // wait on only the embedding-row load per slot
  __shared__ int2 s_meta[kRowChunk];   // (position, token id); position -1 at pad
  if (jc0 + static_cast<int>(threadIdx.x) < j_end) {
    const int64_t slot = row0 + jc0 + threadIdx.x;
    int lo = 0, hi = nseg - 1, k = -1;   // last record with start <= slot
    while (lo <= hi) {
      const int mid = (lo + hi) >> 1;
      if (row_recs[mid].x <= slot) { k = mid; lo = mid + 1; } else { hi = mid - 1; }
    }
    int seg = -1, pos = -1, id = 0;      // pad slot: segment -1, position -1 (R12)
    if (k >= 0 && slot < row_recs[k].x + row_recs[k].y) {
      seg = f + k;
      pos = static_cast<int>(slot - row_recs[k].x);      // restarts at 0 per request
      id = __ldg(&a.ids[row_recs[k].z + pos]);
    }
    if (a.seg_ids) a.seg_ids[slot] = seg;
    if (a.positions) a.positions[slot] = pos;
    s_meta[threadIdx.x] = make_int2(pos, id);
  }
  __syncthreads();
  for (int j = jc0 + warp; j < j_end; j += kWarpsPerBlock) {
    const int64_t slot = row0 + j;
    T* x = reinterpret_cast<T*>(a.X) + slot * d;
    const int2 m = s_meta[j - jc0];
    const int pos = m.x, id = m.y;
    if (pos < 0) {                        // pad slot: zeros
      float z[V] = {};
      for (int i = lane; i < nvec; i += 32) Vec<T>::store(x + i * V, z);
      continue;
    }
    const T* e = reinterpret_cast<const T*>(a.tok_emb) + static_cast<int64_t>(id) * d;
    float v[NV][V];
    float sum = 0.f;
#pragma unroll
    for (int jv = 0; jv < NV; ++jv) {
      const int i = lane + 32 * jv;
      if (i < nvec) {
        Vec<T>::load(e + i * V, v[jv]);
        float p[V];
        if (a.pe_table) {
          const float* pt = a.pe_table + static_cast<int64_t>(pos) * d + i * V;
#pragma unroll
          for (int c = 0; c < V; c += 4) {
            float4 q = __ldg(reinterpret_cast<const float4*>(pt + c));
            p[c] = q.x; p[c + 1] = q.y; p[c + 2] = q.z; p[c + 3] = q.w;
          }
        } else {
          Vec<T>::load(reinterpret_cast<const T*>(a.pos_emb) + static_cast<int64_t>(pos) * d + i * V, p);
        }
        if (a.type_emb) {
#pragma unroll
          for (int c = 0; c < V; c += 4) {
            const float4 ty = *reinterpret_cast<const float4*>(s_type + i * V + c);
            p[c] += ty.x; p[c + 1] += ty.y; p[c + 2] += ty.z; p[c + 3] += ty.w;
          }
        }
#pragma unroll
        for (int c = 0; c < V; ++c) {
          const float t = v[jv][c] * a.emb_scale + p[c];
          v[jv][c] = t;
          sum += t;
        }
      }
    }
    if (a.ln_g) {
      const float mean = warp_sum(sum) / d;
      float sq = 0.f;
#pragma unroll
      for (int jv = 0; jv < NV; ++jv)
        if (lane + 32 * jv < nvec)
#pragma unroll
          for (int c = 0; c < V; ++c) { const float t = v[jv][c] - mean; sq += t * t; }
      const float rstd = rsqrtf(warp_sum(sq) / d + a.ln_eps);
#pragma unroll
      for (int jv = 0; jv < NV; ++jv) {
        const int i = lane + 32 * jv;
        if (i < nvec)
#pragma unroll
          for (int c = 0; c < V; c += 4) {
            const float4 g4 = *reinterpret_cast<const float4*>(s_g + i * V + c);
            const float4 b4 = *reinterpret_cast<const float4*>(s_b + i * V + c);
            v[jv][c] = (v[jv][c] - mean) * rstd * g4.x + b4.x;
            v[jv][c + 1] = (v[jv][c + 1] - mean) * rstd * g4.y + b4.y;
            v[jv][c + 2] = (v[jv][c + 2] - mean) * rstd * g4.z + b4.z;
            v[jv][c + 3] = (v[jv][c + 3] - mean) * rstd * g4.w + b4.w;
          }
      }
    }
#pragma unroll
    for (int jv = 0; jv < NV; ++jv) {
      const int i = lane + 32 * jv;
      if (i < nvec) Vec<T>::store(x + i * V, v[jv]);
    }
  }
}

// LayerNorm: each warp normalises kLnRows rows; all their 16-byte loads are issued before
// the first reduction so each lane keeps kLnRows * NV loads in flight.
constexpr int kLnRows = 2;

template <typename T, int NV>
__global__ void __launch_bounds__(kWarpsPerBlock * 32)
layernorm_kernel(int64_t rows, int d, const T* __restrict__ Z, const float* __restrict__ g,
                 const float* __restrict__ b, float eps, const int32_t* __restrict__ seg_ids,
                 T* __restrict__ Y) {
  constexpr int V = Vec<T>::N;
  const int lane = threadIdx.x & 31;
  const int64_t row0 =
      (static_cast<int64_t>(blockIdx.x) * kWarpsPerBlock + (threadIdx.x >> 5)) * kLnRows;
  pdl_wait();
  pdl_trigger();
  if (row0 >= rows) return;
  const int nvec = d / V;
  float v[kLnRows][NV][V];
  bool pad[kLnRows];
#pragma unroll
  for (int rr = 0; rr < kLnRows; ++rr) {
    const int64_t row = row0 + rr;
    pad[rr] = row >= rows || (seg_ids && __ldg(&seg_ids[row]) < 0);
    if (row >= rows) continue;
    const T* z = Z + row * d;
#pragma unroll
    for (int j = 0; j < NV; ++j) {
      const int i = lane + 32 * j;
      if (i < nvec) Vec<T>::load(z + i * V, v[rr][j]);
    }
  }
#pragma unroll
  for (int rr = 0; rr < kLnRows; ++rr) {
    const int64_t row = row0 + rr;
    if (row >= rows) break;
    T* y = Y + row * d;
    if (pad[rr]) {  // pad row -> 0 (R12)
      float zero[V] = {};
      for (int i = lane; i < nvec; i += 32) Vec<T>::store(y + i * V, zero);
      continue;
    }
    float sum = 0.f;
#pragma unroll
    for (int j = 0; j < NV; ++j)
      if (lane + 32 * j < nvec)
#pragma unroll
        for (int c = 0; c < V; ++c) sum += v[rr][j][c];
    const float mean = warp_sum(sum) / d;
    float sq = 0.f;
#pragma unroll
    for (int j = 0; j < NV; ++j)
      if (lane + 32 * j < nvec)
#pragma unroll
        for (int c = 0; c < V; ++c) { const float t = v[rr][j][c] - mean; sq += t * t; }
    const float rstd = rsqrtf(warp_sum(sq) / d + eps);
#pragma unroll
    for (int j = 0; j < NV; ++j) {
      const int i = lane + 32 * j;
      if (i < nvec) {
        float o[V];
        const float4* gg = reinterpret_cast<const float4*>(g + i * V);
        const float4* bb = reinterpret_cast<const float4*>(b + i * V);
#pragma unroll
        for (int c = 0; c < V; c += 4) {
          const float4 g4 = __ldg(gg + c / 4), b4 = __ldg(bb + c / 4);
          o[c] = (v[rr][j][c] - mean) * rstd * g4.x + b4.x;
          o[c + 1] = (v[rr][j][c + 1] - mean) * rstd * g4.y + b4.y;
          o[c + 2] = (v[rr][j][c + 2] - mean) * rstd * g4.z + b4.z;
          o[c + 3] = (v[rr][j][c + 3] - mean) * rstd * g4.w + b4.w;
        }
        Vec<T>::store(y + i * V, o);
      }
    }
  }
}

// unpack: one CTA per (batch row, kRowChunk-slot chunk).  The chunk's slots are contiguous in
// the rows buffer, so every thread first issues its 16-byte loads of them (independent of the
// segment layout), and only then resolves, one thread per slot, where each slot goes in the
// request-order output (binary search over the row's segment records staged in smem): the
// metadata's dependent loads overlap the data loads instead of preceding them.  Pad slots are
// loaded but not stored.
#ifndef TCB_UNPACK_CHUNK
#define TCB_UNPACK_CHUNK 16
#endif
#ifndef TCB_UNPACK_U
#define TCB_UNPACK_U 4
#endif
constexpr int kUnpackChunk = TCB_UNPACK_CHUNK;   // slots per CTA
static_assert(kUnpackChunk <= kWarpsPerBlock * 32, "one lookup thread per slot of a chunk");
__global__ void __launch_bounds__(kWarpsPerBlock * 32)
unpack_kernel(const int4* __restrict__ segtab, int row_len, int row_bytes_per_slot,
              const uint8_t* __restrict__ rows, uint8_t* __restrict__ out) {
  constexpr int U = TCB_UNPACK_U;
  extern __shared__ int4 recs[];
  __shared__ int64_t s_dst[kUnpackChunk];   // output token index of each slot of the chunk, -1 at pad
  const int row = blockIdx.x;
  const int jc0 = static_cast<int>(blockIdx.y) * kUnpackChunk;
  const int nslots = min(kUnpackChunk, row_len - jc0);
  const int64_t c0 = static_cast<int64_t>(row) * row_len + jc0;
  const int vps = row_bytes_per_slot / 16;             // 16-byte vectors per slot
  const int nvec = nslots * vps;
  const uint4* src = reinterpret_cast<const uint4*>(rows + c0 * row_bytes_per_slot);
  uint4* dst = reinterpret_cast<uint4*>(out);
  pdl_wait();
  pdl_trigger();
  uint4 t[U];
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const int i = threadIdx.x + u * blockDim.x;
    if (i < nvec) t[u] = __ldg(src + i);
  }
  const int S = segtab[0].x;
  const int* row_first = reinterpret_cast<const int*>(segtab + 1 + S);
  const int f = __ldg(&row_first[row]);
  const int nseg = __ldg(&row_first[row + 1]) - f;
  for (int i = threadIdx.x; i < nseg; i += blockDim.x) recs[i] = __ldg(&segtab[1 + f + i]);
  __syncthreads();
  if (threadIdx.x < nslots) {
    const int64_t slot = c0 + threadIdx.x;
    int lo = 0, hi = nseg - 1, k = -1;                 // last record with start <= slot
    while (lo <= hi) {
      const int mid = (lo + hi) >> 1;
      if (recs[mid].x <= slot) { k = mid; lo = mid + 1; } else { hi = mid - 1; }
    }
    int64_t o = -1;
    if (k >= 0 && slot < recs[k].x + recs[k].y) o = recs[k].z + (slot - recs[k].x);
    s_dst[threadIdx.x] = o;
  }
  __syncthreads();
  for (int i0 = threadIdx.x;;) {
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int i = i0 + u * blockDim.x;
      if (i < nvec) {
        const int j = i / vps;
        const int64_t o = s_dst[j];
        if (o >= 0) dst[o * vps + (i - j * vps)] = t[u];
      }
    }
    i0 += U * blockDim.x;
    if (i0 >= nvec) break;
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int i = i0 + u * blockDim.x;
      if (i < nvec) t[u] = __ldg(src + i);
    }
  }
}

__global__ void pe_table_kernel(float* table, int max_pos, int d, int variant) {
  const int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= static_cast<int64_t>(max_pos) * d) return;
  const int pos = static_cast<int>(i / d), dim = static_cast<int>(i % d);
  const int e = dim / 2;
  // Eq. (1)-(2): PE(pos,2e) = sin(pos/10000^(2e/d)); PE(pos,2e+1) = cos(pos/10000^((2e+1)/d))
  // (literal, R1; variant 1 uses 2e/d for both).  Evaluated in double, stored as fp32.
  const double expo = (dim % 2 == 0 || variant == 1) ? (2.0 * e) / d : (2.0 * e + 1.0) / d;
  const double ang = pos / pow(10000.0, expo);
  table[i] = static_cast<float>(dim % 2 == 0 ? sin(ang) : cos(ang));
}

// Runtime -> compile-time vectors-per-lane (registers hold exactly the row).
template <typename F>
bool dispatch_nv(int nv, F&& f) {
  switch (nv) {
    case 1: f(std::integral_constant<int, 1>{}); return true;
    case 2: f(std::integral_constant<int, 2>{}); return true;
    case 3: f(std::integral_constant<int, 3>{}); return true;
    case 4: f(std::integral_constant<int, 4>{}); return true;
    case 5: f(std::integral_constant<int, 5>{}); return true;
    case 6: f(std::integral_constant<int, 6>{}); return true;
    case 7: f(std::integral_constant<int, 7>{}); return true;
    case 8: f(std::integral_constant<int, 8>{}); return true;
    default: return false;
  }
}

}  // namespace

cudaError_t launch_embed(int dtype, const EmbedArgs& a, cudaStream_t s) {
  if (a.num_slots == 0) return cudaSuccess;
  const dim3 grid(static_cast<unsigned>(a.num_rows), static_cast<unsigned>((a.row_len + kRowChunk - 1) / kRowChunk));
  // <= row_len segment records + type embedding, LN gamma, LN beta (fp32, d each)
  const size_t smem = static_cast<size_t>(a.row_len) * sizeof(int4) + 3 * sizeof(float) * a.d;
  const int nv = (a.d / (dtype == 0 ? 4 : 8) + 31) / 32;
  cudaError_t attr_err = cudaSuccess, launch_err = cudaSuccess;
  auto go = [&](auto tag) {
    constexpr int NV = decltype(tag)::value;
    if (dtype == 0) {
      if (smem > 48 * 1024)
        attr_err = cudaFuncSetAttribute(pack_embed_kernel<float, NV>,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
      launch_err = launch_ex(pack_embed_kernel<float, NV>, grid, dim3(kWarpsPerBlock * 32), smem, s, 1, a);
    } else {
      if (smem > 48 * 1024)
        attr_err = cudaFuncSetAttribute(pack_embed_kernel<__nv_bfloat16, NV>,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
      launch_err = launch_ex(pack_embed_kernel<__nv_bfloat16, NV>, grid, dim3(kWarpsPerBlock * 32), smem, s,
                             1, a);
    }
  };
  if (!dispatch_nv(nv, go)) return cudaErrorInvalidValue;
  if (attr_err != cudaSuccess) return attr_err;
  return launch_err;
}

cudaError_t launch_layernorm(int dtype, int64_t rows, int d, const void* Z, const float* g,
                             const float* b, float eps, const int32_t* seg_ids, void* Y,
                             cudaStream_t s) {
  if (rows == 0) return cudaSuccess;
  const int64_t per_block = static_cast<int64_t>(kWarpsPerBlock) * kLnRows;
  const unsigned grid = static_cast<unsigned>((rows + per_block - 1) / per_block);
  const int nv = (d / (dtype == 0 ? 4 : 8) + 31) / 32;
  cudaError_t err = cudaSuccess;
  auto go = [&](auto tag) {
    constexpr int NV = decltype(tag)::value;
    if (dtype == 0)
      err = launch_ex(layernorm_kernel<float, NV>, dim3(grid), dim3(kWarpsPerBlock * 32), 0, s, 1,
                      rows, d, static_cast<const float*>(Z), g, b, eps, seg_ids,
                      static_cast<float*>(Y));
    else
      err = launch_ex(layernorm_kernel<__nv_bfloat16, NV>, dim3(grid), dim3(kWarpsPerBlock * 32), 0,
                      s, 1, rows, d, static_cast<const __nv_bfloat16*>(Z), g, b, eps, seg_ids,
                      static_cast<__nv_bfloat16*>(Y));
  };
  if (!dispatch_nv(nv, go)) return cudaErrorInvalidValue;
  return err;
}

cudaError_t launch_unpack(int dtype, const int4* segtab, int num_rows, int row_len, int d,
                          const void* rows, void* out, cudaStream_t s) {
  if (num_rows == 0) return cudaSuccess;
  const int bytes_per_slot = d * (dtype == 0 ? 4 : 2);
  const dim3 grid(static_cast<unsigned>(num_rows), static_cast<unsigned>((row_len + kUnpackChunk - 1) / kUnpackChunk));
  // <= row_len segment records per row
  const size_t smem = static_cast<size_t>(row_len) * sizeof(int4);
  if (smem > 48 * 1024) {
    const cudaError_t e = cudaFuncSetAttribute(unpack_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                               static_cast<int>(smem));
    if (e != cudaSuccess) return e;
  }
  return launch_ex(unpack_kernel, grid, dim3(kWarpsPerBlock * 32), smem, s, 1, segtab, row_len,
                   bytes_per_slot, static_cast<const uint8_t*>(rows), static_cast<uint8_t*>(out));
}

cudaError_t launch_pe_table(float* table, int max_pos, int d, int variant, cudaStream_t s) {
  const int64_t n = static_cast<int64_t>(max_pos) * d;
  pe_table_kernel<<<static_cast<unsigned>((n + 255) / 256), 256, 0, s>>>(table, max_pos, d, variant);
  return cudaGetLastError();
}

}  // namespace k
}  // namespace tcb
