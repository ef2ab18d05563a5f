// decoder.cu -- decode-step kernels of the Seq2Seq decoder (sm_100a).
//
// The decoder of the paper's setting is auto-regressive (§4.2.2): each step feeds
// every active request's last token through S decoder layers (readings R30-R33).
// The GEMMs of a step (QKV, W_O, W_Q, W_CO, FFN1, FFN2, logits) run on the tcgen05 kernels of
// linear_tc.cu with M = the number of active requests; this file holds what is specific to
// decoding:
//   dec_embed : x[i] = E_tok[y] * emb_scale + PE[t] for the active rows (separate PE: the
//               target position restarts at 0 per request, §4.1.1)
//   dec_attn  : one query per (request, head) over that request's OWN keys only --
//               self-attention over its KV cache positions [0, t] (the new key/value are
//               appended first), cross-attention over its own encoder output, i.e. the
//               segment [seg_start, seg_start + l) of the packed ConcatBatching rows
//               (Eq. (5)-(6) restricted to the request's diagonal block)
//   dec_argmax: greedy argmax over the vocabulary (lowest index on ties, R31), records the
//               token, marks the request finished on EOS or at its t_max (R32)
// Memory-bound and tiny per step: SIMT kernels, one warp per (row, head) / one CTA per row.
#include <cuda_bf16.h>

#include <cfloat>
#include <cstdint>

#include "kernels.h"

namespace tcb {
namespace k {
namespace {

constexpr int DH = 64;
constexpr int kAttnWarps = 4;            // heads per CTA
constexpr int kMaxKeys = 1024;           // smem score buffer per warp (keys are processed in chunks of it)

__global__ void __launch_bounds__(256)
dec_embed_kernel(DecEmbedArgs a) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  pdl_wait();
  pdl_trigger();
  if (warp >= a.rows) return;
  const int r = a.act[warp];
  const int t = a.d_t ? *a.d_t : a.t;
  __nv_bfloat16* x = a.x + static_cast<int64_t>(warp) * a.d;
  if (r < 0) {                                   // padding row of a bucketed graph
    for (int c = lane * 8; c < a.d; c += 256) *reinterpret_cast<uint4*>(x + c) = make_uint4(0, 0, 0, 0);
    return;
  }
  int tok = t == 0 ? a.bos : a.out_tok[static_cast<int64_t>(r) * a.ld_out + t - 1];
  // a request that already finished (whole-batch mode keeps computing it; nothing of it is
  // recorded any more) has no next token: feed EOS
  if (tok < 0) tok = a.eos;
  const __nv_bfloat16* e = a.tok_emb + static_cast<int64_t>(tok) * a.d;
  const float* pe = a.pe + static_cast<int64_t>(t) * a.d;
  for (int c = lane * 8; c < a.d; c += 256) {
    const uint4 v = *reinterpret_cast<const uint4*>(e + c);
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&v);
    uint4 o;
    __nv_bfloat162* ho = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 f = __bfloat1622float2(h[i]);
      ho[i] = __floats2bfloat162_rn(f.x * a.emb_scale + pe[c + 2 * i], f.y * a.emb_scale + pe[c + 2 * i + 1]);
    }
    *reinterpret_cast<uint4*>(x + c) = o;
  }
}

// One warp per (active row i, head h).  Keys of row i: [kstart, kstart + klen) of `kv`
// (row stride ld_kv elements; K at column h*64, V at column voff + h*64).
//   self (append != nullptr): request r = act[i], kstart = r * t_cap, klen = t + 1; the new
//        token's key / value (columns [d, 3d) of its QKV row) are written at position t first
//   cross: kstart = mem_start[r], klen = mem_len[r] (the request's encoder segment)
__global__ void __launch_bounds__(kAttnWarps * 32)
dec_attn_kernel(DecAttnArgs a) {
  __shared__ float sp[kAttnWarps][kMaxKeys];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int i = blockIdx.x;
  const int h = blockIdx.y * kAttnWarps + w;
  pdl_wait();
  pdl_trigger();
  if (h >= a.heads) return;
  const int r = a.act[i];
  if (r < 0) {                                   // padding row of a bucketed graph
    reinterpret_cast<__nv_bfloat162*>(a.out + static_cast<int64_t>(i) * a.d + h * DH)[lane] =
        __floats2bfloat162_rn(0.f, 0.f);
    return;
  }
  const int t = a.d_t ? *a.d_t : a.t;
  int64_t kstart;
  int klen;
  if (a.self) {
    kstart = static_cast<int64_t>(r) * a.t_cap;
    klen = t + 1;
    // append this step's key and value (2 x 64 bf16) at cache position t
    const __nv_bfloat16* src = a.q + static_cast<int64_t>(i) * a.ldq;
    __nv_bfloat16* dst = a.kv + (kstart + t) * a.ld_kv;
    const uint32_t* sk = reinterpret_cast<const uint32_t*>(src + a.d + h * DH);
    const uint32_t* sv = reinterpret_cast<const uint32_t*>(src + 2 * a.d + h * DH);
    reinterpret_cast<uint32_t*>(dst + h * DH)[lane] = sk[lane];
    reinterpret_cast<uint32_t*>(dst + a.voff + h * DH)[lane] = sv[lane];
    __syncwarp();
  } else {
    kstart = a.mem_start[r];
    klen = a.mem_len[r];
  }
  // q of this head in registers (fp32)
  float q[DH];
  const uint4* q4 = reinterpret_cast<const uint4*>(a.q + static_cast<int64_t>(i) * a.ldq + a.qoff + h * DH);
#pragma unroll
  for (int v = 0; v < DH / 8; ++v) {
    const uint4 x = q4[v];
    const __nv_bfloat162* hh = reinterpret_cast<const __nv_bfloat162*>(&x);
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float2 f = __bfloat1622float2(hh[e]);
      q[8 * v + 2 * e] = f.x * a.scale;
      q[8 * v + 2 * e + 1] = f.y * a.scale;
    }
  }
  // Keys in chunks of kMaxKeys (the smem score buffer) with an online max / sum across
  // chunks, so any klen is safe (cross-attention keys = the request's source length, which can
  // exceed the self-attention bound).  For klen <= kMaxKeys this is exactly one pass.
  float m_run = -INFINITY, l = 0.f, o0 = 0.f, o1 = 0.f;
  for (int base = 0; base < klen; base += kMaxKeys) {
    const int n = min(kMaxKeys, klen - base);
    // scores: lane j takes keys j, j + 32, ...
    float m = -INFINITY;
    for (int j = lane; j < n; j += 32) {
      const uint4* k4 = reinterpret_cast<const uint4*>(a.kv + (kstart + base + j) * a.ld_kv + h * DH);
      float s = 0.f;
#pragma unroll
      for (int v = 0; v < DH / 8; ++v) {
        const uint4 x = k4[v];
        const __nv_bfloat162* hh = reinterpret_cast<const __nv_bfloat162*>(&x);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float2 f = __bfloat1622float2(hh[e]);
          s = fmaf(q[8 * v + 2 * e], f.x, s);
          s = fmaf(q[8 * v + 2 * e + 1], f.y, s);
        }
      }
      sp[w][j] = s;
      m = fmaxf(m, s);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    const float mn = fmaxf(m_run, m);
    const float f = m_run == -INFINITY ? 0.f : __expf(m_run - mn);   // rescale earlier chunks
    float lc = 0.f;
    for (int j = lane; j < n; j += 32) {
      const float p = __expf(sp[w][j] - mn);
      sp[w][j] = p;
      lc += p;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) lc += __shfl_xor_sync(0xffffffffu, lc, o);
    __syncwarp();
    l = l * f + lc;
    o0 *= f;
    o1 *= f;
    // o = sum_j p_j v_j: lane owns dims 2*lane, 2*lane + 1 (coalesced 128-byte V rows)
    const __nv_bfloat16* vb = a.kv + (kstart + base) * a.ld_kv + a.voff + h * DH + 2 * lane;
    for (int j = 0; j < n; ++j) {
      const float2 fv = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(vb + j * a.ld_kv));
      const float p = sp[w][j];
      o0 = fmaf(p, fv.x, o0);
      o1 = fmaf(p, fv.y, o1);
    }
    m_run = mn;
    __syncwarp();                                // sp is rewritten by the next chunk
  }
  const float inv = klen > 0 ? 1.f / l : 0.f;
  reinterpret_cast<__nv_bfloat162*>(a.out + static_cast<int64_t>(i) * a.d + h * DH)[lane] =
      __floats2bfloat162_rn(o0 * inv, o1 * inv);
}

// Greedy argmax over one row of bf16 logits (lowest index on ties, R31); records the token
// of active row i (request act[i]) unless the request already finished; finished on EOS or
// when it has produced t_max[r] tokens (R32).  flag[i] = request finished after this step.
__global__ void __launch_bounds__(256)
dec_argmax_kernel(DecArgmaxArgs a) {
  __shared__ float sv[256];
  __shared__ int si[256];
  const int i = blockIdx.x;
  pdl_wait();
  pdl_trigger();
  const __nv_bfloat16* lg = a.logits + static_cast<int64_t>(i) * a.vocab;
  float best = -INFINITY;
  int bi = 0x7fffffff;
  for (int v = threadIdx.x; v < a.vocab; v += blockDim.x) {
    const float x = __bfloat162float(lg[v]);
    if (x > best) { best = x; bi = v; }          // v ascending per thread: first max kept
  }
  sv[threadIdx.x] = best;
  si[threadIdx.x] = bi;
  __syncthreads();
  for (int s = blockDim.x / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) {
      const float ob = sv[threadIdx.x + s];
      const int oi = si[threadIdx.x + s];
      if (ob > sv[threadIdx.x] || (ob == sv[threadIdx.x] && oi < si[threadIdx.x])) {
        sv[threadIdx.x] = ob;
        si[threadIdx.x] = oi;
      }
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const int r = a.act[i];
    if (r < 0) {                                 // padding row of a bucketed graph
      a.flag[i] = 1;
      return;
    }
    const int t = a.d_t ? *a.d_t : a.t;
    const int tok = si[0];
    if (!a.done[r]) {
      a.out_tok[static_cast<int64_t>(r) * a.ld_out + t] = tok;
      if (tok == a.eos || t + 1 >= a.t_max[r]) {
        a.done[r] = 1;
        a.out_len[r] = t + 1;
      }
    }
    a.flag[i] = a.done[r];
  }
}

__global__ void dec_step_advance_kernel(int32_t* d_t) {
  pdl_wait();
  pdl_trigger();
  *d_t += 1;
}

}  // namespace

cudaError_t launch_dec_step_advance(int32_t* d_t, cudaStream_t s) {
  return launch_ex(dec_step_advance_kernel, dim3(1), dim3(1), 0, s, 1, d_t);
}

cudaError_t launch_dec_embed(const DecEmbedArgs& a, cudaStream_t s) {
  if (a.rows == 0) return cudaSuccess;
  return launch_ex(dec_embed_kernel, dim3((a.rows + 7) / 8), dim3(256), 0, s, 1, a);
}

cudaError_t launch_dec_attn(const DecAttnArgs& a, cudaStream_t s) {
  if (a.rows == 0) return cudaSuccess;
  if (a.d / a.heads != DH) return cudaErrorInvalidValue;
  return launch_ex(dec_attn_kernel, dim3(a.rows, (a.heads + kAttnWarps - 1) / kAttnWarps),
                   dim3(kAttnWarps * 32), 0, s, 1, a);
}

cudaError_t launch_dec_argmax(const DecArgmaxArgs& a, cudaStream_t s) {
  if (a.rows == 0) return cudaSuccess;
  return launch_ex(dec_argmax_kernel, dim3(a.rows), dim3(256), 0, s, 1, a);
}


}  // namespace k
}  // namespace tcb
