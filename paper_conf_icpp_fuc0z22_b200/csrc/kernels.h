// kernels.h -- launchers of the sm_100a kernels of libtcb (device code lives in *.cu).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <cstdint>
#include <utility>

namespace tcb {
namespace k {

// Programmatic dependent launch (PDL).  Every kernel of the forward is launched with
// programmaticStreamSerialization, so its CTAs can be scheduled (and run their prologue:
// mbarrier init, TMEM allocation, tensor-map prefetch) as the previous kernel's CTAs retire.
// Device side, pdl_wait() precedes the first global-memory access (read OR write: the
// previous kernel may still read a buffer this one overwrites), and pdl_trigger() lets the
// next kernel launch early.  Without the launch attribute both are no-ops.
#ifdef __CUDACC__
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
#endif
// Host: whether launches carry the PDL attribute (TCB_NO_PDL=1 turns it off), and the
// attribute itself.
bool pdl_enabled();
inline void pdl_attr(cudaLaunchAttribute& a) {
  a.id = cudaLaunchAttributeProgrammaticStreamSerialization;
  a.val.programmaticStreamSerializationAllowed = 1;
}
// cudaLaunchKernelEx with an optional cluster size and the PDL attribute.
template <typename... KArgs, typename... Args>
cudaError_t launch_ex(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                      cudaStream_t s, int cluster, Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  int n = 0;
  if (cluster > 1) {
    attr[n].id = cudaLaunchAttributeClusterDimension;
    attr[n].val.clusterDim.x = cluster;
    attr[n].val.clusterDim.y = 1;
    attr[n].val.clusterDim.z = 1;
    ++n;
  }
  if (pdl_enabled()) pdl_attr(attr[n++]);
  cfg.attrs = attr;
  cfg.numAttrs = n;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// Embedding / metadata / elementwise (elementwise.cu) -------------------------------------
struct EmbedArgs {
  const int4* segtab;          // device segment table (header + records)
  const int32_t* ids;          // [total_tokens]
  const void* tok_emb;         // [vocab, d] dtype
  const void* pos_emb;         // [max_pos, d] dtype (learned PE) or nullptr
  const float* pe_table;       // [max_pos, d] fp32 sinusoidal table or nullptr
  const float* type_emb;       // [d] or nullptr
  const float* ln_g;           // [d] or nullptr (no embedding LN)
  const float* ln_b;
  float emb_scale, ln_eps;
  int32_t d, max_pos;
  int32_t num_rows, row_len;
  int64_t num_slots;
  void* X;                     // out [num_slots, d] dtype
  int32_t* seg_ids;            // out [num_slots] or nullptr
  int32_t* positions;          // out [num_slots] or nullptr
};
cudaError_t launch_embed(int dtype, const EmbedArgs& a, cudaStream_t s);

cudaError_t launch_layernorm(int dtype, int64_t rows, int d, const void* Z, const float* g,
                             const float* b, float eps, const int32_t* seg_ids, void* Y,
                             cudaStream_t s);

cudaError_t launch_unpack(int dtype, const int4* segtab, int num_rows, int row_len, int d,
                          const void* rows, void* out, cudaStream_t s);

cudaError_t launch_pe_table(float* table, int max_pos, int d, int variant, cudaStream_t s);

// Linear layers --------------------------------------------------------------------------
cudaError_t launch_linear_f32(int64_t M, int N, int K, const float* A, const float* W,
                              const float* bias, const float* R, int epi, float* C,
                              cudaStream_t s);

// Tensor-core GEMM (linear_tc.cu).  TMA descriptors are built on the host: A [M, K]
// (128-row boxes, 128B swizzle), W [N, K] (BN/CG-row boxes), C / R [M, N] (32 x 32 boxes,
// 64B swizzle; R is read only by the residual epilogue).
struct GemmMaps {
  CUtensorMap a, w, c, r;
  // optional: W with 64-row boxes (the half-width tail units of the L2-exchange LayerNorm GEMM)
  CUtensorMap w_half;
  bool has_w_half = false;
};
struct GemmShape {
  int cg, bn;  // CTAs per MMA tile (cta_group) and tile width in N
};
GemmShape linear_tc_shape(int N);
bool make_tmap_bf16(CUtensorMap* map, const void* ptr, uint64_t rows, uint64_t cols,
                    uint32_t box_rows, uint32_t box_cols, int swizzle_bytes);
bool make_gemm_a_map(CUtensorMap* map, const void* A, uint64_t M, uint64_t K);
bool make_gemm_w_map(CUtensorMap* map, const void* W, uint64_t N, uint64_t K);
// W with 64-row boxes: the half-width tail units of the L2-exchange LayerNorm GEMM
bool make_gemm_w_half_map(CUtensorMap* map, const void* W, uint64_t N, uint64_t K);
bool make_gemm_c_map(CUtensorMap* map, const void* C, uint64_t M, uint64_t N);
// tile_counter (one int32, zero at launch): dynamic tile order.  a_ready: readiness flags of
// A's 128-row blocks written by the still-running previous kernel (see ready_signal in
// linear_tc.cu; block b is complete at a_target = 4 x the producer's row width); the kernel
// then skips griddepcontrol.wait -- only for an A produced by the immediately preceding
// kernel, and a C no earlier kernel still reads.
cudaError_t launch_linear_bf16_tc(const GemmMaps& maps, int64_t M, int N, int K,
                                  const float* bias, int epi, cudaStream_t s,
                                  int* tile_counter = nullptr, const int* a_ready = nullptr,
                                  int a_target = 0);
// C = LayerNorm(A W^T + bias + R) * gamma + beta over rows of N = 512 columns (pad rows 0).
bool linear_ln_supported(int N);
// lng_stats / lng_cnt (optional scratch, sizes below; cnt zeroed before the launch) select the
// L2-exchange kernel for N = 1024.
cudaError_t launch_linear_ln_bf16_tc(const GemmMaps& maps, int64_t M, int N, int K,
                                     const float* bias, const float* gamma, const float* beta,
                                     float eps, const int32_t* seg_ids, cudaStream_t s,
                                     float2* lng_stats = nullptr, int* lng_cnt = nullptr,
                                     int* ready_out = nullptr, void* scatter_out = nullptr,
                                     const int4* segtab = nullptr);
// scatter_out (with the device segment table): the LayerNorm output of every real slot goes to
// scatter_out[token, :] in request order (the unpack fused into the encoder's last FFN2 + LN2);
// the packed C is not written.  The L2-exchange kernel only; cudaErrorNotSupported otherwise
// (the caller then writes the packed rows and unpacks separately).
size_t linear_ln_scratch_stats_bytes(int64_t M, int N);
size_t linear_ln_scratch_cnt_bytes(int64_t M);

// Attention ------------------------------------------------------------------------------
// tcgen05 kernel (attention_tc.cu): S and O in TMEM, 128-query x 128-key chunks.  item_counter:
// one int32 in device memory, zero at launch (dynamic item scheduling); NULL = static order.
// row_len: the batch's row length when known (<= 128 selects the scheduler-warp variant for
// one-chunk items), 0 otherwise.
cudaError_t launch_attention_bf16_tc(int64_t num_slots, int d_model, int num_heads,
                                     const void* qkv, const int32_t* seg_ids, const int4* segtab,
                                     void* O, int* item_counter, int row_len, cudaStream_t s);
cudaError_t launch_attention_f32(int64_t num_slots, int d_model, int num_heads,
                                 const float* qkv, const int32_t* seg_ids, const int4* segtab,
                                 float* O, cudaStream_t s);

// Decoder (decoder.cu, f4) ------------------------------------------------------------------
struct DecEmbedArgs {
  const int32_t* act;          // [rows] request index of each active row
  const int32_t* out_tok;      // [R, ld_out] generated tokens
  int32_t ld_out, t, bos, eos, d, rows;
  const __nv_bfloat16* tok_emb;  // [vocab, d]
  const float* pe;             // [max_pos, d] fp32 sinusoidal table
  float emb_scale;
  __nv_bfloat16* x;            // out [rows, d]
  const int32_t* d_t;          // if set: the step index is *d_t (CUDA-graph replay), not t
};
struct DecAttnArgs {
  const int32_t* act;
  const __nv_bfloat16* q;      // [rows, ldq]; the query of head h at column qoff + 64h
  int32_t ldq, qoff;
  __nv_bfloat16* kv;           // keys at column 64h, values at column voff + 64h
  int64_t ld_kv;
  int32_t voff;
  int32_t self, t, t_cap;      // self: cache of request r = rows [r t_cap, r t_cap + t]
  const int32_t* mem_start;    // cross: keys [mem_start[r], + mem_len[r])
  const int32_t* mem_len;
  int32_t d, heads, rows;
  float scale;
  __nv_bfloat16* out;          // [rows, d]
  const int32_t* d_t;          // if set: the step index is *d_t, not t
};
struct DecArgmaxArgs {
  const __nv_bfloat16* logits; // [rows, vocab]
  int32_t vocab, rows, t, eos, ld_out;
  const int32_t* act;
  const int32_t* t_max;        // [R]
  int32_t* out_tok;            // [R, ld_out]
  int32_t* out_len;            // [R]
  int32_t* done;               // [R]
  int32_t* flag;               // [rows] finished after this step
  const int32_t* d_t;          // if set: the step index is *d_t, not t
};
// Rows whose act[] entry is < 0 are padding (a graph captured for a bucket of rows): the
// kernels write zeros for them and record nothing.
cudaError_t launch_dec_step_advance(int32_t* d_t, cudaStream_t s);   // ++*d_t
cudaError_t launch_dec_embed(const DecEmbedArgs& a, cudaStream_t s);
cudaError_t launch_dec_attn(const DecAttnArgs& a, cudaStream_t s);
cudaError_t launch_dec_argmax(const DecArgmaxArgs& a, cudaStream_t s);

}  // namespace k
}  // namespace tcb
