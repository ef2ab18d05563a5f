/* tcb_ops.h -- op-level C ABI: each hot-path kernel of tcb_encoder_forward on its own, for
 * per-kernel parity tests and per-kernel roofline timing.  Same conventions as tcb.h
 * (device pointers, caller-owned, async on `stream`, tcb_status + tcb_last_error()).
 * dtype: 0 = fp32, 1 = bf16.  All matrices row-major.
 */
#ifndef TCB_OPS_H
#define TCB_OPS_H
#include "tcb.h"

#ifdef __cplusplus
extern "C" {
#endif

/* Epilogues of the linear layers. */
enum { TCB_EPI_BIAS = 0, TCB_EPI_BIAS_GELU = 1, TCB_EPI_BIAS_RELU = 2, TCB_EPI_BIAS_RESIDUAL = 3 };

/* C[M, N] = epi(A[M, K] . W[N, K]^T + bias[N]) (+ R[M, N] for TCB_EPI_BIAS_RESIDUAL).
 * Eq. (3) for Q/K/V with W_Q|W_K|W_V stacked, and the W_O / FFN linears
 * (P:344-347).  bias is fp32 [N]; A, W, R, C are in `dtype`.  fp32 accumulation.
 * bf16: tcgen05.mma (TMEM accumulators, TMA-fed, sm_100a); needs K % 64 == 0, N % 64 == 0,
 * 16-byte aligned pointers; M arbitrary (>= 0).  fp32: SIMT FFMA kernel, any shape. */
tcb_status tcb_op_linear(int32_t dtype, int64_t M, int32_t N, int32_t K, const void* A,
                         const void* W, const float* bias, const void* R, int32_t epilogue,
                         void* C, tcb_stream_t stream);

/* Fused post-LN residual block (R10): C = LN(A W^T + bias + R) * gamma + beta, row-wise
 * over the N output columns (biased variance, two-pass, fp32) -- tcb_op_linear with
 * TCB_EPI_BIAS_RESIDUAL followed by tcb_op_layernorm in one tcgen05 kernel.  bf16 only and
 * N in {512, 768, 1024} (a cluster of N / 256 CTA pairs owns complete rows, each pair 256
 * columns in TMEM, row statistics exchanged over DSMEM); K % 64 == 0.  Rows whose
 * d_segment_ids entry is < 0 (pad slots) are written as 0; d_segment_ids may be NULL.
 * Returns TCB_ERR_UNSUPPORTED for other shapes. */
tcb_status tcb_op_linear_ln(int64_t M, int32_t N, int32_t K, const void* A, const void* W,
                            const float* bias, const void* R, const float* gamma,
                            const float* beta, float eps, const int32_t* d_segment_ids,
                            void* C, tcb_stream_t stream);

/* Segment-masked multi-head attention, Eq. (5)-(6) over packed rows:
 * O[i, h] = sum_j softmax_j(q_i.k_j / sqrt(d_head) + M_ij) v_j, M_ij = 0 iff slots i and j
 * hold the same request (the diagonal blocks Q_i K_i^T of Eq. (7)), -inf otherwise (R11:
 * masked pairs are skipped, never evaluated with a finite surrogate).  Pad queries give 0.
 *   qkv : [num_slots, 3 d_model] ([Q | K | V], head h = columns [h dh, (h+1) dh) of each)
 *   d_segment_ids : [num_slots] int32 (-1 pad), as written by tcb_embed
 *   d_segtab : the plan's device segment table
 *   O : out [num_slots, d_model]. */
tcb_status tcb_op_attention(int32_t dtype, int64_t num_slots, int32_t d_model,
                            int32_t num_heads, const void* qkv, const int32_t* d_segment_ids,
                            const int32_t* d_segtab, void* O, tcb_stream_t stream);

/* Y[r] = (Z[r] - mean) / sqrt(var + eps) * g + b (biased variance, two-pass, fp32), one
 * warp per row (R10).  If d_segment_ids != NULL, rows with segment id < 0 (pad) are
 * written as 0. */
tcb_status tcb_op_layernorm(int32_t dtype, int64_t rows, int32_t d, const void* Z,
                            const float* g, const float* b, float eps,
                            const int32_t* d_segment_ids, void* Y, tcb_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif
