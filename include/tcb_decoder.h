/* tcb_decoder.h -- C ABI of the auto-regressive decoder of the Seq2Seq setting (SURVEY.md
 * §8(f) f4) with early memory cleaning (§4.2.2).
 *
 * The paper's model has an encoder and a decoder of S layers each; "Decoder outputs go
 * through a final linear layer and activation function to generate final results"
 * (P:340-351), and "the decoder is an auto-regressive model", so requests of one batch
 * finish at different times (§4.2.2).  "Early memory cleaning" removes "the data
 * of requests whose results are generated, instead of waiting the completion of whole batch
 * inference", which the paper makes possible by giving each request (slot) its
 * own tensors.  Readings: R30 decoder layer = post-LN causal
 * self-attention + cross-attention over the request's OWN encoder output (the segment of
 * the packed ConcatBatching rows) + FFN; R31 tied E_tok embedding / output projection (no
 * bias), greedy argmax with lowest index on ties, BOS = 1, EOS = 2; R32 t_max = l_src
 * (capped by the PE table); R33 early cleaning = a finished request leaves the active set
 * and its KV-cache slot is free for reuse.
 *
 * Ownership: tcb_decoder is library-owned (tcb_decoder_destroy): it holds non-owning views
 * of the caller's decoder weight tensors and OWNS its device buffers (KV cache, encoder
 * memory K/V, step activations, logits), sized once at creation.  Conventions (errors,
 * threading, no CPU fallback) as in tcb.h.  bf16 Transformer-family models only
 * (sinusoidal PE, d_model in {512, 768, 1024}, d_head = 64).
 */
#ifndef TCB_DECODER_H
#define TCB_DECODER_H

#include "tcb.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tcb_decoder tcb_decoder;

/* Number of decoder tensors: 20 * num_layers, per layer in the order
 *   w_qkv [3d, d], b_qkv [3d], w_o [d, d], b_o [d], ln1_g [d], ln1_b [d],
 *   w_q [d, d], b_q [d], w_kv [2d, d], b_kv [2d], w_co [d, d], b_co [d], ln2_g, ln2_b,
 *   w_1 [d_ff, d], b_1 [d_ff], w_2 [d, d_ff], b_2 [d], ln3_g, ln3_b
 * matrices bf16 row-major [N, K], vectors fp32 (the encoder's conventions). */
int32_t tcb_decoder_weights_count(const tcb_model_config* cfg);

/* Create a decoder over the encoder weights `enc` (tied E_tok, PE table, model config).
 * max_requests: most requests one decode may hold; max_slots: largest encoder plan
 * (num_slots) whose output it attends; max_target: largest t_max (<= max_pos - 1).
 * Allocates its device buffers (TCB_ERR_OUT_OF_MEMORY if they do not fit). */
tcb_status tcb_decoder_create(const tcb_weights* enc, const void* const* device_tensors,
                              int32_t num_tensors, int32_t max_requests, int64_t max_slots,
                              int32_t max_target, tcb_decoder** out);
void tcb_decoder_destroy(tcb_decoder* dec);

/* Greedy decoding of every placed request of `plan` from its encoder output `d_enc_rows`
 * ([num_slots, d] bf16, what tcb_encoder_forward wrote); request r's memory is its segment
 * [req_row * L + req_col, + l_r) of those rows.
 * Request r (request order, placed ones only) generates tokens until EOS or t_max(r) =
 * min(l_r, max_target) (R32).  early_clean = 1: after each step the finished requests leave
 * the active set (R33); 0: the whole batch keeps computing until its last request finishes
 * (the paper's baseline) -- the tokens are identical either way.
 * Outputs (caller-owned): d_tokens [num_requests, max_target] int32 device, -1 past the end
 * and for unplaced requests; h_lengths [num_requests] host, generated count (0 if unplaced).
 * Blocking: while step t runs, the host reads the finished flags of step t-1 back to build
 * the active set of step t+1 (so a finished request is computed once more, ignored).  Each
 * step is replayed from a CUDA graph captured per bucket of rows (power of two >= the active
 * count, at most max_requests) and per d_tokens buffer, unless the caller is capturing
 * `stream` or TCB_NO_DEC_GRAPH=1. */
tcb_status tcb_decode_greedy(tcb_decoder* dec, const tcb_plan* plan, const void* d_enc_rows,
                             int32_t early_clean, int32_t* d_tokens, int32_t* h_lengths,
                             tcb_stream_t stream);

/* Counters of the last tcb_decode_greedy. */
typedef struct {
  int32_t steps;               /* decode steps run                                        */
  int64_t rows_computed;       /* sum over steps of the active rows (decoder work)         */
  int64_t tokens_generated;    /* sum of h_lengths                                         */
  int64_t kv_bytes_peak;       /* largest live self-attention KV cache over the steps      */
  double kv_bytes_avg;         /* its mean over the steps                                  */
  double ms_total;             /* host wall time of the call                               */
} tcb_decode_stats;
tcb_status tcb_decoder_stats(const tcb_decoder* dec, tcb_decode_stats* out);

/* Debug / parity: copy the bf16 logits of the LAST step ([rows of that step, vocab], row i
 * = the i-th active request of that step) to host memory; *rows receives the row count. */
tcb_status tcb_decoder_last_logits(const tcb_decoder* dec, void* h_logits, int64_t capacity_elems,
                                   int32_t* rows);

#ifdef __cplusplus
}
#endif
#endif
