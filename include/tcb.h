/* tcb.h -- C ABI of the B200-native ConcatBatching encoder (TCB, Fu et al., ICPP'22).
 *
 * Citations "P:<line>" are lines of the paper text; "R<k>" are the readings of
 * the paper listed in DESIGN.md §3.  Everything here is extern "C", takes plain pointers
 * and sizes, and never lets a C++ exception or abort cross the boundary: every call
 * validates its arguments and returns a tcb_status; the message of the last failure on the
 * calling thread is available from tcb_last_error().
 *
 * Memory ownership:
 *   - tcb_plan     : library-owned HOST object (tcb_plan_destroy).
 *   - tcb_weights  : library-owned handle holding non-owning views of caller DEVICE tensors
 *                    plus a small library-owned device table (sinusoidal PE) and the TMA
 *                    descriptors of the weight matrices (tcb_weights_destroy).
 *   - activations, workspace, device segment table, token ids, outputs: caller-owned device
 *     memory.  No call below allocates device memory after tcb_weights_create, so
 *     tcb_encoder_forward / tcb_unpack are CUDA-graph capturable.
 * Execution: every device call is asynchronous on the caller's stream.  Kernel faults
 * surface at the caller's next synchronisation; launch errors return TCB_ERR_CUDA.
 * Threading: distinct plans / streams may be used concurrently; plans and weights are
 * read-only after creation.
 */
#ifndef TCB_H
#define TCB_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* tcb_stream_t; /* == cudaStream_t; NULL = legacy default stream */

typedef enum {
  TCB_OK = 0,
  TCB_ERR_INVALID_ARGUMENT = -1,   /* null pointer, n < 0, a length <= 0, row_len <= 0 or
                                      row_len % 8 != 0, bad enum, size mismatch          */
  TCB_ERR_REQUEST_TOO_LONG = -2,   /* a request longer than a row (constraint (11),
                                      P:958-961; reading R15: reject, never truncate)     */
  TCB_ERR_UNSUPPORTED = -3,        /* model shape outside what the kernels implement      */
  TCB_ERR_CUDA = -4,               /* a CUDA runtime / driver call failed                  */
  TCB_ERR_OUT_OF_MEMORY = -5,
  TCB_ERR_WORKSPACE_TOO_SMALL = -6,
  TCB_ERR_NO_DEVICE = -7           /* no sm_100 device visible: there is no CPU fallback   */
} tcb_status;

/* Message of the last failing tcb_* call on this thread ("" if none).  Valid until the
 * next tcb_* call on the same thread. */
const char* tcb_last_error(void);
const char* tcb_version(void);

/* ======================================================================================
 * 1. Packing (host).  The problem statement: request n has a sentence of l_n words
 *    (P:856-860); a batch is B rows x L words; x^{tk}_n = 1 puts request n in
 *    row k, at most once (constraint (10)) and with sum l_n <= L per
 *    row (constraint (11)).  Pure ConcatBatching concatenates requests end to
 *    end with padding only at the row tail (Fig. 1(c); §4.1).
 * ==================================================================================== */
typedef enum {
  TCB_PACK_FIRST_FIT = 0,            /* request -> lowest-index row with room, input order
                                        (R14: Alg. 1's "greedily put")         */
  TCB_PACK_NEXT_FIT = 1,             /* only the most recently opened row is considered   */
  TCB_PACK_FIRST_FIT_DECREASING = 2, /* First-Fit over a stable descending-length order   */
  TCB_PACK_NAIVE = 3,                /* NaiveBatching: one request per row, input order
                                        (TNB, Fig. 1(a); R17)                    */
  TCB_PACK_LENGTH_SORTED = 4         /* one request per row, stable ascending length
                                        (TurboTransformers-like; R18)           */
} tcb_pack_policy;

typedef struct tcb_plan tcb_plan;

/* Assign requests to rows.
 *   lengths  : [n] host int32, request order, each in [1, row_len]
 *   n        : number of requests, >= 0 (n == 0 gives an empty plan with 0 rows)
 *   row_len  : L, > 0 and a multiple of 8 (16-byte rows for bf16 vectors)
 *   max_rows : B cap; 0 = unbounded.  When the cap is hit the remaining requests that fit
 *              no row are left unplaced (req_row = -1) and the status is still TCB_OK (R16:
 *              the scheduler defers them, Alg. 1 picks a subset).
 *   policy   : tcb_pack_policy
 *   out      : receives a new plan (tcb_plan_destroy).
 * Within a row, requests are laid out contiguously from column 0 in placement order
 * (slotted plans below leave gaps at slot tails: those slots are pad, like the row tail).
 * Segments (placed requests) are numbered globally in (row, column) order (R13). */
tcb_status tcb_pack(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                    int32_t policy, tcb_plan** out);

/* Slotted ConcatBatching (§4.2; Eq. (8); Alg. 2 l.4-7; reading R26).
 * Each row is divided into floor(row_len / z) slots of z words (the tail is unused); in
 * input order each request goes to the first slot (rows in order, slots left to right) with
 * room, opening a new row when none has room (up to max_rows, 0 = unbounded).  Requests
 * never straddle a slot; inside a slot they are contiguous from the slot start.  A request
 * longer than z, or one that finds no slot under the row cap, is left unplaced (req_row = -1,
 * status OK: deferred, R26).  slot_len = 0 selects z = the largest length (Alg. 2 l.4);
 * slot_len = row_len is tcb_pack(TCB_PACK_FIRST_FIT).  The plan is an ordinary plan: the
 * kernels are unchanged, because attention already restricts every query to its own request
 * (Eq. (8)'s per-slot softmax is the special case where a slot holds one request).
 *   slot_len : z in [0, row_len]; tcb_plan_info.slot_len reports the z used.
 * Errors as tcb_pack (a request longer than row_len is TCB_ERR_REQUEST_TOO_LONG). */
tcb_status tcb_pack_slotted(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                            int32_t slot_len, tcb_plan** out);
void tcb_plan_destroy(tcb_plan* plan);

typedef struct {
  int32_t num_requests, num_placed, num_rows, row_len, num_segments;
  int32_t slot_len;            /* slotted plans: slot size z; 0 for the other policies      */
  int64_t total_tokens;        /* sum of all lengths (token_ids / outputs are this long)   */
  int64_t placed_tokens;       /* T: non-pad tokens in the rows                            */
  int64_t num_slots;           /* M = num_rows * row_len                                  */
  int64_t qtiles;              /* ceil(M / 128)                                            */
  int64_t kv_tiles_visited;    /* 128x128 (q,k) tiles touching a diagonal block; defined
                                  when row_len % 128 == 0, else -1 (§8(c) o9)              */
  int64_t kv_tiles_dense;      /* num_rows * (row_len/128)^2: pure ConcatBatching's dense
                                  work; -1 when row_len % 128 != 0             */
  int64_t useful_score_elems;  /* sum_i l_i^2 over placed requests                          */
  int64_t executed_score_elems;/* per head: S = QK^T elements the attention kernel computes
                                  on the tensor cores (128-query x 128-key chunks over each
                                  query block's key interval)                             */
  int64_t softmax_score_elems; /* per head: of those, the elements that go through the
                                  softmax exponentials (32-row x 32-key groups intersecting
                                  the rows' own requests; dead groups are skipped)         */
} tcb_plan_info;

tcb_status tcb_plan_info_get(const tcb_plan* plan, tcb_plan_info* info);

/* Host copies of the plan.  Any pointer may be NULL to skip that array.
 *   req_row, req_col : [num_requests] (-1 when unplaced)
 *   seg_req, seg_start (flattened slot index row*L+col) : [num_segments]
 *   cu_seqlens : [num_segments + 1], over compact real tokens in segment order (R13)
 *   segment_ids, positions : [num_slots], -1 at pad slots (R12); positions restart at 0 per
 *                            request (separate PE, §4.1.1; R2)
 *   qtile_kv : [2 * qtiles]: for each 128-slot q-tile of the flattened rows,
 *              [start of the segment of its first real slot, end of the segment of its
 *              last real slot), or (-1, -1). */
tcb_status tcb_plan_copy(const tcb_plan* plan, int32_t* req_row, int32_t* req_col,
                         int32_t* seg_req, int32_t* seg_start, int32_t* cu_seqlens,
                         int32_t* segment_ids, int32_t* positions, int32_t* qtile_kv);

/* The device form of a plan: the segment table the kernels expand.  Layout (int32 words):
 *   header (4 words)  {num_segments S, num_slots, row_len, total_tokens (low 31 bits)};
 *   S records (4 words each, 16-byte aligned), one per segment in (row, column) order:
 *                     {slot_start, length, token_offset (request-order index of its first
 *                      token), request};
 *   row index (num_rows + 1 words, padded to a multiple of 4): row_first[r] = index of the
 *                     first segment of row r, row_first[num_rows] = S;
 *   query-block order (qtiles words, padded to a multiple of 4): the 128-slot query blocks
 *                     by decreasing number of 128-key chunks of their key interval (ties by
 *                     index) -- the attention kernel hands out its items in this order.
 * tcb_plan_segtab_words gives the word count
 * (4 * (1 + S) + round_up(num_rows + 1, 4) + round_up(qtiles, 4));
 * tcb_plan_write_segtab writes it into a HOST buffer of at least that many words; the caller
 * copies it to the device (16-byte aligned) and passes that pointer as d_segtab below.  A
 * plan of the same (num_rows, row_len) may later be written into the same device buffer (if
 * it is large enough) and a captured CUDA graph replayed: no kernel reads the host plan. */
int64_t tcb_plan_segtab_words(const tcb_plan* plan);
tcb_status tcb_plan_write_segtab(const tcb_plan* plan, int32_t* host_dst, int64_t capacity_words);

/* ======================================================================================
 * 2. Model and weights.
 *    Encoder of S layers: masked self-attention (Eq. (5)-(6)) with
 *    W_O, residual and LayerNorm, then FFN with residual and LayerNorm
 *    (post-LN, R10); d_head = d_model / num_heads is the sqrt(d) of Eq. (4)/(5) (R6).
 * ==================================================================================== */
typedef struct {
  int32_t num_layers, d_model, num_heads, d_ff, vocab, max_pos;
  int32_t dtype;        /* 0 = fp32 (SIMT path), 1 = bf16 (tensor-core path)              */
  int32_t act;          /* 0 = GELU (erf form), 1 = ReLU (R9)                              */
  int32_t pe;           /* 0 = sin_paper (Eq. (1)-(2) literal, R1), 1 = sin_vaswani,
                           2 = learned table indexed by the restarted position (R4)       */
  int32_t emb_ln;       /* 1 = LayerNorm after the embedding sum (BERT, R5)                */
  int32_t use_type_emb; /* 1 = add token-type-0 embedding (BERT, R5)                       */
  float ln_eps, emb_ln_eps, emb_scale;                                     /* R3, R10 */
} tcb_model_config;

typedef struct tcb_weights tcb_weights;

/* Number of tensors tcb_weights_create expects: 5 + 12 * num_layers, in this order
 * (shapes row-major; "mat" tensors in the model dtype, "vec" tensors always fp32):
 *   tok_emb [vocab, d] mat, pos_emb [max_pos or 1, d] mat, type_emb [d] vec,
 *   emb_ln_g [d] vec, emb_ln_b [d] vec, then per layer:
 *   w_qkv [3d, d] mat (rows: Q then K then V output features; head h = columns
 *   [h*dh, (h+1)*dh) of each, R7), b_qkv [3d] vec, w_o [d, d] mat, b_o [d] vec,
 *   ln1_g [d] vec, ln1_b [d] vec, w_1 [d_ff, d] mat, b_1 [d_ff] vec, w_2 [d, d_ff] mat,
 *   b_2 [d] vec, ln2_g [d] vec, ln2_b [d] vec.
 * All pointers are device pointers, 16-byte aligned; they must outlive the handle. */
int32_t tcb_weights_count(const tcb_model_config* cfg);

/* Validates the config (TCB_ERR_UNSUPPORTED when: d_model % num_heads != 0; bf16 and
 * (d_head != 64 or d_model % 64 != 0 or d_ff % 64 != 0); fp32 and d_head > 64 or
 * d_head % 2 != 0; d_model > 4096), builds the sinusoidal PE table on the device and the
 * weight TMA descriptors.  Requires a visible sm_100 device (else TCB_ERR_NO_DEVICE). */
tcb_status tcb_weights_create(const tcb_model_config* cfg, const void* const* device_tensors,
                              int32_t num_tensors, tcb_weights** out);
void tcb_weights_destroy(tcb_weights* w);

/* Workspace bytes for a forward over num_slots = num_rows * row_len slots. */
tcb_status tcb_workspace_size(const tcb_model_config* cfg, int64_t num_slots, size_t* bytes);

/* ======================================================================================
 * 3. Device path.
 * ==================================================================================== */

/* pack_embed: X[slot] = E_tok[id] * emb_scale + PE(position(slot)) (+ E_type[0]; then
 * LN_emb when emb_ln) for real slots, 0 for pad slots; positions restart per request
 * (separate PE, §4.1.1; Eq. (1)-(2) P:329-333).
 *   d_segtab     : device segment table (tcb_plan_write_segtab)
 *   d_token_ids  : [total_tokens] device int32, request order
 *   d_rows       : out [num_slots, d_model] device, model dtype
 *   d_segment_ids, d_positions : out [num_slots] device int32 or NULL (-1 at pad) */
tcb_status tcb_embed(const tcb_weights* w, const tcb_plan* plan, const int32_t* d_segtab,
                     const int32_t* d_token_ids, void* d_rows, int32_t* d_segment_ids,
                     int32_t* d_positions, tcb_stream_t stream);

/* Whole encoder: pack_embed, then S x [QKV GEMM -> segment-masked attention (Eq. (5)) ->
 * W_O GEMM + bias + residual -> LN1 -> FFN1 GEMM + bias + act -> FFN2 GEMM + bias +
 * residual -> LN2].  d_rows receives the last layer's hidden states [num_slots, d_model]
 * (pad slots 0).  The plan is read only for its shape (num_rows, row_len) and validation;
 * the device segment table is what the kernels use.  Unless the caller is capturing
 * `stream`, the call replays a CUDA graph of its own launch sequence (captured on a private
 * stream on the first call with the same shape and the same d_segtab / d_token_ids / d_rows /
 * d_workspace pointers, at most 4 kept per weights handle; TCB_NO_FWD_GRAPH=1 launches
 * directly); inside a caller's capture the kernels are captured into that graph.  The workspace holds, for bf16
 * d in {512, 768, 1024}, the row-statistics scratch of the LayerNorm GEMMs; its counters are
 * zeroed by the call (one memset on the stream). */
tcb_status tcb_encoder_forward(const tcb_weights* w, const tcb_plan* plan,
                               const int32_t* d_segtab, const int32_t* d_token_ids,
                               void* d_rows, void* d_workspace, size_t workspace_bytes,
                               tcb_stream_t stream);

/* tcb_encoder_forward followed by tcb_unpack into d_out, with the unpack fused into the last
 * layer's FFN2 + LN2 where the L2-exchange LayerNorm GEMM runs (bf16, d in {512, 768, 1024}):
 * its epilogue writes each real slot's row to d_out[token_offset(seg) + position] (Concat of
 * Eq. (8)) instead of to d_rows, so the packed rows are not written back and read
 * again.  Elsewhere (fp32, other d) it is the two calls.  d_out as for tcb_unpack; d_rows is
 * used as the layer buffer and holds no defined result afterwards.  Graph replay as for
 * tcb_encoder_forward (d_out is part of the cache key). */
tcb_status tcb_encoder_forward_unpacked(const tcb_weights* w, const tcb_plan* plan,
                                        const int32_t* d_segtab, const int32_t* d_token_ids,
                                        void* d_rows, void* d_out, void* d_workspace,
                                        size_t workspace_bytes, tcb_stream_t stream);

/* unpack: out[token_offset(seg) + j] = rows[slot_start(seg) + j] for every segment -- the
 * per-request responses (Concat of Eq. (8)).  d_out is
 * [total_tokens, d_model] in the model dtype; rows of unplaced requests are not written. */
tcb_status tcb_unpack(const tcb_weights* w, const tcb_plan* plan, const int32_t* d_segtab,
                      const void* d_rows, void* d_out, tcb_stream_t stream);

/* Host buffers in, host buffers out (§8(b) with host data): a session owns the device side of
 * a fixed batch shape -- two slots of {segment table, token ids, rows, workspace, outputs}
 * in device memory and a pinned staging copy of the segment table -- all allocated by
 * tcb_session_create, none by tcb_session_run.
 *   num_rows, row_len : the batch shape every plan must have (a scheduler's B x L);
 *   max_tokens        : the largest total_tokens of a plan (outputs are [max_tokens, d]).
 * tcb_session_run(plan, h_token_ids, h_out) enqueues on `stream`, using the slots in turn:
 * the plan's segment table is written into the slot's pinned staging (waiting for that slot's
 * previous upload) and copied host->device with h_token_ids ([total_tokens] int32; pinned
 * memory makes the copies asynchronous) on a stream the session owns -- after the slot's
 * previous forward, so the upload overlaps the compute of the other slot -- then `stream`
 * waits for the upload and tcb_encoder_forward_unpacked runs, then the
 * per-request outputs are copied device->host into h_out ([total_tokens, d_model], model
 * dtype) -- on `copy_stream` when not NULL (after an event on `stream`, so the copy overlaps
 * the next call's compute), else on `stream`.  *ticket identifies the call;
 * tcb_session_wait(ticket) blocks the host until that call's outputs are in h_out.
 * Errors: a plan of another shape or with more than max_tokens tokens ->
 * TCB_ERR_INVALID_ARGUMENT; CUDA failures -> TCB_ERR_CUDA. */
typedef struct tcb_session tcb_session;
tcb_status tcb_session_create(const tcb_weights* w, int32_t num_rows, int32_t row_len,
                              int64_t max_tokens, tcb_session** out);
tcb_status tcb_session_run(tcb_session* s, const tcb_plan* plan, const int32_t* h_token_ids,
                           void* h_out, tcb_stream_t stream, tcb_stream_t copy_stream,
                           int64_t* ticket);
tcb_status tcb_session_wait(tcb_session* s, int64_t ticket);
void tcb_session_destroy(tcb_session* s);

/* ======================================================================================
 * 4. Instrumentation.
 * ==================================================================================== */
/* Number of kernel launches this library has issued since load (all threads). */
int64_t tcb_launch_count(void);

/* When enabled, tcb_encoder_forward / tcb_unpack record a CUDA event pair around every
 * kernel they launch (kernel classes below) on the launching stream; tcb_profile_collect
 * synchronises those events and adds their durations into ms[TCB_KCLASS_COUNT] and
 * launches[TCB_KCLASS_COUNT] (either may be NULL), then clears the record (and recycles its
 * events).  Under stream capture the pairs become external event-record nodes of the graph:
 * after each replay, tcb_profile_snapshot sums the same records WITHOUT clearing them (call
 * tcb_profile_collect once the graph will not be replayed again).  The event nodes serialise
 * the timed launches (no programmatic overlap across them). */
enum {
  TCB_K_EMBED = 0, TCB_K_GEMM_QKV = 1, TCB_K_ATTN = 2, TCB_K_GEMM_O = 3, TCB_K_LN = 4,
  TCB_K_GEMM_FFN1 = 5, TCB_K_GEMM_FFN2 = 6, TCB_K_UNPACK = 7, TCB_KCLASS_COUNT = 8
};
tcb_status tcb_profile_enable(int32_t on);
tcb_status tcb_profile_collect(double* ms, int64_t* launches);
tcb_status tcb_profile_snapshot(double* ms, int64_t* launches);

/* ======================================================================================
 * 5. Online request scheduling (host; §5; §8(f) row f2).
 *    Request n has arrival a_n, deadline d_n and length l_n; one batch of
 *    B rows x L words runs per time slot; utility v_n = 1/l_n counts only if n
 *    is scheduled inside [a_n, d_n] (Eq. (9)-(13)).  Per time slot the waiting
 *    set N_t (arrived, not yet scheduled, deadline not passed) is turned into
 *    one batch by:
 *      TCB_SCHED_DAS  Alg. 1 (§5.2): per row a utility-dominant
 *                     set N_U (the first p = max(1, floor(eta * s)) requests by utility,
 *                     s = how many of them fit the row), then the deadline-aware set N_D
 *                     (v >= q * mean v(N_U)) in deadline order, then the rest by utility,
 *                     each placed only if it fits; if everything left fits, it all goes
 *                     in (l.4-5).  eta + q = 1 gives the eta*q/(eta*q+1) competitive ratio
 *                     of Theorem 5.1 (1/5 at eta = q = 1/2).  Readings R27.
 *      TCB_SCHED_FCFS / _SJF / _DEF  the baselines of §6.2.4: arrival /
 *                     length / deadline order (ties: arrival, then id), First-Fit into
 *                     the B rows.
 *    Within a row, requests occupy consecutive columns from 0 in the order they are put in.
 * ==================================================================================== */
typedef enum {
  TCB_SCHED_DAS = 0,
  TCB_SCHED_FCFS = 1,
  TCB_SCHED_SJF = 2,
  TCB_SCHED_DEF = 3
} tcb_sched_policy;

/* One batch from a given waiting set (stateless).
 *   lengths/arrival/deadline/ids : [n] host arrays describing N_t (ids unique; they only
 *                                  break ties); every length in [1, L]
 *   B, L                         : batch rows and row length
 *   eta, q                       : DAS parameters in (0, 1] (ignored by the baselines)
 *   row, col                     : [n] outputs, -1 when the request is not in the batch
 * Errors: TCB_ERR_INVALID_ARGUMENT (bad sizes / NULL / policy / eta, q),
 *         TCB_ERR_REQUEST_TOO_LONG (a length > L). */
tcb_status tcb_sched_batch(int32_t policy, const int32_t* lengths, const double* arrival,
                           const double* deadline, const int64_t* ids, int32_t n, int32_t B,
                           int32_t L, double eta, double q, int32_t* row, int32_t* col);

/* Stateful online scheduler: a queue of submitted requests, one batch per time slot. */
typedef struct tcb_scheduler tcb_scheduler;
typedef struct {
  int64_t submitted;   /* requests ever submitted                                        */
  int64_t waiting;     /* in the queue now (arrived or not)                               */
  int64_t scheduled;   /* put into some batch (a response is produced)      */
  int64_t expired;     /* dropped at a slot start after their deadline (utility 0)       */
  int64_t batches;     /* tcb_sched_next_batch calls that succeeded                      */
  double utility;      /* sum of 1/l over scheduled requests: the objective (9)          */
} tcb_sched_stats;

/* batch_rows = B > 0, row_len = L > 0 and a multiple of 8; library-owned (destroy). */
tcb_status tcb_sched_create(int32_t policy, int32_t batch_rows, int32_t row_len, double eta,
                            double q, tcb_scheduler** out);
void tcb_sched_destroy(tcb_scheduler* sched);
/* Enqueue n requests (copied).  A length > row_len is TCB_ERR_REQUEST_TOO_LONG (nothing is
 * enqueued); deadline < arrival is TCB_ERR_INVALID_ARGUMENT. */
tcb_status tcb_sched_submit(tcb_scheduler* sched, int32_t n, const int64_t* ids,
                            const int32_t* lengths, const double* arrival,
                            const double* deadline);
/* The time slot starting at `now`: requests with deadline < now are dropped (expired);
 * N_t = queued requests with arrival <= now; the policy picks the batch, which leaves the
 * queue.  Outputs: ids_out / lengths_out [capacity] = the chosen requests in (row, column)
 * order, *n_out = their count; if plan_out != NULL, *plan_out = a new plan of exactly B rows
 * whose request order is that output order (gather the token ids in that order; empty rows
 * are all pad), ready for tcb_plan_write_segtab / tcb_encoder_forward (a fixed B x L shape,
 * so a captured CUDA graph can be replayed with each slot's segment table).  If capacity is
 * smaller than the batch, nothing is scheduled (expired requests are still dropped), *n_out =
 * the size needed and the status is TCB_ERR_INVALID_ARGUMENT. */
tcb_status tcb_sched_next_batch(tcb_scheduler* sched, double now, int64_t* ids_out,
                                int32_t* lengths_out, int32_t capacity, int32_t* n_out,
                                tcb_plan** plan_out);
tcb_status tcb_sched_stats_get(const tcb_scheduler* sched, tcb_sched_stats* out);

#ifdef __cplusplus
}
#endif
#endif /* TCB_H */
