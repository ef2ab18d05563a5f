/* oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Declarations of the float64 CPU oracle of the ConcatBatching encoder forward
 * (TCB, Fu et al., ICPP'22).  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load liboracle.so.  The product path
 * (paper_conf_icpp_fuc0z22_b200/) never includes, links or calls anything here, and this
 * file includes nothing from the product.  Citations "P:<line>" are lines of the paper
 * text; readings "R<k>" are listed in DESIGN.md §3.
 */
#ifndef TCB_ORACLE_H
#define TCB_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Return codes (same meaning as the product's, declared independently). */
#define ORACLE_OK 0
#define ORACLE_ERR_INVALID (-1)
#define ORACLE_ERR_TOO_LONG (-2)

/* Packing policies (R14, R17, R18). */
#define ORACLE_FIRST_FIT 0
#define ORACLE_NEXT_FIT 1
#define ORACLE_FIRST_FIT_DECREASING 2
#define ORACLE_NAIVE 3
#define ORACLE_LENGTH_SORTED 4

#define ORACLE_SCHED_DAS 0
#define ORACLE_SCHED_FCFS 1
#define ORACLE_SCHED_SJF 2
#define ORACLE_SCHED_DEF 3

typedef struct {
  int32_t num_layers, d_model, num_heads, d_ff;
  int32_t act;          /* 0 gelu (erf), 1 relu                          (R9)  */
  int32_t pe;           /* 0 sin_paper, 1 sin_vaswani, 2 learned         (R1, R4) */
  int32_t emb_ln;       /* BERT embedding LayerNorm                      (R5)  */
  int32_t use_type_emb; /* BERT token-type-0 embedding                   (R5)  */
  double ln_eps, emb_ln_eps, emb_scale;                               /* (R3, R10) */
} oracle_cfg;

int oracle_pack(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                int32_t policy, int32_t* req_row, int32_t* req_col, int32_t* num_rows);
/* o1, slotted ConcatBatching (§4.2, Alg. 2, R26): First-Fit over slots of z words. */
int oracle_pack_slotted(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                        int32_t slot_len, int32_t* req_row, int32_t* req_col, int32_t* num_rows,
                        int32_t* slot_len_used);
/* f2 (§5, Alg. 1, R27): one time slot's batch of B rows from the waiting set; row/col per
 * waiting request (-1 = not chosen).  policy: DAS 0, FCFS 1, SJF 2, DEF 3. */
int oracle_sched_batch(int32_t policy, const int32_t* lengths, const double* arrival,
                       const double* deadline, const int64_t* ids, int32_t n, int32_t B,
                       int32_t L, double eta, double q, int32_t* row, int32_t* col);

int oracle_layout(const int32_t* lengths, int32_t n, const int32_t* req_row,
                  const int32_t* req_col, int32_t num_rows, int32_t row_len, int32_t qtile,
                  int32_t* segment_ids, int32_t* positions, int32_t* tok_index,
                  int32_t* seg_req, int32_t* seg_start, int32_t* cu_seqlens,
                  int32_t* qtile_kv, int32_t* num_segments);

double oracle_pe(int32_t pos, int32_t dim, int32_t d_model, int32_t variant);

void oracle_embed(const oracle_cfg* cfg, const double* tok_emb, const double* pos_emb,
                  const double* type_emb, const double* emb_ln_g, const double* emb_ln_b,
                  const int32_t* ids, int32_t num_slots, const int32_t* segment_ids,
                  const int32_t* positions, const int32_t* tok_index, double* x);

void oracle_linear(const double* x, const double* w, const double* b, const double* res,
                   int32_t rows, int32_t n, int32_t k, int32_t act, double* y);

void oracle_attention(const double* qkv, const int32_t* segment_ids, int32_t num_rows,
                      int32_t row_len, int32_t d_model, int32_t num_heads, double* o);

void oracle_layernorm(const double* z, const double* g, const double* b, int32_t rows,
                      int32_t d, double eps, double* y);

int oracle_encoder(const oracle_cfg* cfg, const double* const* weights, int32_t num_weights,
                   const int32_t* ids, int32_t num_rows, int32_t row_len,
                   const int32_t* segment_ids, const int32_t* positions,
                   const int32_t* tok_index, double* x);

void oracle_unpack(const double* x, int32_t num_slots, int32_t d, const int32_t* tok_index,
                   double* out);

/* f4 decoder (§4.2.2; readings R30-R33).  dec weights: 20 per layer in the order
 * w_qkv b_qkv w_o b_o ln1_g ln1_b w_q b_q w_kv b_kv w_co b_co ln2_g ln2_b w_1 b_1 w_2 b_2
 * ln3_g ln3_b.  x [t, d] (embedded target prefix) is updated in place; mem [l, d]. */
int oracle_decoder_stack(const oracle_cfg* cfg, const double* const* w, int32_t num_w,
                         int32_t t, int32_t l, double* x, const double* mem);
int oracle_decode_greedy(const oracle_cfg* cfg, const double* const* enc_w, int32_t n_enc_w,
                         const double* const* dec_w, int32_t n_dec_w, int32_t vocab,
                         const int32_t* src, int32_t l, int32_t t_max, int32_t bos, int32_t eos,
                         int32_t* tokens, int32_t* n_out, double* logits);

#ifdef __cplusplus
}
#endif
#endif
