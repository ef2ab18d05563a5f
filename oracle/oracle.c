/* oracle.c -- TEST INFRASTRUCTURE ONLY: the float64 CPU oracle of the ConcatBatching
 * encoder forward (TCB, Fu et al., ICPP'22).  Plain, slow, obviously correct.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline, --impl reference) may
 * load this library.  It shares no code, header, table or helper with the CUDA path in
 * paper_conf_icpp_fuc0z22_b200/.  Citations "P:<line>" are lines of the paper text;
 * readings "R<k>" are DESIGN.md §3.
 *
 * Arithmetic rules: float64 throughout; every sum accumulates its terms in ascending index
 * order from 0.0; compiled with -O2 -ffp-contract=off (no FMA contraction, no fast-math);
 * libm exp/erf/sqrt/sin/cos/pow.  OpenMP only splits independent outputs (tokens, or
 * (row, head, query) triples), never a sum, so results do not depend on the thread count.
 *
 * Pins (tests/test_oracle_*.py): P1 brute-force slot scan + golden fixture F1 (layout),
 * P2 brute-force First-Fit + feasibility + FF<=1.7 OPT (pack), P3 closed-form PE,
 * P4 concat == alone bitwise (the method's correctness claim),
 * P5 textbook SDPA (attention), P6 torch.nn.TransformerEncoderLayer f64 (layer stack),
 * P7 cross-policy agreement, P8 identities, P9 brute-force tile enumeration.
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------------------ */
/* o1: packing.  A request n of length l_n is put in one row k (x^{tk}_n = 1)  */
/* at most once (constraint (10)) and every row holds at most L words         */
/* (constraint (11)).  The paper "greedily put[s]" requests into the current  */
/* batch row (Alg. 1); reading R14 makes that First-Fit in input order.       */
/* ------------------------------------------------------------------------------------ */

static const int32_t* g_sort_len; /* comparator context (single-threaded use) */
static int g_sort_desc;

static int cmp_by_length(const void* a, const void* b) {
  int32_t i = *(const int32_t*)a, j = *(const int32_t*)b;
  int32_t li = g_sort_len[i], lj = g_sort_len[j];
  if (li != lj) return g_sort_desc ? (lj > li ? 1 : -1) : (li > lj ? 1 : -1);
  return (i > j) - (i < j); /* ties by input index: a stable order */
}

int oracle_pack(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                int32_t policy, int32_t* req_row, int32_t* req_col, int32_t* num_rows) {
  if (n < 0 || row_len <= 0 || max_rows < 0 || policy < 0 || policy > 4) return ORACLE_ERR_INVALID;
  if (n > 0 && (!lengths || !req_row || !req_col)) return ORACLE_ERR_INVALID;
  if (!num_rows) return ORACLE_ERR_INVALID;
  for (int32_t i = 0; i < n; ++i) {
    if (lengths[i] <= 0) return ORACLE_ERR_INVALID;
    if (lengths[i] > row_len) return ORACLE_ERR_TOO_LONG; /* R15: constraint (11) */
  }
  /* processing order */
  int32_t* order = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  for (int32_t i = 0; i < n; ++i) order[i] = i;
  if (policy == ORACLE_FIRST_FIT_DECREASING || policy == ORACLE_LENGTH_SORTED) {
    g_sort_len = lengths;
    g_sort_desc = (policy == ORACLE_FIRST_FIT_DECREASING);
    qsort(order, (size_t)n, sizeof(int32_t), cmp_by_length);
  }
  int32_t* fill = (int32_t*)calloc((size_t)(n > 0 ? n : 1), sizeof(int32_t));
  int32_t rows = 0;
  int32_t current = -1; /* Next-Fit's open row */
  const int32_t cap = (max_rows == 0) ? n : max_rows;
  for (int32_t t = 0; t < n; ++t) {
    const int32_t r = order[t];
    const int32_t l = lengths[r];
    int32_t row = -1;
    if (policy == ORACLE_FIRST_FIT || policy == ORACLE_FIRST_FIT_DECREASING) {
      for (int32_t k = 0; k < rows; ++k) /* lowest-index row with room */
        if (row_len - fill[k] >= l) { row = k; break; }
      if (row < 0 && rows < cap) row = rows++;
    } else if (policy == ORACLE_NEXT_FIT) {
      if (current >= 0 && row_len - fill[current] >= l) row = current;
      else if (rows < cap) { row = rows++; current = row; }
    } else { /* NAIVE / LENGTH_SORTED: one request per row (R17, R18) */
      if (rows < cap) row = rows++;
    }
    if (row >= 0) {
      req_row[r] = row;
      req_col[r] = fill[row];
      fill[row] += l;
    } else {
      req_row[r] = -1; /* R16: unplaced */
      req_col[r] = -1;
    }
  }
  *num_rows = rows;
  free(order);
  free(fill);
  return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* o1 (slotted ConcatBatching, §4.2; Alg. 2; reading R26).         */
/* Each row of L words is divided into floor(L / z) slots of z words ("Divide each row of */
/* the batch into multiple slots based on the slot size z", Alg. 2 l.5); the tail        */
/* L - floor(L/z)*z is unused.  Requests are put into slots greedily (Alg. 2 l.7): in    */
/* input order, each request goes to the first slot (rows in order, slots left to right) */
/* whose residual is >= its length; if none, a new row is opened (while rows < max_rows, */
/* 0 = unbounded), else it is deferred (req_row = -1).  A request never straddles a slot */
/* boundary; within a slot requests are contiguous from the slot start in placement      */
/* order.  z = 0 selects z = the largest request length (Alg. 2 l.4 with H_U = all       */
/* requests).  z == L is pure ConcatBatching First-Fit ("a special case whose slot size  */
/* is equal to the batch length L").                                        */
/* ------------------------------------------------------------------------------------ */
int oracle_pack_slotted(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                        int32_t slot_len, int32_t* req_row, int32_t* req_col, int32_t* num_rows,
                        int32_t* slot_len_used) {
  if (n < 0 || row_len <= 0 || max_rows < 0 || slot_len < 0 || slot_len > row_len)
    return ORACLE_ERR_INVALID;
  if (n > 0 && (!lengths || !req_row || !req_col)) return ORACLE_ERR_INVALID;
  if (!num_rows || !slot_len_used) return ORACLE_ERR_INVALID;
  int32_t z = slot_len;
  for (int32_t i = 0; i < n; ++i) {
    if (lengths[i] <= 0) return ORACLE_ERR_INVALID;
    if (lengths[i] > row_len) return ORACLE_ERR_TOO_LONG;
  }
  if (z == 0) {
    for (int32_t i = 0; i < n; ++i) if (lengths[i] > z) z = lengths[i];
    if (z == 0) z = row_len; /* no requests */
  }
  const int32_t per_row = row_len / z;
  const int32_t cap = (max_rows == 0) ? n : max_rows;
  /* fill[row * per_row + j] = words used in slot j of row */
  int32_t* fill = (int32_t*)calloc((size_t)(n > 0 ? n : 1) * (size_t)per_row, sizeof(int32_t));
  int32_t rows = 0;
  for (int32_t r = 0; r < n; ++r) {
    const int32_t l = lengths[r];
    int32_t slot = -1;
    if (l <= z) {
      for (int32_t s = 0; s < rows * per_row; ++s)
        if (z - fill[s] >= l) { slot = s; break; }
      if (slot < 0 && rows < cap) { slot = rows * per_row; ++rows; }
    }
    if (slot >= 0) {
      req_row[r] = slot / per_row;
      req_col[r] = (slot % per_row) * z + fill[slot];
      fill[slot] += l;
    } else {
      req_row[r] = -1; /* deferred (R26) */
      req_col[r] = -1;
    }
  }
  *num_rows = rows;
  *slot_len_used = z;
  free(fill);
  return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* §8(f) f2: request scheduling (§5).  One time slot's batch H_t of B rows chosen from the  */
/* waiting set N_t (requests arrived, not yet scheduled, deadline not passed; the caller    */
/* passes exactly that set).  Utility v_n = 1 / l_n.              */
/* ORACLE_SCHED_DAS follows Alg. 1 (§5.2) line by line, with the   */
/* readings R27 of DESIGN.md:                                                              */
/*   - rows k = 0..B-1 in order; a request placed in a row leaves N_t (constraint (10));   */
/*   - l.4-5: if the remaining requests fit the row, all of them go in, in N_t order      */
/*     (arrival, then id);                                                                 */
/*   - l.7: utility order = v non-increasing = length ascending, ties by arrival then id; */
/*   - l.8: s = the largest prefix count of that order whose lengths sum to <= L;        */
/*   - l.9: p = max(1, floor(eta * s)) (p_tk = eta s_tk, and p >= 1);       */
/*   - l.11: N_D = requests after the first p whose v >= q * mean(v over N_U) ("no less   */
/*     than"), evaluated in double as 1.0/l >= q * (sum(1.0/l) / p), the sum */
/*     in utility order;                                                                   */
/*   - l.12: N_D in deadline order (ties arrival, id), each placed if it still fits;     */
/*   - l.13-14: then the rest (utility order), each placed if it still fits.             */
/* Within a row, requests occupy columns in the order they are put in.  The baselines of */
/* §6.2.4 put requests in their priority order into the first row with room */
/* (First-Fit): FCFS = arrival order, SJF = length ascending, DEF = deadline ascending     */
/* (ties: arrival, then id).                                                               */
/* ------------------------------------------------------------------------------------ */
typedef struct {
  const int32_t* len;
  const double* arr;
  const double* dl;
  const int64_t* id;
  int key; /* 0 = arrival, 1 = length (utility), 2 = deadline */
} sched_ctx;

static int sched_before(const sched_ctx* c, int32_t a, int32_t b) {
  if (c->key == 1 && c->len[a] != c->len[b]) return c->len[a] < c->len[b];
  if (c->key == 2 && c->dl[a] != c->dl[b]) return c->dl[a] < c->dl[b];
  if (c->arr[a] != c->arr[b]) return c->arr[a] < c->arr[b];
  return c->id[a] < c->id[b];
}

/* plain insertion sort of idx[0..m) by the context key (stable, obviously correct) */
static void sched_sort(const sched_ctx* c, int32_t* idx, int32_t m) {
  for (int32_t i = 1; i < m; ++i) {
    int32_t v = idx[i], j = i - 1;
    while (j >= 0 && sched_before(c, v, idx[j])) { idx[j + 1] = idx[j]; --j; }
    idx[j + 1] = v;
  }
}

int oracle_sched_batch(int32_t policy, const int32_t* lengths, const double* arrival,
                       const double* deadline, const int64_t* ids, int32_t n, int32_t B,
                       int32_t L, double eta, double q, int32_t* row, int32_t* col) {
  if (n < 0 || B < 0 || L <= 0 || policy < 0 || policy > 3) return ORACLE_ERR_INVALID;
  if (n > 0 && (!lengths || !arrival || !deadline || !ids || !row || !col)) return ORACLE_ERR_INVALID;
  for (int32_t i = 0; i < n; ++i) {
    if (lengths[i] <= 0) return ORACLE_ERR_INVALID;
    if (lengths[i] > L) return ORACLE_ERR_TOO_LONG;
    row[i] = -1;
    col[i] = -1;
  }
  sched_ctx c = {lengths, arrival, deadline, ids, 0};
  int32_t* idx = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  if (policy != ORACLE_SCHED_DAS) {
    int32_t* used = (int32_t*)calloc((size_t)(B > 0 ? B : 1), sizeof(int32_t));
    for (int32_t i = 0; i < n; ++i) idx[i] = i;
    c.key = policy == ORACLE_SCHED_FCFS ? 0 : (policy == ORACLE_SCHED_SJF ? 1 : 2);
    sched_sort(&c, idx, n);
    for (int32_t t = 0; t < n; ++t) {
      const int32_t r = idx[t];
      for (int32_t k = 0; k < B; ++k)
        if (used[k] + lengths[r] <= L) {
          row[r] = k; col[r] = used[k]; used[k] += lengths[r];
          break;
        }
    }
    free(used);
    free(idx);
    return ORACLE_OK;
  }
  for (int32_t k = 0; k < B; ++k) {
    /* N_t: the requests not placed yet */
    int32_t m = 0;
    int64_t total = 0;
    for (int32_t i = 0; i < n; ++i)
      if (row[i] < 0) { idx[m++] = i; total += lengths[i]; }
    if (m == 0) break;
    int32_t used = 0;
    if (total <= L) {                               /* l.4-5 */
      c.key = 0;
      sched_sort(&c, idx, m);
      for (int32_t t = 0; t < m; ++t) {
        row[idx[t]] = k; col[idx[t]] = used; used += lengths[idx[t]];
      }
      continue;
    }
    c.key = 1;                                      /* l.7: utility order */
    sched_sort(&c, idx, m);
    int32_t s = 0;                                  /* l.8 */
    int64_t pre = 0;
    while (s < m && pre + lengths[idx[s]] <= L) { pre += lengths[idx[s]]; ++s; }
    int32_t p = (int32_t)floor(eta * (double)s);    /* l.9 */
    if (p < 1) p = 1;
    double vsum = 0.0;
    for (int32_t t = 0; t < p; ++t) {               /* l.10: N_U into the row */
      const int32_t r = idx[t];
      row[r] = k; col[r] = used; used += lengths[r];
      vsum += 1.0 / (double)lengths[r];
    }
    const double thr = q * (vsum / (double)p);
    int32_t* nd = (int32_t*)malloc(sizeof(int32_t) * (size_t)m);
    int32_t nnd = 0;
    for (int32_t t = p; t < m; ++t)                 /* l.11: N_D */
      if (1.0 / (double)lengths[idx[t]] >= thr) nd[nnd++] = idx[t];
    c.key = 2;                                      /* l.12: deadline order, greedy */
    sched_sort(&c, nd, nnd);
    for (int32_t t = 0; t < nnd; ++t) {
      const int32_t r = nd[t];
      if (used + lengths[r] <= L) { row[r] = k; col[r] = used; used += lengths[r]; }
    }
    for (int32_t t = p; t < m; ++t) {               /* l.13-14: the rest, utility order */
      const int32_t r = idx[t];
      int in_nd = 0;
      for (int32_t u = 0; u < nnd; ++u) if (nd[u] == r) in_nd = 1;
      if (in_nd || row[r] >= 0) continue;
      if (used + lengths[r] <= L) { row[r] = k; col[r] = used; used += lengths[r]; }
    }
    free(nd);
  }
  free(idx);
  return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* o1 (layout): per-slot metadata of the packed rows.  Segments are numbered globally in  */
/* (row, column) order (R13); pad slots have segment -1, position -1, tok_index -1 (R12). */
/* Positions restart at 0 at each request's first token: separate PE, R2.     */
/* ------------------------------------------------------------------------------------ */
int oracle_layout(const int32_t* lengths, int32_t n, const int32_t* req_row,
                  const int32_t* req_col, int32_t num_rows, int32_t row_len, int32_t qtile,
                  int32_t* segment_ids, int32_t* positions, int32_t* tok_index,
                  int32_t* seg_req, int32_t* seg_start, int32_t* cu_seqlens,
                  int32_t* qtile_kv, int32_t* num_segments) {
  if (n < 0 || num_rows < 0 || row_len <= 0 || qtile <= 0) return ORACLE_ERR_INVALID;
  const int64_t M = (int64_t)num_rows * row_len;
  /* request-order token offsets over ALL requests (placed or not) */
  int64_t* cu_req = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  cu_req[0] = 0;
  for (int32_t r = 0; r < n; ++r) cu_req[r + 1] = cu_req[r] + lengths[r];
  /* which request covers each slot: a direct scan over requests */
  int32_t* owner = (int32_t*)malloc(sizeof(int32_t) * (size_t)(M > 0 ? M : 1));
  for (int64_t s = 0; s < M; ++s) owner[s] = -1;
  for (int32_t r = 0; r < n; ++r) {
    if (req_row[r] < 0) continue;
    for (int32_t j = 0; j < lengths[r]; ++j)
      owner[(int64_t)req_row[r] * row_len + req_col[r] + j] = r;
  }
  /* walk slots in flattened (row, column) order; a new segment starts wherever the owner
   * changes to a request (requests are contiguous, and two requests never share a slot) */
  int32_t S = 0;
  int32_t compact = 0;
  cu_seqlens[0] = 0;
  for (int64_t s = 0; s < M; ++s) {
    const int32_t r = owner[s];
    if (r < 0) {
      segment_ids[s] = -1; positions[s] = -1; tok_index[s] = -1;
      continue;
    }
    const int64_t col = s % row_len;
    if (col == req_col[r]) { /* first token of request r */
      seg_req[S] = r;
      seg_start[S] = (int32_t)s;
      ++S;
      cu_seqlens[S] = cu_seqlens[S - 1] + lengths[r];
    }
    segment_ids[s] = S - 1;
    positions[s] = (int32_t)(col - req_col[r]);
    tok_index[s] = (int32_t)(cu_req[r] + positions[s]);
    ++compact;
  }
  *num_segments = S;
  /* q-tiles of `qtile` flattened slots: [start of the segment of the first real slot,
   * end of the segment of the last real slot); -1,-1 if the tile holds no real slot. */
  const int64_t ntiles = (M + qtile - 1) / qtile;
  for (int64_t t = 0; t < ntiles; ++t) {
    int64_t lo = -1, hi = -1;
    for (int64_t s = t * qtile; s < M && s < (t + 1) * qtile; ++s) {
      if (segment_ids[s] < 0) continue;
      const int32_t sg = segment_ids[s];
      const int64_t st = seg_start[sg];
      const int64_t en = st + lengths[seg_req[sg]];
      if (lo < 0) lo = st;
      hi = en;
    }
    qtile_kv[2 * t] = (int32_t)lo;
    qtile_kv[2 * t + 1] = (int32_t)hi;
  }
  free(owner);
  free(cu_req);
  (void)compact;
  return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* o2: embedding + separate positional encoding.                                         */
/* Eq. (1): PE(pos, 2e)   = sin(pos / 10000^(2e/d_model))           */
/* Eq. (2): PE(pos, 2e+1) = cos(pos / 10000^((2e+1)/d_model))      (R1 literal) */
/* variant 1 (sin_vaswani) uses 2e/d_model in both.                                      */
/* ------------------------------------------------------------------------------------ */
double oracle_pe(int32_t pos, int32_t dim, int32_t d_model, int32_t variant) {
  const int32_t e = dim / 2;
  if (dim % 2 == 0) return sin((double)pos / pow(10000.0, (double)(2 * e) / d_model));
  const double expo = (variant == 0) ? (double)(2 * e + 1) / d_model : (double)(2 * e) / d_model;
  return cos((double)pos / pow(10000.0, expo));
}

static void layernorm_row(const double* z, const double* g, const double* b, int32_t d,
                          double eps, double* y) {
  double mean = 0.0;
  for (int32_t c = 0; c < d; ++c) mean += z[c];
  mean /= d;
  double var = 0.0;
  for (int32_t c = 0; c < d; ++c) var += (z[c] - mean) * (z[c] - mean);
  var /= d; /* biased variance (R10) */
  const double inv = 1.0 / sqrt(var + eps);
  for (int32_t c = 0; c < d; ++c) y[c] = (z[c] - mean) * inv * g[c] + b[c];
}

void oracle_embed(const oracle_cfg* cfg, const double* tok_emb, const double* pos_emb,
                  const double* type_emb, const double* emb_ln_g, const double* emb_ln_b,
                  const int32_t* ids, int32_t num_slots, const int32_t* segment_ids,
                  const int32_t* positions, const int32_t* tok_index, double* x) {
  const int32_t d = cfg->d_model;
#pragma omp parallel for schedule(static)
  for (int32_t s = 0; s < num_slots; ++s) {
    double* xs = x + (int64_t)s * d;
    if (segment_ids[s] < 0) { /* pad slot: zeros (R12) */
      for (int32_t c = 0; c < d; ++c) xs[c] = 0.0;
      continue;
    }
    const int32_t id = ids[tok_index[s]];
    const int32_t pos = positions[s];
    for (int32_t c = 0; c < d; ++c) {
      double v = tok_emb[(int64_t)id * d + c] * cfg->emb_scale;
      if (cfg->pe == 2) v += pos_emb[(int64_t)pos * d + c];  /* learned, restarted pos (R4) */
      else v += oracle_pe(pos, c, d, cfg->pe);
      if (cfg->use_type_emb) v += type_emb[c];
      xs[c] = v;
    }
    if (cfg->emb_ln) {
      double tmp[8192];
      layernorm_row(xs, emb_ln_g, emb_ln_b, d, cfg->emb_ln_eps, tmp);
      for (int32_t c = 0; c < d; ++c) xs[c] = tmp[c];
    }
  }
}

/* ------------------------------------------------------------------------------------ */
/* o3/o5/o6: y = act(x W^T + b) (+ res).  Eq. (3) Q = X W_Q with W stored [n, k] */
/* (output feature major); biases per R8; act 0 none, 1 gelu(erf), 2 relu (R9).          */
/* ------------------------------------------------------------------------------------ */
void oracle_linear(const double* x, const double* w, const double* b, const double* res,
                   int32_t rows, int32_t n, int32_t k, int32_t act, double* y) {
#pragma omp parallel for schedule(static)
  for (int32_t t = 0; t < rows; ++t) {
    for (int32_t o = 0; o < n; ++o) {
      double acc = 0.0;
      for (int32_t i = 0; i < k; ++i) acc += x[(int64_t)t * k + i] * w[(int64_t)o * k + i];
      acc = acc + b[o];
      if (act == 1) acc = 0.5 * acc * (1.0 + erf(acc / sqrt(2.0)));
      else if (act == 2) acc = acc > 0.0 ? acc : 0.0;
      if (res) acc = acc + res[(int64_t)t * n + o];
      y[(int64_t)t * n + o] = acc;
    }
  }
}

/* ------------------------------------------------------------------------------------ */
/* o4: customized self-attention, Eq. (5)-(6):                               */
/*   Att_CB(Q,K,V) = softmax(Q K^T / sqrt(d) + M) V,  M = 0 on the diagonal blocks        */
/*   Q_i K_i^T and -inf elsewhere.  Per head h (columns [h dh, (h+1) dh) of Q/K/V, R7),   */
/*   sqrt(d) with d = dh (R6).  Keys j run over the WHOLE batch row in ascending order;   */
/*   a masked score is -inf, so p_ij = exp(-inf - m) = 0 exactly (R11).  Pad queries      */
/*   produce 0 (R12).  qkv is [slots, 3 d_model] = [Q | K | V].                           */
/* ------------------------------------------------------------------------------------ */
void oracle_attention(const double* qkv, const int32_t* segment_ids, int32_t num_rows,
                      int32_t row_len, int32_t d_model, int32_t num_heads, double* o) {
  const int32_t dh = d_model / num_heads;
  const int64_t ld = 3 * (int64_t)d_model;
  const double scale = sqrt((double)dh);
  const int64_t total = (int64_t)num_rows * num_heads * row_len;
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t job = 0; job < total; ++job) {
    const int32_t row = (int32_t)(job / ((int64_t)num_heads * row_len));
    const int32_t h = (int32_t)((job / row_len) % num_heads);
    const int32_t i = (int32_t)(job % row_len);
    const int64_t qi = (int64_t)row * row_len + i;
    double* oi = o + qi * d_model + (int64_t)h * dh;
    if (segment_ids[qi] < 0) {
      for (int32_t c = 0; c < dh; ++c) oi[c] = 0.0;
      continue;
    }
    double* s = (double*)malloc(sizeof(double) * (size_t)row_len);
    double m = -INFINITY;
    for (int32_t j = 0; j < row_len; ++j) {
      const int64_t kj = (int64_t)row * row_len + j;
      if (segment_ids[kj] != segment_ids[qi]) { s[j] = -INFINITY; continue; } /* M = -inf */
      double dot = 0.0;
      for (int32_t c = 0; c < dh; ++c)
        dot += qkv[qi * ld + (int64_t)h * dh + c] * qkv[kj * ld + d_model + (int64_t)h * dh + c];
      s[j] = dot / scale;
      if (s[j] > m) m = s[j];
    }
    double den = 0.0;
    for (int32_t j = 0; j < row_len; ++j) {
      s[j] = exp(s[j] - m); /* exp(-inf) = 0 exactly */
      den += s[j];
    }
    for (int32_t c = 0; c < dh; ++c) {
      double acc = 0.0;
      for (int32_t j = 0; j < row_len; ++j) {
        const int64_t kj = (int64_t)row * row_len + j;
        acc += (s[j] / den) * qkv[kj * ld + 2 * (int64_t)d_model + (int64_t)h * dh + c];
      }
      oi[c] = acc;
    }
    free(s);
  }
}

void oracle_layernorm(const double* z, const double* g, const double* b, int32_t rows,
                      int32_t d, double eps, double* y) {
#pragma omp parallel for schedule(static)
  for (int32_t t = 0; t < rows; ++t) layernorm_row(z + (int64_t)t * d, g, b, d, eps, y + (int64_t)t * d);
}

/* ------------------------------------------------------------------------------------ */
/* o2..o7: the encoder stack of S layers, each: self-attention (masked, Eq. 5) */
/* -> W_O + residual -> LN1 -> FFN + residual -> LN2  (post-LN, R10).          */
/* weights: tok_emb, pos_emb, type_emb, emb_ln_g, emb_ln_b, then per layer                 */
/* w_qkv, b_qkv, w_o, b_o, ln1_g, ln1_b, w_1, b_1, w_2, b_2, ln2_g, ln2_b.                 */
/* x: out [num_rows*row_len, d_model]; pad slots hold whatever the layer math gives them   */
/* except that they are forced to 0 (they are never read as keys: R12).                    */
/* ------------------------------------------------------------------------------------ */
int oracle_encoder(const oracle_cfg* cfg, const double* const* weights, int32_t num_weights,
                   const int32_t* ids, int32_t num_rows, int32_t row_len,
                   const int32_t* segment_ids, const int32_t* positions,
                   const int32_t* tok_index, double* x) {
  if (num_weights != 5 + 12 * cfg->num_layers) return ORACLE_ERR_INVALID;
  const int32_t d = cfg->d_model, f = cfg->d_ff;
  const int32_t M = num_rows * row_len;
  if (M == 0) return ORACLE_OK;
  double* qkv = (double*)malloc(sizeof(double) * (size_t)M * 3 * d);
  double* att = (double*)malloc(sizeof(double) * (size_t)M * d);
  double* z = (double*)malloc(sizeof(double) * (size_t)M * d);
  double* x1 = (double*)malloc(sizeof(double) * (size_t)M * d);
  double* h = (double*)malloc(sizeof(double) * (size_t)M * f);
  oracle_embed(cfg, weights[0], weights[1], weights[2], weights[3], weights[4], ids, M,
               segment_ids, positions, tok_index, x);
  const int32_t act = cfg->act == 0 ? 1 : 2;
  for (int32_t layer = 0; layer < cfg->num_layers; ++layer) {
    const double* const* W = weights + 5 + 12 * layer;
    oracle_linear(x, W[0], W[1], NULL, M, 3 * d, d, 0, qkv);               /* Eq. (3) */
    oracle_attention(qkv, segment_ids, num_rows, row_len, d, cfg->num_heads, att); /* (5) */
    oracle_linear(att, W[2], W[3], x, M, d, d, 0, z);                      /* W_O + res */
    oracle_layernorm(z, W[4], W[5], M, d, cfg->ln_eps, x1);                /* LN1 */
    oracle_linear(x1, W[6], W[7], NULL, M, f, d, act, h);                  /* FFN1 + act */
    oracle_linear(h, W[8], W[9], x1, M, d, f, 0, z);                       /* FFN2 + res */
    oracle_layernorm(z, W[10], W[11], M, d, cfg->ln_eps, x);               /* LN2 */
    for (int32_t s = 0; s < M; ++s)
      if (segment_ids[s] < 0)
        for (int32_t c = 0; c < d; ++c) x[(int64_t)s * d + c] = 0.0;
  }
  free(qkv); free(att); free(z); free(x1); free(h);
  return ORACLE_OK;
}

/* o8: scatter each real slot back to its request-order token index (P:752-754 Concat). */
void oracle_unpack(const double* x, int32_t num_slots, int32_t d, const int32_t* tok_index,
                   double* out) {
  for (int32_t s = 0; s < num_slots; ++s) {
    if (tok_index[s] < 0) continue;
    memcpy(out + (int64_t)tok_index[s] * d, x + (int64_t)s * d, sizeof(double) * (size_t)d);
  }
}

/* ---------------------------------------------------------------------------------------
 * f4: the decoder of the paper's Seq2Seq setting.  "These embeddings are sent
 * to the encoder and decoder, each of which contains S layers ... Decoder outputs go
 * through a final linear layer and activation function to generate final results"
 * (P:340-351); the decoder "is an auto-regressive model" (§4.2.2).  Readings
 * R30-R33: standard post-LN decoder layer of [32] (causal self-attention,
 * cross-attention over the request's OWN encoder output -- the segment-aware form --, FFN),
 * target tokens embedded like the source (tied E_tok, separate PE restarting at 0 per
 * request), output projection tied to E_tok without bias, greedy argmax (lowest index on
 * ties), BOS = 1, EOS = 2, at most t_max generated tokens.
 * Plain definition: every step recomputes the whole target prefix (no KV cache).
 * ------------------------------------------------------------------------------------- */

/* softmax(Q K^T / sqrt(dh)) V per head for tq queries over tk keys; causal: query i sees
 * keys j <= i + causal_off only (masked terms are -inf -> exp = 0 exactly, R11). */
static void attend(const double* q, int64_t ldq, const double* k, const double* v, int64_t ldkv,
                   int32_t tq, int32_t tk, int32_t d_model, int32_t num_heads, int32_t causal,
                   double* o) {
  const int32_t dh = d_model / num_heads;
  const double scale = sqrt((double)dh);
  double* s = (double*)malloc(sizeof(double) * (size_t)(tk > 0 ? tk : 1));
  for (int32_t h = 0; h < num_heads; ++h) {
    for (int32_t i = 0; i < tq; ++i) {
      double m = -INFINITY;
      for (int32_t j = 0; j < tk; ++j) {
        if (causal && j > i) { s[j] = -INFINITY; continue; }
        double dot = 0.0;
        for (int32_t c = 0; c < dh; ++c)
          dot += q[(int64_t)i * ldq + (int64_t)h * dh + c] * k[(int64_t)j * ldkv + (int64_t)h * dh + c];
        s[j] = dot / scale;
        if (s[j] > m) m = s[j];
      }
      double den = 0.0;
      for (int32_t j = 0; j < tk; ++j) {
        s[j] = exp(s[j] - m);
        den += s[j];
      }
      for (int32_t c = 0; c < dh; ++c) {
        double acc = 0.0;
        for (int32_t j = 0; j < tk; ++j)
          acc += (s[j] / den) * v[(int64_t)j * ldkv + (int64_t)h * dh + c];
        o[(int64_t)i * d_model + (int64_t)h * dh + c] = acc;
      }
    }
  }
  free(s);
}

int oracle_decoder_stack(const oracle_cfg* cfg, const double* const* w, int32_t num_w,
                         int32_t t, int32_t l, double* x, const double* mem) {
  if (num_w != 20 * cfg->num_layers || t <= 0 || l <= 0) return ORACLE_ERR_INVALID;
  const int32_t d = cfg->d_model, f = cfg->d_ff;
  double* qkv = (double*)malloc(sizeof(double) * (size_t)t * 3 * d);
  double* qc = (double*)malloc(sizeof(double) * (size_t)t * d);
  double* kv = (double*)malloc(sizeof(double) * (size_t)l * 2 * d);
  double* att = (double*)malloc(sizeof(double) * (size_t)t * d);
  double* z = (double*)malloc(sizeof(double) * (size_t)t * d);
  double* x1 = (double*)malloc(sizeof(double) * (size_t)t * d);
  double* x2 = (double*)malloc(sizeof(double) * (size_t)t * d);
  double* h = (double*)malloc(sizeof(double) * (size_t)t * f);
  const int32_t act = cfg->act == 0 ? 1 : 2;
  for (int32_t layer = 0; layer < cfg->num_layers; ++layer) {
    const double* const* W = w + 20 * layer;
    /* causal self-attention over the request's own target prefix */
    oracle_linear(x, W[0], W[1], NULL, t, 3 * d, d, 0, qkv);
    attend(qkv, 3 * (int64_t)d, qkv + d, qkv + 2 * d, 3 * (int64_t)d, t, t, d, cfg->num_heads, 1, att);
    oracle_linear(att, W[2], W[3], x, t, d, d, 0, z);
    oracle_layernorm(z, W[4], W[5], t, d, cfg->ln_eps, x1);
    /* cross-attention over the request's own encoder output (segment-aware) */
    oracle_linear(x1, W[6], W[7], NULL, t, d, d, 0, qc);
    oracle_linear(mem, W[8], W[9], NULL, l, 2 * d, d, 0, kv);
    attend(qc, d, kv, kv + d, 2 * (int64_t)d, t, l, d, cfg->num_heads, 0, att);
    oracle_linear(att, W[10], W[11], x1, t, d, d, 0, z);
    oracle_layernorm(z, W[12], W[13], t, d, cfg->ln_eps, x2);
    /* FFN */
    oracle_linear(x2, W[14], W[15], NULL, t, f, d, act, h);
    oracle_linear(h, W[16], W[17], x2, t, d, f, 0, z);
    oracle_layernorm(z, W[18], W[19], t, d, cfg->ln_eps, x);
  }
  free(qkv); free(qc); free(kv); free(att); free(z); free(x1); free(x2); free(h);
  return ORACLE_OK;
}

/* Greedy decode of ONE request run alone (no padding, no other request): encoder over its
 * l source tokens, then up to t_max steps of the decoder on the full prefix BOS y_1..y_k;
 * y_{k+1} = argmax over the vocabulary of x_last . E_tok^T (lowest index on ties); stops
 * after EOS.  tokens[0..n_out) = y_1..; logits (nullable) [t_max, vocab] per step. */
int oracle_decode_greedy(const oracle_cfg* cfg, const double* const* enc_w, int32_t n_enc_w,
                         const double* const* dec_w, int32_t n_dec_w, int32_t vocab,
                         const int32_t* src, int32_t l, int32_t t_max, int32_t bos, int32_t eos,
                         int32_t* tokens, int32_t* n_out, double* logits) {
  if (l <= 0 || t_max <= 0 || vocab <= 0) return ORACLE_ERR_INVALID;
  const int32_t d = cfg->d_model;
  int32_t* seg = (int32_t*)malloc(sizeof(int32_t) * (size_t)l);
  int32_t* pos = (int32_t*)malloc(sizeof(int32_t) * (size_t)l);
  int32_t* tok = (int32_t*)malloc(sizeof(int32_t) * (size_t)l);
  for (int32_t i = 0; i < l; ++i) { seg[i] = 0; pos[i] = i; tok[i] = i; }
  double* mem = (double*)malloc(sizeof(double) * (size_t)l * d);
  int rc = oracle_encoder(cfg, enc_w, n_enc_w, src, 1, l, seg, pos, tok, mem);
  int32_t* y = (int32_t*)malloc(sizeof(int32_t) * (size_t)(t_max + 1));
  double* x = (double*)malloc(sizeof(double) * (size_t)(t_max + 1) * d);
  double* lg = (double*)malloc(sizeof(double) * (size_t)vocab);
  const double* E = enc_w[0];
  y[0] = bos;
  int32_t k = 0;
  while (rc == ORACLE_OK && k < t_max) {
    const int32_t t = k + 1;                               /* prefix length incl. BOS */
    for (int32_t i = 0; i < t; ++i)                        /* embed: E[y_i] * scale + PE(i) */
      for (int32_t c = 0; c < d; ++c) {
        const double pe = cfg->pe == 2 ? enc_w[1][(int64_t)i * d + c] : oracle_pe(i, c, d, cfg->pe);
        x[(int64_t)i * d + c] = E[(int64_t)y[i] * d + c] * cfg->emb_scale + pe;
      }
    rc = oracle_decoder_stack(cfg, dec_w, n_dec_w, t, l, x, mem);
    if (rc != ORACLE_OK) break;
    const double* xl = x + (int64_t)(t - 1) * d;
    int32_t best = 0;
    for (int32_t v = 0; v < vocab; ++v) {
      double acc = 0.0;
      for (int32_t c = 0; c < d; ++c) acc += xl[c] * E[(int64_t)v * d + c];
      lg[v] = acc;
      if (acc > lg[best]) best = v;
    }
    if (logits)
      for (int32_t v = 0; v < vocab; ++v) logits[(int64_t)k * vocab + v] = lg[v];
    y[t] = best;
    tokens[k] = best;
    ++k;
    if (best == eos) break;
  }
  *n_out = k;
  free(seg); free(pos); free(tok); free(mem); free(y); free(x); free(lg);
  return rc;
}
