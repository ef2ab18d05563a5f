// pack.cpp -- host packer of libtcb: tcb_pack and the plan accessors (include/tcb.h §1).
//
// ConcatBatching puts several requests end to end in one batch row of L words with padding
// only at the tail (Fig. 1(c); §4.1), subject to constraint (10) (each
// request at most once) and (11) (sum of lengths in a row <= L).
// The default row rule is First-Fit in input order (reading R14 of Alg. 1's "greedily
// put").  First-Fit here runs in O(n log B): a max-segment-tree over the
// residual capacity of all candidate rows finds the leftmost row with room; rows not yet
// opened have residual L, so "leftmost row with room" also opens new rows in order.
#include <nvtx3/nvToolsExt.h>   // header-only NVTX3 host range
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <new>
#include <numeric>

#include "tcb_internal.h"

namespace tcb {

static thread_local std::string g_last_error;

void set_error(const std::string& msg) { g_last_error = msg; }
void clear_error() { g_last_error.clear(); }
tcb_status fail(tcb_status st, const std::string& msg) {
  g_last_error = msg;
  return st;
}

namespace {

// Max segment tree over row residuals; leftmost index with value >= need.
class ResidualTree {
 public:
  ResidualTree(int32_t rows, int32_t init) : n_(1) {
    while (n_ < rows) n_ <<= 1;
    t_.assign(2 * static_cast<size_t>(n_), -1);
    for (int32_t i = 0; i < rows; ++i) t_[n_ + i] = init;
    for (int32_t i = n_ - 1; i >= 1; --i) t_[i] = std::max(t_[2 * i], t_[2 * i + 1]);
  }
  int32_t leftmost_at_least(int32_t need) const {
    if (t_[1] < need) return -1;
    int32_t i = 1;
    while (i < n_) i = (t_[2 * i] >= need) ? 2 * i : 2 * i + 1;
    return i - n_;
  }
  void sub(int32_t row, int32_t v) {
    int32_t i = n_ + row;
    t_[i] -= v;
    for (i >>= 1; i >= 1; i >>= 1) t_[i] = std::max(t_[2 * i], t_[2 * i + 1]);
  }

 private:
  int32_t n_;
  std::vector<int32_t> t_;
};

void compute_info(tcb_plan* p) {
  tcb_plan_info& I = p->info;
  std::memset(&I, 0, sizeof(I));
  I.num_requests = p->n;
  I.num_rows = p->num_rows;
  I.row_len = p->row_len;
  I.num_segments = static_cast<int32_t>(p->seg_req.size());
  I.num_placed = I.num_segments;
  I.total_tokens = p->tok_off.empty() ? 0 : p->tok_off.back();
  const int64_t L = p->row_len;
  I.num_slots = static_cast<int64_t>(p->num_rows) * L;
  I.qtiles = (I.num_slots + 127) / 128;
  std::vector<int32_t> seg_end(p->seg_req.size());
  for (size_t s = 0; s < p->seg_req.size(); ++s) {
    const int64_t l = p->lengths[p->seg_req[s]];
    I.placed_tokens += l;
    I.useful_score_elems += l * l;
    seg_end[s] = p->seg_start[s] + static_cast<int32_t>(l);
  }
  // Per-slot segment index (-1 pad), used for the tile counters below.
  std::vector<int32_t> seg_of(static_cast<size_t>(I.num_slots), -1);
  for (size_t s = 0; s < p->seg_req.size(); ++s)
    for (int32_t k = p->seg_start[s]; k < seg_end[s]; ++k) seg_of[k] = static_cast<int32_t>(s);
  // 128x128 tile counters (§8(c) o9), defined when rows are whole q-tiles.
  if (L % 128 == 0) {
    I.kv_tiles_dense = static_cast<int64_t>(p->num_rows) * (L / 128) * (L / 128);
    for (int64_t t = 0; t < I.qtiles; ++t) {
      int32_t first = -1, last = -1;
      for (int64_t k = t * 128; k < std::min<int64_t>(I.num_slots, (t + 1) * 128); ++k)
        if (seg_of[k] >= 0) { if (first < 0) first = seg_of[k]; last = seg_of[k]; }
      if (first < 0) continue;
      const int64_t lo = p->seg_start[first], hi = seg_end[last];
      I.kv_tiles_visited += (hi - 1) / 128 - lo / 128 + 1;
    }
  } else {
    I.kv_tiles_dense = -1;
    I.kv_tiles_visited = -1;
  }
  // Score elements the tcgen05 attention kernel (attention_tc.cu) evaluates, per head.  An
  // item is a block of kAttnQBlock query slots; its key interval [lo, hi) spans its first to
  // its last request, walked in kAttnKChunk-key chunks from kbase = lo rounded down to 8:
  //   executed: every chunk is a full kAttnQBlock x kAttnKChunk S = QK^T tile on the tensor core;
  //   softmax : inside a chunk, a group of kAttnSmRows query rows x kAttnSmKeys keys goes
  //             through the exponentials iff it intersects the union of those rows' intervals
  //             (dead groups are skipped, P = 0).
  for (int64_t q0 = 0; q0 < I.num_slots; q0 += kAttnQBlock) {
    constexpr int kG = kAttnQBlock / kAttnSmRows;
    int64_t glo[kG], ghi[kG];
    int64_t lo = -1, hi = -1;
    for (int g = 0; g < kG; ++g) {
      glo[g] = -1; ghi[g] = -1;
      for (int64_t k = q0 + g * kAttnSmRows; k < std::min<int64_t>(I.num_slots, q0 + (g + 1) * kAttnSmRows); ++k) {
        if (seg_of[k] < 0) continue;
        const int64_t a = p->seg_start[seg_of[k]], b = seg_end[seg_of[k]];
        if (glo[g] < 0 || a < glo[g]) glo[g] = a;
        if (b > ghi[g]) ghi[g] = b;
      }
      if (glo[g] >= 0) {
        if (lo < 0 || glo[g] < lo) lo = glo[g];
        if (ghi[g] > hi) hi = ghi[g];
      }
    }
    if (lo < 0) continue;
    const int64_t kbase = lo & ~static_cast<int64_t>(7);
    const int64_t nch = (hi - kbase + kAttnKChunk - 1) / kAttnKChunk;
    I.executed_score_elems += nch * kAttnQBlock * kAttnKChunk;
    for (int g = 0; g < kG; ++g) {
      if (glo[g] < 0) continue;
      for (int64_t gk = kbase; gk < kbase + nch * kAttnKChunk; gk += kAttnSmKeys)
        if (gk < ghi[g] && gk + kAttnSmKeys > glo[g]) I.softmax_score_elems += kAttnSmRows * kAttnSmKeys;
    }
  }
}

tcb_status validate_pack(const char* fn, const int32_t* lengths, int32_t n, int32_t row_len,
                         int32_t max_rows, tcb_plan** out) {
  const std::string f(fn);
  if (!out) return fail(TCB_ERR_INVALID_ARGUMENT, f + ": out is NULL");
  *out = nullptr;
  if (n < 0) return fail(TCB_ERR_INVALID_ARGUMENT, f + ": n < 0");
  if (n > 0 && !lengths) return fail(TCB_ERR_INVALID_ARGUMENT, f + ": lengths is NULL");
  if (row_len <= 0 || row_len % 8 != 0)
    return fail(TCB_ERR_INVALID_ARGUMENT, f + ": row_len must be a positive multiple of 8");
  if (max_rows < 0) return fail(TCB_ERR_INVALID_ARGUMENT, f + ": max_rows < 0");
  for (int32_t i = 0; i < n; ++i) {
    if (lengths[i] <= 0)
      return fail(TCB_ERR_INVALID_ARGUMENT, f + ": lengths[" + std::to_string(i) + "] <= 0");
    if (lengths[i] > row_len)
      return fail(TCB_ERR_REQUEST_TOO_LONG, f + ": request " + std::to_string(i) + " has " +
                                                std::to_string(lengths[i]) + " tokens > row_len " +
                                                std::to_string(row_len));
  }
  return TCB_OK;
}

}  // namespace

void init_plan(tcb_plan* p, const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
               int32_t policy) {
  p->n = n;
  p->row_len = row_len;
  p->max_rows = max_rows;
  p->policy = policy;
  p->lengths.assign(lengths, lengths + n);
  p->req_row.assign(n, -1);
  p->req_col.assign(n, -1);
  p->tok_off.resize(static_cast<size_t>(n) + 1);
  p->tok_off[0] = 0;
  for (int32_t i = 0; i < n; ++i) p->tok_off[i + 1] = p->tok_off[i] + lengths[i];
}

// Segments in (row, column) order from req_row / req_col; then the counters.
void finish_plan(tcb_plan* p) {
  std::vector<std::vector<int32_t>> members(p->num_rows);
  for (int32_t r = 0; r < p->n; ++r)
    if (p->req_row[r] >= 0) members[p->req_row[r]].push_back(r);
  for (int32_t k = 0; k < p->num_rows; ++k) {
    std::sort(members[k].begin(), members[k].end(),
              [&](int32_t a, int32_t b) { return p->req_col[a] < p->req_col[b]; });
    for (int32_t r : members[k]) {
      p->seg_req.push_back(r);
      p->seg_start.push_back(k * p->row_len + p->req_col[r]);
    }
  }
  compute_info(p);
  p->info.slot_len = p->slot_len;
}

}  // namespace tcb

using tcb::fail;

extern "C" {

const char* tcb_last_error(void) { return tcb::g_last_error.c_str(); }
const char* tcb_version(void) { return "tcb-b200 0.1 (sm_100a)"; }

tcb_status tcb_pack(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                    int32_t policy, tcb_plan** out) {
  nvtxRangePushA("tcb_pack");
  struct Pop { ~Pop() { nvtxRangePop(); } } pop_;
  tcb::clear_error();
  tcb_status st = tcb::validate_pack("tcb_pack", lengths, n, row_len, max_rows, out);
  if (st != TCB_OK) return st;
  if (policy < TCB_PACK_FIRST_FIT || policy > TCB_PACK_LENGTH_SORTED)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_pack: unknown policy");
  tcb_plan* p = new (std::nothrow) tcb_plan();
  if (!p) return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_pack: out of host memory");
  try {
    tcb::init_plan(p, lengths, n, row_len, max_rows, policy);
    std::vector<int32_t> order(n);
    std::iota(order.begin(), order.end(), 0);
    if (policy == TCB_PACK_FIRST_FIT_DECREASING)
      std::stable_sort(order.begin(), order.end(),
                       [&](int32_t a, int32_t b) { return lengths[a] > lengths[b]; });
    else if (policy == TCB_PACK_LENGTH_SORTED)
      std::stable_sort(order.begin(), order.end(),
                       [&](int32_t a, int32_t b) { return lengths[a] < lengths[b]; });

    const int32_t cap = max_rows > 0 ? max_rows : std::max<int32_t>(n, 1);
    std::vector<int32_t> used;
    auto place = [&](int32_t r, int32_t row) {
      if (row >= static_cast<int32_t>(used.size())) used.resize(row + 1, 0);
      p->req_row[r] = row;
      p->req_col[r] = used[row];
      used[row] += lengths[r];
    };
    if (policy == TCB_PACK_FIRST_FIT || policy == TCB_PACK_FIRST_FIT_DECREASING) {
      tcb::ResidualTree tree(cap, row_len);
      for (int32_t r : order) {
        const int32_t row = tree.leftmost_at_least(lengths[r]);
        if (row < 0) continue;  // R16: unplaced
        tree.sub(row, lengths[r]);
        place(r, row);
      }
    } else if (policy == TCB_PACK_NEXT_FIT) {
      int32_t cur = -1;
      for (int32_t r : order) {
        if (cur >= 0 && used[cur] + lengths[r] <= row_len) {
          place(r, cur);
        } else if (cur + 1 < cap) {
          ++cur;
          place(r, cur);
        }
      }
    } else {  // NAIVE, LENGTH_SORTED: one request per row
      int32_t next = 0;
      for (int32_t r : order) {
        if (next >= cap) break;
        place(r, next++);
      }
    }
    p->num_rows = static_cast<int32_t>(used.size());
    tcb::finish_plan(p);
  } catch (const std::bad_alloc&) {
    delete p;
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_pack: out of host memory");
  } catch (...) {
    delete p;
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_pack: internal error");
  }
  *out = p;
  return TCB_OK;
}

tcb_status tcb_pack_slotted(const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
                            int32_t slot_len, tcb_plan** out) {
  tcb::clear_error();
  tcb_status st = tcb::validate_pack("tcb_pack_slotted", lengths, n, row_len, max_rows, out);
  if (st != TCB_OK) return st;
  if (slot_len < 0 || slot_len > row_len)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_pack_slotted: slot_len must be in [0, row_len]");
  tcb_plan* p = new (std::nothrow) tcb_plan();
  if (!p) return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_pack_slotted: out of host memory");
  try {
    tcb::init_plan(p, lengths, n, row_len, max_rows, TCB_PACK_FIRST_FIT);
    int32_t z = slot_len;
    if (z == 0) z = n > 0 ? *std::max_element(lengths, lengths + n) : row_len;  // Alg. 2 l.4
    p->slot_len = z;
    const int32_t per_row = row_len / z;
    const int32_t cap = max_rows > 0 ? max_rows : std::max<int32_t>(n, 1);
    // First-Fit over slots (row-major): the leftmost slot with residual >= l; slots of rows
    // not yet opened have residual z, so "no open slot fits" opens the next row.
    tcb::ResidualTree tree(static_cast<int32_t>(std::min<int64_t>(
                               static_cast<int64_t>(cap) * per_row, INT32_MAX)), z);
    std::vector<int32_t> fill;
    int32_t rows = 0;
    for (int32_t r = 0; r < n; ++r) {
      if (lengths[r] > z) continue;  // longer than a slot: deferred (R26)
      const int32_t slot = tree.leftmost_at_least(lengths[r]);
      if (slot < 0) continue;        // row cap reached: deferred
      if (slot >= static_cast<int32_t>(fill.size())) fill.resize(slot + 1, 0);
      tree.sub(slot, lengths[r]);
      p->req_row[r] = slot / per_row;
      p->req_col[r] = (slot % per_row) * z + fill[slot];
      fill[slot] += lengths[r];
      rows = std::max(rows, slot / per_row + 1);
    }
    p->num_rows = rows;
    tcb::finish_plan(p);
  } catch (const std::bad_alloc&) {
    delete p;
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_pack_slotted: out of host memory");
  } catch (...) {
    delete p;
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_pack_slotted: internal error");
  }
  *out = p;
  return TCB_OK;
}

void tcb_plan_destroy(tcb_plan* plan) { delete plan; }

tcb_status tcb_plan_info_get(const tcb_plan* plan, tcb_plan_info* info) {
  tcb::clear_error();
  if (!plan || !info) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_plan_info_get: NULL argument");
  *info = plan->info;
  return TCB_OK;
}

tcb_status tcb_plan_copy(const tcb_plan* p, int32_t* req_row, int32_t* req_col,
                         int32_t* seg_req, int32_t* seg_start, int32_t* cu_seqlens,
                         int32_t* segment_ids, int32_t* positions, int32_t* qtile_kv) {
  tcb::clear_error();
  if (!p) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_plan_copy: plan is NULL");
  const size_t S = p->seg_req.size();
  const int64_t M = p->info.num_slots;
  if (req_row) std::copy(p->req_row.begin(), p->req_row.end(), req_row);
  if (req_col) std::copy(p->req_col.begin(), p->req_col.end(), req_col);
  if (seg_req) std::copy(p->seg_req.begin(), p->seg_req.end(), seg_req);
  if (seg_start) std::copy(p->seg_start.begin(), p->seg_start.end(), seg_start);
  if (cu_seqlens) {
    cu_seqlens[0] = 0;
    for (size_t s = 0; s < S; ++s) cu_seqlens[s + 1] = cu_seqlens[s] + p->lengths[p->seg_req[s]];
  }
  if (segment_ids || positions || qtile_kv) {
    std::vector<int32_t> seg(static_cast<size_t>(M), -1);
    for (size_t s = 0; s < S; ++s) {
      const int32_t l = p->lengths[p->seg_req[s]];
      for (int32_t j = 0; j < l; ++j) {
        seg[p->seg_start[s] + j] = static_cast<int32_t>(s);
        if (positions) positions[p->seg_start[s] + j] = j;
      }
    }
    if (segment_ids) std::copy(seg.begin(), seg.end(), segment_ids);
    if (positions)
      for (int64_t k = 0; k < M; ++k)
        if (seg[k] < 0) positions[k] = -1;
    if (qtile_kv) {
      for (int64_t t = 0; t < p->info.qtiles; ++t) {
        int32_t first = -1, last = -1;
        for (int64_t k = t * 128; k < std::min<int64_t>(M, (t + 1) * 128); ++k)
          if (seg[k] >= 0) { if (first < 0) first = seg[k]; last = seg[k]; }
        qtile_kv[2 * t] = first < 0 ? -1 : p->seg_start[first];
        qtile_kv[2 * t + 1] = last < 0 ? -1 : p->seg_start[last] + p->lengths[p->seg_req[last]];
      }
    }
  }
  return TCB_OK;
}

int64_t tcb_plan_segtab_words(const tcb_plan* p) {
  if (!p) return -1;
  return 4 * (1 + static_cast<int64_t>(p->seg_req.size())) + (p->num_rows + 1 + 3) / 4 * 4 +
         (p->info.qtiles + 3) / 4 * 4;
}

tcb_status tcb_plan_write_segtab(const tcb_plan* p, int32_t* dst, int64_t capacity_words) {
  tcb::clear_error();
  if (!p || !dst) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_plan_write_segtab: NULL argument");
  const int64_t need = tcb_plan_segtab_words(p);
  if (capacity_words < need)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_plan_write_segtab: capacity " +
                                              std::to_string(capacity_words) + " < " +
                                              std::to_string(need) + " words");
  if (p->info.num_slots > INT32_MAX || p->info.total_tokens > INT32_MAX)
    return fail(TCB_ERR_UNSUPPORTED, "tcb_plan_write_segtab: more than 2^31 slots or tokens");
  dst[0] = static_cast<int32_t>(p->seg_req.size());
  dst[1] = static_cast<int32_t>(p->info.num_slots);
  dst[2] = p->row_len;
  dst[3] = static_cast<int32_t>(p->info.total_tokens);
  for (size_t s = 0; s < p->seg_req.size(); ++s) {
    const int32_t r = p->seg_req[s];
    int32_t* rec = dst + 4 * (1 + s);
    rec[0] = p->seg_start[s];
    rec[1] = p->lengths[r];
    rec[2] = static_cast<int32_t>(p->tok_off[r]);
    rec[3] = r;
  }
  // row index: segments are in (row, column) order, so row_first is a running count
  int32_t* row_first = dst + 4 * (1 + p->seg_req.size());
  const int32_t S = static_cast<int32_t>(p->seg_req.size());
  int32_t s = 0;
  for (int32_t k = 0; k <= p->num_rows; ++k) {
    while (s < S && p->seg_start[s] < static_cast<int64_t>(k) * p->row_len) ++s;
    row_first[k] = s;
  }
  // attention work order: the 128-slot query blocks by decreasing number of 128-key chunks
  // of their key interval (the attention kernel's item cost; longest first, ties by index),
  // so a dynamically scheduled grid ends on short items
  int32_t* qorder = row_first + (p->num_rows + 1 + 3) / 4 * 4;
  const int64_t QT = p->info.qtiles, M = p->info.num_slots;
  std::vector<int32_t> nch(static_cast<size_t>(QT), 0);
  {
    int64_t s0 = 0;
    for (int64_t t = 0; t < QT; ++t) {
      const int64_t q0 = t * 128, q1 = std::min<int64_t>(M, q0 + 128);
      while (s0 < S && static_cast<int64_t>(p->seg_start[s0]) + p->lengths[p->seg_req[s0]] <= q0) ++s0;
      int64_t lo = -1, hi = -1;
      for (int64_t k = s0; k < S && p->seg_start[k] < q1; ++k) {
        const int64_t a = p->seg_start[k], b = a + p->lengths[p->seg_req[k]];
        if (b <= q0) continue;
        if (lo < 0) lo = a;
        hi = b;
      }
      if (lo >= 0) {
        const int64_t kb = lo & ~static_cast<int64_t>(7);
        nch[t] = static_cast<int32_t>((hi - kb + 127) / 128);
      }
    }
  }
  std::vector<int32_t> ord(static_cast<size_t>(QT));
  for (int64_t t = 0; t < QT; ++t) ord[t] = static_cast<int32_t>(t);
  std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) { return nch[a] > nch[b]; });
  for (int64_t t = 0; t < (QT + 3) / 4 * 4; ++t) qorder[t] = t < QT ? ord[t] : 0;
  const int64_t padded = (p->num_rows + 1 + 3) / 4 * 4;
  for (int64_t k = p->num_rows + 1; k < padded; ++k) row_first[k] = S;
  return TCB_OK;
}

}  // extern "C"
