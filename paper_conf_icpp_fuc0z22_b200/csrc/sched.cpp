// sched.cpp -- online request scheduler of libtcb (include/tcb.h §5; §8(f) row f2).
//
// §5: each request n has arrival a_n, deadline d_n and length l_n; one batch of
// B rows x L words runs per time slot; utility v_n = 1/l_n counts for requests scheduled in
// [a_n, d_n] (Eq. (9)-(13)).  Per time slot the scheduler takes the waiting set N_t
// (arrived, not scheduled, deadline not passed: P:1004-1009) and fills B rows:
//   DAS (Alg. 1): per row, if everything left fits it all goes in (l.4-5);
//     else N_U = the first p = max(1, floor(eta s)) requests in utility order (s = how many
//     of that order fit the row, l.7-10), N_D = the others with v >= q * mean v(N_U) placed
//     in deadline order if they fit (l.11-12), then the rest in utility order if they fit
//     (l.13-14).  Readings R27.
//   FCFS / SJF / DEF (§6.2.4): priority order, First-Fit into the B rows.
//
// The waiting set is kept indexed across time slots, so a batch costs O(B (L + placed log L))
// instead of re-sorting N_t (the paper reports the scheduler at ~2 % of a batch, P:1805-1811;
// on B200 a batch is well under a millisecond):
//   * per length l (utility order = length ascending, ties arrival then id): a bucket in
//     (arrival, id) order with a head pointer, and a min-heap in (deadline, arrival, id)
//     order; removal is lazy (an alive flag), heads/tops skip dead entries;
//   * two min-trees over the lengths 1..L hold each bucket's head (arrival key) and each
//     heap's top (deadline key), so "the earliest request of length <= r" is O(log L);
//   * not-yet-arrived requests wait in an arrival min-heap, arrived ones in a deadline
//     min-heap for expiry.
// Each placement rule is the sequential rule restated: in a priority order with "place if it
// fits", a request skipped once never fits later (residuals only shrink), so the next request
// placed is the first one in that order among those that fit now -- a min-tree query.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <functional>
#include <new>
#include <numeric>
#include <vector>

#include "tcb_internal.h"

namespace tcb {
namespace {

struct Req {
  int64_t id;
  int32_t len;
  double arrival, deadline;
};

// Keys are stored by value next to the request handle so that heap / tree comparisons do
// not chase pointers into the request slab.
struct AKey {                      // utility order inside a length bucket, FCFS order
  double a;
  int64_t id;
  int32_t r;                       // handle, -1 = empty
  bool operator<(const AKey& o) const { return a != o.a ? a < o.a : id < o.id; }
};
struct DKey {                      // deadline order (N_D, DEF)
  double d, a;
  int64_t id;
  int32_t r;
  bool operator<(const DKey& o) const {
    if (d != o.d) return d < o.d;
    return a != o.a ? a < o.a : id < o.id;
  }
};

template <class K>
struct MinTree {                   // min over leaves 1..L of a key (r < 0 = empty leaf)
  int32_t leaves = 1;
  std::vector<K> t;
  void init(int32_t L) {
    leaves = 1;
    while (leaves < L + 1) leaves <<= 1;
    K e{};
    e.r = -1;
    t.assign(2 * leaves, e);
  }
  static const K& pick(const K& x, const K& y) {
    if (x.r < 0) return y;
    if (y.r < 0) return x;
    return y < x ? y : x;
  }
  void set(int32_t l, const K& k) {
    int32_t i = leaves + l;
    t[i] = k;
    for (i >>= 1; i >= 1; i >>= 1) t[i] = pick(t[2 * i], t[2 * i + 1]);
  }
  int32_t min_upto(int32_t lim) const {        // handle of the min over [1, lim], or -1
    if (lim < 1) return -1;
    K best{};
    best.r = -1;
    int32_t lo = leaves + 1, hi = leaves + lim + 1;
    while (lo < hi) {
      if (lo & 1) best = pick(best, t[lo++]);
      if (hi & 1) best = pick(best, t[--hi]);
      lo >>= 1;
      hi >>= 1;
    }
    return best.r;
  }
};

struct Index {
  int32_t L = 0;
  std::vector<Req> reqs;            // slab (handles are indices)
  std::vector<char> alive;          // arrived, not scheduled, not expired
  std::vector<std::vector<AKey>> bucket;     // [L+1] arrival order
  std::vector<size_t> head;
  std::vector<char> bucket_sorted;
  std::vector<std::vector<DKey>> dheap;      // [L+1] deadline min-heaps
  MinTree<AKey> tarr;
  MinTree<DKey> tdl;
  int64_t tokens = 0;
  int32_t count = 0;

  AKey akey(int32_t r) const { return {reqs[r].arrival, reqs[r].id, r}; }
  DKey dkey(int32_t r) const { return {reqs[r].deadline, reqs[r].arrival, reqs[r].id, r}; }
  bool arr_less(int32_t a, int32_t b) const { return akey(a) < akey(b); }
  bool dl_less(int32_t a, int32_t b) const { return dkey(a) < dkey(b); }

  void init(int32_t row_len) {
    L = row_len;
    bucket.assign(L + 1, {});
    head.assign(L + 1, 0);
    bucket_sorted.assign(L + 1, 1);
    dheap.assign(L + 1, {});
    tarr.init(L);
    tdl.init(L);
  }

  // first alive entry of bucket l (sorting it first if arrivals came out of order)
  int32_t bucket_head(int32_t l) {
    auto& b = bucket[l];
    if (!bucket_sorted[l]) {
      std::vector<AKey> keep;
      for (size_t j = head[l]; j < b.size(); ++j)
        if (alive[b[j].r]) keep.push_back(b[j]);
      std::sort(keep.begin(), keep.end());
      b.swap(keep);
      head[l] = 0;
      bucket_sorted[l] = 1;
    }
    while (head[l] < b.size() && !alive[b[head[l]].r]) ++head[l];
    if (head[l] > 4096 && head[l] * 2 > b.size()) {      // drop the consumed prefix
      b.erase(b.begin(), b.begin() + static_cast<std::ptrdiff_t>(head[l]));
      head[l] = 0;
    }
    return head[l] < b.size() ? b[head[l]].r : -1;
  }
  int32_t heap_top(int32_t l) {
    auto& h = dheap[l];
    auto greater = [](const DKey& x, const DKey& y) { return y < x; };
    while (!h.empty() && !alive[h.front().r]) {
      std::pop_heap(h.begin(), h.end(), greater);
      h.pop_back();
    }
    return h.empty() ? -1 : h.front().r;
  }
  // The tree leaves always hold the bucket head / heap top of each length, so activation
  // and removal only touch a leaf when they change it.
  void activate(int32_t r) {
    const int32_t l = reqs[r].len;
    auto& b = bucket[l];
    const AKey k = akey(r);
    if (b.size() > head[l] && k < b.back()) bucket_sorted[l] = 0;
    b.push_back(k);
    auto greater = [](const DKey& x, const DKey& y) { return y < x; };
    const DKey dk = dkey(r);
    dheap[l].push_back(dk);
    std::push_heap(dheap[l].begin(), dheap[l].end(), greater);
    alive[r] = 1;
    tokens += l;
    ++count;
    const AKey& la = tarr.t[tarr.leaves + l];
    if (la.r < 0 || k < la) tarr.set(l, k);
    const DKey& ld = tdl.t[tdl.leaves + l];
    if (ld.r < 0 || dk < ld) tdl.set(l, dk);
  }
  void remove(int32_t r) {
    const int32_t l = reqs[r].len;
    alive[r] = 0;
    tokens -= l;
    --count;
    if (tarr.t[tarr.leaves + l].r == r) {
      const int32_t a = bucket_head(l);
      if (a >= 0) tarr.set(l, bucket[l][head[l]]);
      else { AKey e{}; e.r = -1; tarr.set(l, e); }
    }
    if (tdl.t[tdl.leaves + l].r == r) {
      const int32_t d = heap_top(l);
      if (d >= 0) tdl.set(l, dheap[l].front());
      else { DKey e{}; e.r = -1; tdl.set(l, e); }
    }
  }
  // alive requests of bucket l from its head, in order (f returns false to stop)
  template <class F>
  void walk(int32_t l, F&& f) {
    if (bucket_head(l) < 0) return;
    const auto& b = bucket[l];
    for (size_t j = head[l]; j < b.size(); ++j)
      if (alive[b[j].r] && !f(b[j].r)) return;
  }
};

// First-Fit over B rows: max-residual segment tree.
struct RowTree {
  int32_t m = 1;
  std::vector<int32_t> t;
  RowTree(int32_t B, int32_t L) {
    while (m < B) m <<= 1;
    t.assign(2 * m, -1);
    for (int32_t k = 0; k < B; ++k) t[m + k] = L;
    for (int32_t i = m - 1; i >= 1; --i) t[i] = std::max(t[2 * i], t[2 * i + 1]);
  }
  int32_t maxres() const { return t[1]; }
  int32_t first_fit(int32_t l) const {  // leftmost row with residual >= l, or -1
    if (t[1] < l) return -1;
    int32_t i = 1;
    while (i < m) i = (t[2 * i] >= l) ? 2 * i : 2 * i + 1;
    return i - m;
  }
  int32_t take(int32_t k, int32_t l) {  // returns the column
    int32_t i = m + k;
    const int32_t c = t[i];
    t[i] -= l;
    for (i >>= 1; i >= 1; i >>= 1) t[i] = std::max(t[2 * i], t[2 * i + 1]);
    return c;
  }
};

// One batch over the alive requests of `x`; appends (request, row, col) in placement order.
void schedule(Index& x, int32_t policy, int32_t B, double eta, double q,
              std::vector<int32_t>& out_req, std::vector<int32_t>& out_row,
              std::vector<int32_t>& out_col) {
  const int32_t L = x.L;
  if (B <= 0 || x.count == 0) return;
  if (policy != TCB_SCHED_DAS) {
    RowTree rows(B, L);
    auto place = [&](int32_t r) {
      const int32_t k = rows.first_fit(x.reqs[r].len);
      const int32_t res = rows.take(k, x.reqs[r].len);
      out_req.push_back(r);
      out_row.push_back(k);
      out_col.push_back(L - res);
      x.remove(r);
    };
    if (policy == TCB_SCHED_SJF) {
      for (int32_t l = 1; l <= L && l <= rows.maxres(); ++l)
        for (int32_t r = x.bucket_head(l); r >= 0 && l <= rows.maxres(); r = x.bucket_head(l))
          place(r);
    } else {
      const bool by_dl = policy == TCB_SCHED_DEF;
      for (;;) {
        const int32_t lim = std::min(rows.maxres(), L);
        const int32_t r = by_dl ? x.tdl.min_upto(lim) : x.tarr.min_upto(lim);
        if (r < 0) break;
        place(r);
      }
    }
    return;
  }
  std::vector<int32_t> tmp;
  for (int32_t k = 0; k < B && x.count > 0; ++k) {
    int32_t used = 0;
    auto put = [&](int32_t r) {
      out_req.push_back(r);
      out_row.push_back(k);
      out_col.push_back(used);
      used += x.reqs[r].len;
      x.remove(r);
    };
    if (x.tokens <= L) {                              // l.4-5: all of it, arrival order
      tmp.clear();
      for (int32_t l = 1; l <= L; ++l) x.walk(l, [&](int32_t r) { tmp.push_back(r); return true; });
      std::sort(tmp.begin(), tmp.end(), [&](int32_t a, int32_t b) { return x.arr_less(a, b); });
      for (int32_t r : tmp) put(r);
      continue;
    }
    // l.7-8: s = how many of the utility order fit the row
    int32_t s = 0;
    int64_t pre = 0;
    bool stop = false;
    for (int32_t l = 1; l <= L && !stop; ++l)
      x.walk(l, [&](int32_t) {
        if (pre + l > L) { stop = true; return false; }
        pre += l;
        ++s;
        return true;
      });
    int32_t p = static_cast<int32_t>(std::floor(eta * static_cast<double>(s)));  // l.9
    if (p < 1) p = 1;
    // l.10: N_U = the first p in utility order
    tmp.clear();
    for (int32_t l = 1; l <= L && static_cast<int32_t>(tmp.size()) < p; ++l)
      x.walk(l, [&](int32_t r) {
        tmp.push_back(r);
        return static_cast<int32_t>(tmp.size()) < p;
      });
    double vsum = 0.0;
    for (int32_t r : tmp) {
      put(r);
      vsum += 1.0 / static_cast<double>(x.reqs[r].len);
    }
    // l.11: N_D = lengths l with 1.0/l >= q * mean (a prefix of the lengths)
    const double thr = q * (vsum / static_cast<double>(p));
    int32_t lD = 0;
    for (int32_t l = 1; l <= L; ++l)
      if (1.0 / static_cast<double>(l) >= thr) lD = l;
    // l.12: deadline order, placed when it fits
    for (;;) {
      const int32_t r = x.tdl.min_upto(std::min(lD, L - used));
      if (r < 0) break;
      put(r);
    }
    // l.13-14: the rest (lengths > lD) in utility order, placed when it fits
    for (int32_t l = lD + 1; l <= L - used; ++l)
      for (int32_t r = x.bucket_head(l); r >= 0 && l <= L - used; r = x.bucket_head(l)) put(r);
  }
}

}  // namespace
}  // namespace tcb

struct tcb_scheduler {
  int32_t policy = 0, B = 0, L = 0;
  double eta = 0.5, q = 0.5;
  tcb::Index x;
  std::vector<tcb::AKey> pending;                    // min-heap: not arrived yet
  std::vector<std::pair<double, int32_t>> expiry;    // min-heap by deadline: activated
  tcb_sched_stats stats{};
};

using tcb::fail;

namespace {

bool params_ok(double eta, double q) { return eta > 0.0 && eta <= 1.0 && q > 0.0 && q <= 1.0; }

// Handles are never reused while stale bucket / heap entries may name them; instead the
// index is rebuilt from the live requests once most of the slab is dead (amortised O(1)).
void compact(tcb_scheduler* s) {
  tcb::Index& x = s->x;
  tcb::Index y;
  y.init(x.L);
  std::vector<int32_t> act;
  for (int32_t r = 0; r < static_cast<int32_t>(x.reqs.size()); ++r)
    if (x.alive[r]) act.push_back(r);
  std::sort(act.begin(), act.end(), [&](int32_t a, int32_t b) { return x.arr_less(a, b); });
  std::vector<std::pair<double, int32_t>> new_exp;
  std::vector<tcb::AKey> new_pend;
  for (int32_t r : act) {
    const int32_t h = static_cast<int32_t>(y.reqs.size());
    y.reqs.push_back(x.reqs[r]);
    y.alive.push_back(0);
    y.activate(h);
    new_exp.push_back({y.reqs[h].deadline, h});
  }
  for (const tcb::AKey& k : s->pending) {
    const int32_t h = static_cast<int32_t>(y.reqs.size());
    y.reqs.push_back(x.reqs[k.r]);
    y.alive.push_back(0);
    new_pend.push_back({k.a, k.id, h});
  }
  s->x = std::move(y);
  std::make_heap(new_exp.begin(), new_exp.end(), std::greater<>());
  std::make_heap(new_pend.begin(), new_pend.end(),
                 [](const tcb::AKey& a, const tcb::AKey& b) { return b < a; });
  s->expiry.swap(new_exp);
  s->pending.swap(new_pend);
}

}  // namespace

extern "C" {

tcb_status tcb_sched_batch(int32_t policy, const int32_t* lengths, const double* arrival,
                           const double* deadline, const int64_t* ids, int32_t n, int32_t B,
                           int32_t L, double eta, double q, int32_t* row, int32_t* col) {
  tcb::clear_error();
  if (policy < TCB_SCHED_DAS || policy > TCB_SCHED_DEF)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_batch: unknown policy");
  if (n < 0 || B < 0 || L <= 0)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_batch: n < 0, B < 0 or L <= 0");
  if (n > 0 && (!lengths || !arrival || !deadline || !ids || !row || !col))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_batch: NULL array");
  if (!params_ok(eta, q))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_batch: eta and q must be in (0, 1]");
  for (int32_t i = 0; i < n; ++i) {
    if (lengths[i] <= 0) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_batch: length <= 0");
    if (lengths[i] > L)
      return fail(TCB_ERR_REQUEST_TOO_LONG, "tcb_sched_batch: request " + std::to_string(i) +
                                                " is longer than L");
  }
  try {
    tcb::Index x;
    x.init(L);
    x.reqs.resize(n);
    x.alive.assign(n, 0);
    std::vector<int32_t> order(n);
    std::iota(order.begin(), order.end(), 0);
    for (int32_t i = 0; i < n; ++i) x.reqs[i] = {ids[i], lengths[i], arrival[i], deadline[i]};
    std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return x.arr_less(a, b); });
    for (int32_t i : order) x.activate(i);
    std::vector<int32_t> rr, kk, cc;
    tcb::schedule(x, policy, B, eta, q, rr, kk, cc);
    for (int32_t i = 0; i < n; ++i) { row[i] = -1; col[i] = -1; }
    for (size_t j = 0; j < rr.size(); ++j) { row[rr[j]] = kk[j]; col[rr[j]] = cc[j]; }
  } catch (const std::bad_alloc&) {
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_sched_batch: out of host memory");
  }
  return TCB_OK;
}

tcb_status tcb_sched_create(int32_t policy, int32_t batch_rows, int32_t row_len, double eta,
                            double q, tcb_scheduler** out) {
  tcb::clear_error();
  if (!out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_create: out is NULL");
  *out = nullptr;
  if (policy < TCB_SCHED_DAS || policy > TCB_SCHED_DEF)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_create: unknown policy");
  if (batch_rows <= 0 || row_len <= 0 || row_len % 8 != 0)
    return fail(TCB_ERR_INVALID_ARGUMENT,
                "tcb_sched_create: batch_rows must be > 0 and row_len a positive multiple of 8");
  if (!params_ok(eta, q))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_create: eta and q must be in (0, 1]");
  tcb_scheduler* s = new (std::nothrow) tcb_scheduler();
  if (!s) return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_sched_create: out of host memory");
  try {
    s->x.init(row_len);
  } catch (const std::bad_alloc&) {
    delete s;
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_sched_create: out of host memory");
  }
  s->policy = policy;
  s->B = batch_rows;
  s->L = row_len;
  s->eta = eta;
  s->q = q;
  *out = s;
  return TCB_OK;
}

void tcb_sched_destroy(tcb_scheduler* s) { delete s; }

tcb_status tcb_sched_submit(tcb_scheduler* s, int32_t n, const int64_t* ids,
                            const int32_t* lengths, const double* arrival,
                            const double* deadline) {
  tcb::clear_error();
  if (!s) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_submit: scheduler is NULL");
  if (n < 0) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_submit: n < 0");
  if (n > 0 && (!ids || !lengths || !arrival || !deadline))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_submit: NULL array");
  for (int32_t i = 0; i < n; ++i) {
    if (lengths[i] <= 0) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_submit: length <= 0");
    if (lengths[i] > s->L)
      return fail(TCB_ERR_REQUEST_TOO_LONG, "tcb_sched_submit: request " + std::to_string(i) +
                                                " is longer than row_len (constraint (11))");
    if (!(deadline[i] >= arrival[i]))
      return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_submit: deadline < arrival");
  }
  try {
    tcb::Index& x = s->x;
    auto later = [](const tcb::AKey& a, const tcb::AKey& b) { return b < a; };
    for (int32_t i = 0; i < n; ++i) {
      const int32_t h = static_cast<int32_t>(x.reqs.size());
      x.reqs.push_back({ids[i], lengths[i], arrival[i], deadline[i]});
      x.alive.push_back(0);
      s->pending.push_back({arrival[i], ids[i], h});
      std::push_heap(s->pending.begin(), s->pending.end(), later);
    }
  } catch (const std::bad_alloc&) {
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_sched_submit: out of host memory");
  }
  s->stats.submitted += n;
  s->stats.waiting += n;
  return TCB_OK;
}

tcb_status tcb_sched_next_batch(tcb_scheduler* s, double now, int64_t* ids_out,
                                int32_t* lengths_out, int32_t capacity, int32_t* n_out,
                                tcb_plan** plan_out) {
  tcb::clear_error();
  if (!s || !n_out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_next_batch: NULL argument");
  if (capacity < 0 || (capacity > 0 && (!ids_out || !lengths_out)))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_next_batch: bad output arrays");
  if (plan_out) *plan_out = nullptr;
  *n_out = 0;
  try {
    if (s->x.reqs.size() > 65536 &&
        s->x.reqs.size() > 4 * (static_cast<size_t>(s->x.count) + s->pending.size()))
      compact(s);
    tcb::Index& x = s->x;
    // arrivals up to now join N_t; then requests whose deadline passed expire (utility 0)
    auto later = [](const tcb::AKey& a, const tcb::AKey& b) { return b < a; };
    while (!s->pending.empty() && s->pending.front().a <= now) {
      const int32_t r = s->pending.front().r;
      std::pop_heap(s->pending.begin(), s->pending.end(), later);
      s->pending.pop_back();
      x.activate(r);
      s->expiry.push_back({x.reqs[r].deadline, r});
      std::push_heap(s->expiry.begin(), s->expiry.end(), std::greater<>());
    }
    while (!s->expiry.empty() && s->expiry.front().first < now) {
      const int32_t r = s->expiry.front().second;
      std::pop_heap(s->expiry.begin(), s->expiry.end(), std::greater<>());
      s->expiry.pop_back();
      if (x.alive[r]) {
        x.remove(r);
        ++s->stats.expired;
        --s->stats.waiting;
      }
    }
    // the batch cannot exceed B * L requests (every length >= 1)
    if (capacity < std::min<int64_t>(static_cast<int64_t>(s->B) * s->L, x.count) &&
        capacity < x.count) {
      // check the exact size without consuming: schedule on a copy
      tcb::Index y = x;
      std::vector<int32_t> rr, kk, cc;
      tcb::schedule(y, s->policy, s->B, s->eta, s->q, rr, kk, cc);
      if (static_cast<int64_t>(rr.size()) > capacity) {
        *n_out = static_cast<int32_t>(rr.size());
        return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_next_batch: capacity < batch size (" +
                                                  std::to_string(rr.size()) + ")");
      }
    }
    std::vector<int32_t> rr, kk, cc;
    tcb::schedule(x, s->policy, s->B, s->eta, s->q, rr, kk, cc);
    const int32_t nc = static_cast<int32_t>(rr.size());
    std::vector<int32_t> ord(nc);
    std::iota(ord.begin(), ord.end(), 0);
    std::sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) {
      return kk[a] != kk[b] ? kk[a] < kk[b] : cc[a] < cc[b];
    });
    tcb_plan* p = nullptr;
    if (plan_out) {
      p = new tcb_plan();
      std::vector<int32_t> clen(nc);
      for (int32_t t = 0; t < nc; ++t) clen[t] = x.reqs[rr[ord[t]]].len;
      tcb::init_plan(p, clen.data(), nc, s->L, s->B, TCB_PACK_FIRST_FIT);
      for (int32_t t = 0; t < nc; ++t) {
        p->req_row[t] = kk[ord[t]];
        p->req_col[t] = cc[ord[t]];
      }
      p->num_rows = s->B;                        // fixed batch shape
      tcb::finish_plan(p);
    }
    for (int32_t t = 0; t < nc; ++t) {
      const int32_t r = rr[ord[t]];
      ids_out[t] = x.reqs[r].id;
      lengths_out[t] = x.reqs[r].len;
      s->stats.utility += 1.0 / static_cast<double>(x.reqs[r].len);
    }
    s->stats.scheduled += nc;
    s->stats.waiting -= nc;
    s->stats.batches += 1;
    *n_out = nc;
    if (plan_out) *plan_out = p;
  } catch (const std::bad_alloc&) {
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_sched_next_batch: out of host memory");
  }
  return TCB_OK;
}

tcb_status tcb_sched_stats_get(const tcb_scheduler* s, tcb_sched_stats* out) {
  tcb::clear_error();
  if (!s || !out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_stats_get: NULL argument");
  *out = s->stats;
  return TCB_OK;
}

}  // extern "C"
