// sched.cpp -- online request scheduler of libtcb (include/tcb.h §4; §8(f) row f2).
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
// Per slot the waiting set is indexed once (O(m log m)); each DAS row then costs O(L + taken)
// instead of re-sorting N_t per row:
//   * utility order = length ascending (ties arrival, id), i.e. length buckets 1..L, each in
//     (arrival, id) order;
//   * N_D is "length <= l_D" for the largest l_D with 1.0/l_D >= q * mean -- evaluated with
//     the same double expression as the definition, so the set is identical;
//   * "deadline order, place if it fits" places next the earliest-deadline request among
//     those whose length fits the residual (a request skipped once never fits later, as the
//     residual only shrinks), so each placement scans the heads of the buckets <= residual;
//   * the rest in utility order likewise places the shortest fitting request next.
// Removal is lazy (a placed flag; bucket heads skip placed entries).
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <new>
#include <numeric>
#include <vector>

#include "tcb_internal.h"

struct tcb_scheduler {
  int32_t policy = 0, B = 0, L = 0;
  double eta = 0.5, q = 0.5;
  struct Req {
    int64_t id;
    int32_t len;
    double arrival, deadline;
  };
  std::vector<Req> queue;  // submitted, not yet scheduled or expired
  tcb_sched_stats stats{};
};

namespace tcb {
namespace {

struct Ctx {
  const int32_t* len;
  const double* arr;
  const double* dl;
  const int64_t* id;
};

bool by_arrival(const Ctx& c, int32_t a, int32_t b) {
  if (c.arr[a] != c.arr[b]) return c.arr[a] < c.arr[b];
  return c.id[a] < c.id[b];
}
bool by_deadline(const Ctx& c, int32_t a, int32_t b) {
  if (c.dl[a] != c.dl[b]) return c.dl[a] < c.dl[b];
  return by_arrival(c, a, b);
}
bool by_utility(const Ctx& c, int32_t a, int32_t b) {
  if (c.len[a] != c.len[b]) return c.len[a] < c.len[b];
  return by_arrival(c, a, b);
}

// One batch: row[i], col[i] for each waiting request i (-1 = not chosen).
void schedule_batch(int32_t policy, const Ctx& c, int32_t n, int32_t B, int32_t L, double eta,
                    double q, int32_t* row, int32_t* col) {
  for (int32_t i = 0; i < n; ++i) { row[i] = -1; col[i] = -1; }
  if (n == 0 || B == 0) return;
  if (policy != TCB_SCHED_DAS) {
    std::vector<int32_t> order(n);
    std::iota(order.begin(), order.end(), 0);
    if (policy == TCB_SCHED_FCFS)
      std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return by_arrival(c, a, b); });
    else if (policy == TCB_SCHED_SJF)
      std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return by_utility(c, a, b); });
    else
      std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return by_deadline(c, a, b); });
    // First-Fit over B rows: max-residual segment tree
    int32_t m = 1;
    while (m < B) m <<= 1;
    std::vector<int32_t> t(2 * m, -1);
    for (int32_t k = 0; k < B; ++k) t[m + k] = L;
    for (int32_t i = m - 1; i >= 1; --i) t[i] = std::max(t[2 * i], t[2 * i + 1]);
    for (int32_t r : order) {
      const int32_t l = c.len[r];
      if (t[1] < l) continue;
      int32_t i = 1;
      while (i < m) i = (t[2 * i] >= l) ? 2 * i : 2 * i + 1;
      const int32_t k = i - m;
      row[r] = k;
      col[r] = L - t[i];
      t[i] -= l;
      for (i >>= 1; i >= 1; i >>= 1) t[i] = std::max(t[2 * i], t[2 * i + 1]);
    }
    return;
  }
  // ---- DAS ----
  std::vector<int32_t> arr_order(n);
  std::iota(arr_order.begin(), arr_order.end(), 0);
  std::sort(arr_order.begin(), arr_order.end(), [&](int32_t a, int32_t b) { return by_arrival(c, a, b); });
  // length buckets: utility order (arrival, id) and deadline order
  std::vector<std::vector<int32_t>> ub(L + 1), db(L + 1);
  for (int32_t r : arr_order) ub[c.len[r]].push_back(r);
  for (int32_t l = 1; l <= L; ++l) {
    db[l] = ub[l];
    std::sort(db[l].begin(), db[l].end(), [&](int32_t a, int32_t b) { return by_deadline(c, a, b); });
  }
  std::vector<size_t> uh(L + 1, 0), dh(L + 1, 0);   // lazy heads
  std::vector<char> placed(n, 0);
  size_t ah = 0;
  int64_t left_tokens = 0;
  int32_t left = n;
  for (int32_t i = 0; i < n; ++i) left_tokens += c.len[i];
  auto uhead = [&](int32_t l) -> int32_t {
    while (uh[l] < ub[l].size() && placed[ub[l][uh[l]]]) ++uh[l];
    return uh[l] < ub[l].size() ? ub[l][uh[l]] : -1;
  };
  auto dhead = [&](int32_t l) -> int32_t {
    while (dh[l] < db[l].size() && placed[db[l][dh[l]]]) ++dh[l];
    return dh[l] < db[l].size() ? db[l][dh[l]] : -1;
  };
  std::vector<int32_t> nu;
  for (int32_t k = 0; k < B && left > 0; ++k) {
    int32_t used = 0;
    auto put = [&](int32_t r) {
      row[r] = k;
      col[r] = used;
      used += c.len[r];
      placed[r] = 1;
      left_tokens -= c.len[r];
      --left;
    };
    if (left_tokens <= L) {                       // l.4-5: everything left, arrival order
      for (; ah < arr_order.size(); ++ah)
        if (!placed[arr_order[ah]]) put(arr_order[ah]);
      continue;
    }
    // l.7-8: s = how many of the utility order fit the row
    int32_t s = 0;
    {
      int64_t pre = 0;
      bool stop = false;
      for (int32_t l = 1; l <= L && !stop; ++l) {
        size_t j = uh[l];
        for (; j < ub[l].size(); ++j) {
          if (placed[ub[l][j]]) continue;
          if (pre + l > L) { stop = true; break; }
          pre += l;
          ++s;
        }
      }
    }
    int32_t p = static_cast<int32_t>(std::floor(eta * static_cast<double>(s)));  // l.9
    if (p < 1) p = 1;
    // l.10: N_U = the first p in utility order
    nu.clear();
    for (int32_t l = 1; l <= L && static_cast<int32_t>(nu.size()) < p; ++l)
      for (int32_t r = uhead(l); r >= 0 && static_cast<int32_t>(nu.size()) < p; r = uhead(l)) {
        nu.push_back(r);
        placed[r] = 1;                             // claim (re-marked by put below)
      }
    double vsum = 0.0;
    for (int32_t r : nu) {
      placed[r] = 0;
      put(r);
      vsum += 1.0 / static_cast<double>(c.len[r]);
    }
    // l.11: N_D = lengths l with 1.0/l >= q * mean (a prefix of lengths)
    const double thr = q * (vsum / static_cast<double>(p));
    int32_t lD = 0;
    for (int32_t l = 1; l <= L; ++l)
      if (1.0 / static_cast<double>(l) >= thr) lD = l;
    // l.12: deadline order, placed when it fits
    while (used < L) {
      int32_t best = -1;
      const int32_t lim = std::min(lD, L - used);
      for (int32_t l = 1; l <= lim; ++l) {
        const int32_t r = dhead(l);
        if (r >= 0 && (best < 0 || by_deadline(c, r, best))) best = r;
      }
      if (best < 0) break;
      put(best);
    }
    // l.13-14: the rest (lengths > lD) in utility order, placed when it fits
    for (int32_t l = lD + 1; l <= L - used; ++l)
      for (int32_t r = uhead(l); r >= 0 && l <= L - used; r = uhead(l)) put(r);
  }
}

}  // namespace
}  // namespace tcb

using tcb::fail;

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
  if (!(eta > 0.0 && eta <= 1.0) || !(q > 0.0 && q <= 1.0))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_batch: eta and q must be in (0, 1]");
  for (int32_t i = 0; i < n; ++i) {
    if (lengths[i] <= 0) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_batch: length <= 0");
    if (lengths[i] > L)
      return fail(TCB_ERR_REQUEST_TOO_LONG, "tcb_sched_batch: request " + std::to_string(i) +
                                                " is longer than L");
  }
  try {
    tcb::schedule_batch(policy, tcb::Ctx{lengths, arrival, deadline, ids}, n, B, L, eta, q, row,
                        col);
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
  if (!(eta > 0.0 && eta <= 1.0) || !(q > 0.0 && q <= 1.0))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_create: eta and q must be in (0, 1]");
  tcb_scheduler* s = new (std::nothrow) tcb_scheduler();
  if (!s) return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_sched_create: out of host memory");
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
    for (int32_t i = 0; i < n; ++i)
      s->queue.push_back({ids[i], lengths[i], arrival[i], deadline[i]});
  } catch (const std::bad_alloc&) {
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_sched_submit: out of host memory");
  }
  s->stats.submitted += n;
  s->stats.waiting = static_cast<int64_t>(s->queue.size());
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
    // expire (deadline passed: the request failed, utility 0), then N_t = arrived ones
    std::vector<tcb_scheduler::Req> keep;
    keep.reserve(s->queue.size());
    for (const auto& r : s->queue) {
      if (r.deadline < now) ++s->stats.expired;
      else keep.push_back(r);
    }
    s->queue.swap(keep);
    std::vector<int32_t> wait;
    for (int32_t i = 0; i < static_cast<int32_t>(s->queue.size()); ++i)
      if (s->queue[i].arrival <= now) wait.push_back(i);
    const int32_t m = static_cast<int32_t>(wait.size());
    std::vector<int32_t> len(m), row(m), col(m);
    std::vector<double> arr(m), dl(m);
    std::vector<int64_t> id(m);
    for (int32_t j = 0; j < m; ++j) {
      const auto& r = s->queue[wait[j]];
      len[j] = r.len; arr[j] = r.arrival; dl[j] = r.deadline; id[j] = r.id;
    }
    tcb::schedule_batch(s->policy, tcb::Ctx{len.data(), arr.data(), dl.data(), id.data()}, m,
                        s->B, s->L, s->eta, s->q, row.data(), col.data());
    std::vector<int32_t> chosen;
    for (int32_t j = 0; j < m; ++j)
      if (row[j] >= 0) chosen.push_back(j);
    std::sort(chosen.begin(), chosen.end(), [&](int32_t a, int32_t b) {
      return row[a] != row[b] ? row[a] < row[b] : col[a] < col[b];
    });
    const int32_t nc = static_cast<int32_t>(chosen.size());
    if (nc > capacity) {
      // nothing is consumed: the caller retries with a larger buffer
      s->stats.waiting = static_cast<int64_t>(s->queue.size());
      *n_out = nc;
      return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_sched_next_batch: capacity < batch size (" +
                                                std::to_string(nc) + ")");
    }
    tcb_plan* p = nullptr;
    if (plan_out) {
      p = new tcb_plan();
      std::vector<int32_t> clen(nc);
      for (int32_t t = 0; t < nc; ++t) clen[t] = len[chosen[t]];
      tcb::init_plan(p, clen.data(), nc, s->L, s->B, TCB_PACK_FIRST_FIT);
      for (int32_t t = 0; t < nc; ++t) {
        p->req_row[t] = row[chosen[t]];
        p->req_col[t] = col[chosen[t]];
      }
      p->num_rows = s->B;                        // fixed batch shape
      tcb::finish_plan(p);
    }
    std::vector<char> take(s->queue.size(), 0);
    for (int32_t t = 0; t < nc; ++t) {
      const int32_t j = chosen[t];
      ids_out[t] = id[j];
      lengths_out[t] = len[j];
      take[wait[j]] = 1;
      s->stats.utility += 1.0 / static_cast<double>(len[j]);
    }
    keep.clear();
    for (size_t i = 0; i < s->queue.size(); ++i)
      if (!take[i]) keep.push_back(s->queue[i]);
    s->queue.swap(keep);
    s->stats.scheduled += nc;
    s->stats.batches += 1;
    s->stats.waiting = static_cast<int64_t>(s->queue.size());
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
