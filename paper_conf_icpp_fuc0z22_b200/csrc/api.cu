// api.cu -- the device half of the libtcb C ABI (include/tcb.h, include/tcb_ops.h):
// weights handle, workspace layout, tcb_embed / tcb_encoder_forward / tcb_unpack, the
// op-level entry points and the launch/profiling instrumentation.  Host code only; every
// arithmetic step runs in the kernels of elementwise.cu, linear_tc.cu, linear_f32.cu and
// attention.cu.  There is no CPU fallback: without an sm_100 device every device call
// returns TCB_ERR_NO_DEVICE.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>   // header-only NVTX3: host ranges for nsys / ncu timelines

#include "kernels.h"
#include "tcb_internal.h"

using tcb::fail;

namespace {

std::atomic<int64_t> g_launches{0};

// ---- profiling: CUDA event pairs around each launch ----------------------------------------
struct ProfRec {
  int cls;
  cudaEvent_t a, b;
};
std::mutex g_prof_mu;
bool g_prof_on = false;
std::vector<ProfRec> g_prof;
std::vector<cudaEvent_t> g_event_pool;

cudaEvent_t pool_event() {
  if (!g_event_pool.empty()) {
    cudaEvent_t e = g_event_pool.back();
    g_event_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

// Under stream capture the pair is recorded as external event-record nodes, so a graph
// captured with profiling on times every launch on each replay (tcb_profile_snapshot).
struct ProfScope {
  bool on;
  int cls;
  cudaStream_t s;
  unsigned flags = cudaEventRecordDefault;
  cudaEvent_t a = nullptr, b = nullptr;
  ProfScope(int c, cudaStream_t st) : on(false), cls(c), s(st) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    if (!g_prof_on) return;
    on = true;
    a = pool_event();
    b = pool_event();
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &cs) == cudaSuccess && cs == cudaStreamCaptureStatusActive)
      flags = cudaEventRecordExternal;
    cudaGetLastError();
    cudaEventRecordWithFlags(a, s, flags);
  }
  ~ProfScope() {
    if (!on) return;
    cudaEventRecordWithFlags(b, s, flags);
    std::lock_guard<std::mutex> g(g_prof_mu);
    g_prof.push_back({cls, a, b});
  }
};

tcb_status cuda_fail(cudaError_t e, const char* what) {
  return fail(TCB_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define TCB_LAUNCH(cls, stream, expr)                                 \
  do {                                                                \
    ProfScope _ps((cls), (stream));                                   \
    cudaError_t _e = (expr);                                          \
    g_launches.fetch_add(1, std::memory_order_relaxed);               \
    if (_e != cudaSuccess) return cuda_fail(_e, #expr);               \
  } while (0)

tcb_status check_device() {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
    cudaGetLastError();
    return fail(TCB_ERR_NO_DEVICE, "no CUDA device visible (libtcb has no CPU fallback)");
  }
  int dev = 0, major = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  if (major != 10)
    return fail(TCB_ERR_NO_DEVICE, "libtcb is built for sm_100a (B200); device has major " +
                                       std::to_string(major));
  return TCB_OK;
}

constexpr size_t align256(size_t x) { return (x + 255) & ~static_cast<size_t>(255); }

struct WsLayout {
  size_t seg, qkv, att, z, x1, h, lnst, lncnt, lncnt_per_launch, attn_cnt, gemm_cnt, ready,
      ready_per_launch, total;
};
WsLayout ws_layout(const tcb_model_config& c, int64_t M) {
  const size_t es = c.dtype == 0 ? 4 : 2;
  WsLayout L{};
  size_t off = 0;
  L.seg = off; off += align256(sizeof(int32_t) * static_cast<size_t>(M));
  L.qkv = off; off += align256(es * static_cast<size_t>(M) * 3 * c.d_model);
  L.att = off; off += align256(es * static_cast<size_t>(M) * c.d_model);
  L.z = off;   off += align256(es * static_cast<size_t>(M) * c.d_model);
  L.x1 = off;  off += align256(es * static_cast<size_t>(M) * c.d_model);
  L.h = off;   off += align256(es * static_cast<size_t>(M) * c.d_ff);
  // row-statistics scratch of the L2-exchange LayerNorm GEMM (bf16, d = 512 / 768 / 1024): partials
  // per 256-row tile, and one zeroed counter region per fused launch (2 per layer)
  L.lnst = off;
  L.lncnt = off;
  L.lncnt_per_launch = 0;
  if (c.dtype == 1 && (c.d_model == 512 || c.d_model == 768 || c.d_model == 1024)) {
    off += align256(tcb::k::linear_ln_scratch_stats_bytes(M, c.d_model));
    L.lncnt = off;
    L.lncnt_per_launch = align256(tcb::k::linear_ln_scratch_cnt_bytes(M));
    off += L.lncnt_per_launch * 2 * static_cast<size_t>(c.num_layers);
  }
  // bf16 attention: one dynamic item counter per layer.  [lncnt, total) is the zeroed region
  // (one memset per forward).
  L.attn_cnt = off;
  if (c.dtype == 1) off += align256(sizeof(int32_t) * static_cast<size_t>(c.num_layers));
  // bf16: dynamic tile counters of the QKV and FFN1 GEMMs (2 per layer) and the 128-row block
  // readiness flags of the W_O and FFN2 outputs (2 per layer), for the tail overlap of a
  // GEMM with the LayerNorm GEMM before it
  L.gemm_cnt = off;
  L.ready = off;
  L.ready_per_launch = 0;
  if (c.dtype == 1) {
    off += align256(sizeof(int32_t) * 2 * static_cast<size_t>(c.num_layers));
    L.ready = off;
    L.ready_per_launch = align256(sizeof(int32_t) * 2 * static_cast<size_t>((M + 255) / 256));
    off += L.ready_per_launch * 2 * static_cast<size_t>(c.num_layers);
  }
  L.total = off;
  return L;
}

tcb_status validate_cfg(const tcb_model_config* c) {
  if (!c) return fail(TCB_ERR_INVALID_ARGUMENT, "config is NULL");
  if (c->num_layers < 0 || c->d_model <= 0 || c->num_heads <= 0 || c->d_ff <= 0 ||
      c->vocab <= 0 || c->max_pos <= 0 || (c->dtype != 0 && c->dtype != 1) ||
      (c->act != 0 && c->act != 1) || c->pe < 0 || c->pe > 2)
    return fail(TCB_ERR_INVALID_ARGUMENT, "invalid model config field");
  if (c->d_model % c->num_heads != 0)
    return fail(TCB_ERR_UNSUPPORTED, "d_model % num_heads != 0");
  const int dh = c->d_model / c->num_heads;
  if (c->dtype == 1) {
    if (dh != 64 || c->d_model % 64 != 0 || c->d_ff % 64 != 0 || c->d_model > 2048)
      return fail(TCB_ERR_UNSUPPORTED,
                  "bf16 path needs d_head == 64, d_model % 64 == 0, d_ff % 64 == 0, d_model <= 2048");
  } else {
    if (dh > 64 || dh % 2 != 0 || c->d_model % 4 != 0 || c->d_model > 1024)
      return fail(TCB_ERR_UNSUPPORTED,
                  "fp32 path needs d_head <= 64 and even, d_model % 4 == 0, d_model <= 1024");
  }
  return TCB_OK;
}

}  // namespace

struct tcb_weights {
  tcb_model_config cfg{};
  std::vector<const void*> t;
  float* pe_table = nullptr;
  struct LayerMaps {
    CUtensorMap qkv, o, w1, w2;  // W operands (built once)
    CUtensorMap w2h;             // W_2 with 64-row boxes (half-width tail units of the LN GEMM)
  };
  std::vector<LayerMaps> maps;
  // activation TMA descriptors, rebuilt when the (rows, workspace) pointers change:
  // A-role (GEMM input) and C-role (GEMM output / residual input) views of each buffer
  std::mutex mu;
  std::mutex graph_mu;                    // fwd_graphs
  const void* c_rows = nullptr;
  const void* c_ws = nullptr;
  int64_t c_M = -1;
  // tcb_encoder_forward's instantiated CUDA graphs, keyed on the launch geometry and buffers
  // (the kernels read everything plan-specific from the device segment table)
  struct FwdGraph {
    int64_t M;
    int32_t rows, row_len;
    const void *segtab, *ids, *drows, *ws, *dout;
    cudaGraphExec_t exec;
    uint64_t launches, last_use;
  };
  std::vector<FwdGraph> fwd_graphs;
  uint64_t fwd_tick = 0;
  cudaStream_t cap_stream = nullptr;      // private stream the graphs are captured on
  CUtensorMap aX{}, aAtt{}, aX1{}, aH{};
  CUtensorMap cQkv{}, cZ{}, cH{}, cX{}, cX1{};

  const void* tok_emb() const { return t[0]; }
  const void* pos_emb() const { return t[1]; }
  const float* type_emb() const { return static_cast<const float*>(t[2]); }
  const float* emb_ln_g() const { return static_cast<const float*>(t[3]); }
  const float* emb_ln_b() const { return static_cast<const float*>(t[4]); }
  const void* L(int layer, int i) const { return t[5 + 12 * layer + i]; }
  const float* Lf(int layer, int i) const { return static_cast<const float*>(L(layer, i)); }
};

namespace {

enum { W_QKV = 0, B_QKV, W_O, B_O, LN1_G, LN1_B, W_1, B_1, W_2, B_2, LN2_G, LN2_B };

// bf16 attention: the tcgen05 kernel (attention_tc.cu).
cudaError_t attention_bf16(int64_t M, int d, int heads, const void* qkv, const int32_t* seg,
                           const int4* segtab, void* out, int* item_counter, int row_len,
                           cudaStream_t s) {
  return tcb::k::launch_attention_bf16_tc(M, d, heads, qkv, seg, segtab, out, item_counter,
                                          row_len, s);
}

tcb_status embed_impl(const tcb_weights* w, const tcb_plan* plan, const int32_t* d_segtab,
                      const int32_t* d_ids, void* d_rows, int32_t* d_seg, int32_t* d_pos,
                      cudaStream_t s) {
  const tcb_model_config& c = w->cfg;
  tcb::k::EmbedArgs a{};
  a.segtab = reinterpret_cast<const int4*>(d_segtab);
  a.ids = d_ids;
  a.tok_emb = w->tok_emb();
  a.pos_emb = c.pe == 2 ? w->pos_emb() : nullptr;
  a.pe_table = c.pe == 2 ? nullptr : w->pe_table;
  a.type_emb = c.use_type_emb ? w->type_emb() : nullptr;
  a.ln_g = c.emb_ln ? w->emb_ln_g() : nullptr;
  a.ln_b = c.emb_ln ? w->emb_ln_b() : nullptr;
  a.emb_scale = c.emb_scale;
  a.ln_eps = c.emb_ln_eps;
  a.d = c.d_model;
  a.max_pos = c.max_pos;
  a.num_rows = plan->num_rows;
  a.row_len = plan->row_len;
  a.num_slots = plan->info.num_slots;
  a.X = d_rows;
  a.seg_ids = d_seg;
  a.positions = d_pos;
  TCB_LAUNCH(TCB_K_EMBED, s, tcb::k::launch_embed(c.dtype, a, s));
  return TCB_OK;
}

tcb_status validate_plan_for(const tcb_weights* w, const tcb_plan* p) {
  if (!w || !p) return fail(TCB_ERR_INVALID_ARGUMENT, "weights or plan is NULL");
  if (p->info.num_slots > INT32_MAX)
    return fail(TCB_ERR_UNSUPPORTED, "more than 2^31 slots in one forward");
  if (p->num_rows > 0 && p->row_len > w->cfg.max_pos)
    return fail(TCB_ERR_UNSUPPORTED, "row_len " + std::to_string(p->row_len) +
                                         " exceeds max_pos " + std::to_string(w->cfg.max_pos));
  return TCB_OK;
}

}  // namespace

extern "C" {

int64_t tcb_launch_count(void) { return g_launches.load(); }

tcb_status tcb_profile_enable(int32_t on) {
  tcb::clear_error();
  std::lock_guard<std::mutex> g(g_prof_mu);
  g_prof_on = on != 0;
  return TCB_OK;
}

tcb_status tcb_profile_collect(double* ms, int64_t* launches) {
  tcb::clear_error();
  std::lock_guard<std::mutex> g(g_prof_mu);
  if (ms) for (int i = 0; i < TCB_KCLASS_COUNT; ++i) ms[i] = 0.0;
  if (launches) for (int i = 0; i < TCB_KCLASS_COUNT; ++i) launches[i] = 0;
  tcb_status st = TCB_OK;
  for (const ProfRec& r : g_prof) {
    float t = 0.f;
    cudaError_t e = cudaEventSynchronize(r.b);
    if (e == cudaSuccess) e = cudaEventElapsedTime(&t, r.a, r.b);
    if (e != cudaSuccess) st = cuda_fail(e, "tcb_profile_collect");
    if (ms) ms[r.cls] += t;
    if (launches) launches[r.cls] += 1;
    g_event_pool.push_back(r.a);
    g_event_pool.push_back(r.b);
  }
  g_prof.clear();
  return st;
}

tcb_status tcb_profile_snapshot(double* ms, int64_t* launches) {
  tcb::clear_error();
  std::lock_guard<std::mutex> g(g_prof_mu);
  if (ms) for (int i = 0; i < TCB_KCLASS_COUNT; ++i) ms[i] = 0.0;
  if (launches) for (int i = 0; i < TCB_KCLASS_COUNT; ++i) launches[i] = 0;
  tcb_status st = TCB_OK;
  for (const ProfRec& r : g_prof) {
    float t = 0.f;
    cudaError_t e = cudaEventSynchronize(r.b);
    if (e == cudaSuccess) e = cudaEventElapsedTime(&t, r.a, r.b);
    if (e != cudaSuccess) st = cuda_fail(e, "tcb_profile_snapshot");
    if (ms) ms[r.cls] += t;
    if (launches) launches[r.cls] += 1;
  }
  return st;
}

int32_t tcb_weights_count(const tcb_model_config* cfg) {
  return cfg ? 5 + 12 * cfg->num_layers : -1;
}

tcb_status tcb_workspace_size(const tcb_model_config* cfg, int64_t num_slots, size_t* bytes) {
  tcb::clear_error();
  if (tcb_status st = validate_cfg(cfg)) return st;
  if (!bytes || num_slots < 0) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_workspace_size");
  *bytes = ws_layout(*cfg, num_slots).total;
  return TCB_OK;
}

tcb_status tcb_weights_create(const tcb_model_config* cfg, const void* const* tensors,
                              int32_t num_tensors, tcb_weights** out) {
  tcb::clear_error();
  if (!out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_weights_create: out is NULL");
  *out = nullptr;
  if (tcb_status st = validate_cfg(cfg)) return st;
  if (!tensors || num_tensors != tcb_weights_count(cfg))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_weights_create: expected " +
                                              std::to_string(tcb_weights_count(cfg)) + " tensors");
  for (int i = 0; i < num_tensors; ++i) {
    if (!tensors[i] || (reinterpret_cast<uintptr_t>(tensors[i]) & 15))
      return fail(TCB_ERR_INVALID_ARGUMENT,
                  "tcb_weights_create: tensor " + std::to_string(i) + " is NULL or not 16-byte aligned");
  }
  if (tcb_status st = check_device()) return st;
  tcb_weights* w = new (std::nothrow) tcb_weights();
  if (!w) return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_weights_create");
  w->cfg = *cfg;
  w->t.assign(tensors, tensors + num_tensors);
  const tcb_model_config& c = *cfg;
  if (c.pe != 2) {
    cudaError_t e = cudaMalloc(&w->pe_table, sizeof(float) * static_cast<size_t>(c.max_pos) * c.d_model);
    if (e != cudaSuccess) { delete w; return fail(TCB_ERR_OUT_OF_MEMORY, "PE table allocation"); }
    e = tcb::k::launch_pe_table(w->pe_table, c.max_pos, c.d_model, c.pe, nullptr);
    g_launches.fetch_add(1);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { cudaFree(w->pe_table); delete w; return cuda_fail(e, "PE table"); }
  }
  if (c.dtype == 1) {
    w->maps.resize(c.num_layers);
    for (int l = 0; l < c.num_layers; ++l) {
      const int d = c.d_model, f = c.d_ff;
      bool ok = tcb::k::make_gemm_w_map(&w->maps[l].qkv, w->L(l, W_QKV), 3 * d, d) &&
                tcb::k::make_gemm_w_map(&w->maps[l].o, w->L(l, W_O), d, d) &&
                tcb::k::make_gemm_w_map(&w->maps[l].w1, w->L(l, W_1), f, d) &&
                tcb::k::make_gemm_w_map(&w->maps[l].w2, w->L(l, W_2), d, f) &&
                tcb::k::make_gemm_w_half_map(&w->maps[l].w2h, w->L(l, W_2), d, f);
      if (!ok) {
        if (w->pe_table) cudaFree(w->pe_table);
        delete w;
        return fail(TCB_ERR_CUDA, "cuTensorMapEncodeTiled failed for a weight matrix");
      }
    }
  }
  *out = w;
  return TCB_OK;
}

void tcb_weights_destroy(tcb_weights* w) {
  if (!w) return;
  for (auto& g : w->fwd_graphs) cudaGraphExecDestroy(g.exec);
  if (w->cap_stream) cudaStreamDestroy(w->cap_stream);
  if (w->pe_table) cudaFree(w->pe_table);
  delete w;
}

tcb_status tcb_embed(const tcb_weights* w, const tcb_plan* plan, const int32_t* d_segtab,
                     const int32_t* d_token_ids, void* d_rows, int32_t* d_segment_ids,
                     int32_t* d_positions, tcb_stream_t stream) {
  tcb::clear_error();
  if (tcb_status st = validate_plan_for(w, plan)) return st;
  const int64_t M = plan->info.num_slots;
  if (M == 0) return TCB_OK;
  if (!d_segtab || !d_rows || (plan->info.total_tokens > 0 && !d_token_ids))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_embed: NULL device pointer");
  return embed_impl(w, plan, d_segtab, d_token_ids, d_rows, d_segment_ids, d_positions,
                    reinterpret_cast<cudaStream_t>(stream));
}

namespace {
tcb_status forward_impl(const tcb_weights* wc, const tcb_plan* plan, const int32_t* d_segtab,
                        const int32_t* d_token_ids, void* d_rows, void* d_out, void* d_ws,
                        size_t ws_bytes, tcb_stream_t stream);
}  // namespace

// The public forward replays a CUDA graph of its own launch sequence when it can: on a
// non-default stream that is not being captured by the caller, with profiling off, and
// TCB_NO_FWD_GRAPH unset.  The graph is captured on the first call with a given geometry and
// set of buffers (LRU of 4 per weights handle) and replayed for any later plan of the same
// B x L (every plan-specific value is read from the device segment table); otherwise the
// kernels are launched directly.  Either way the work is the same.
namespace {
// d_out == NULL: tcb_encoder_forward; else tcb_encoder_forward_unpacked
tcb_status forward_entry(const tcb_weights* wc, const tcb_plan* plan, const int32_t* d_segtab,
                         const int32_t* d_token_ids, void* d_rows, void* d_out, void* d_ws,
                         size_t ws_bytes, tcb_stream_t stream) {
  static const bool no_graph =
      std::getenv("TCB_NO_FWD_GRAPH") != nullptr || std::getenv("TCB_DEBUG_SYNC") != nullptr;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  bool use_graph = !no_graph && wc && plan && plan->info.num_slots > 0 && d_segtab && d_rows &&
                   d_ws;
  if (use_graph) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    use_graph = !g_prof_on;
  }
  if (use_graph && s != nullptr) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone) {
      cudaGetLastError();
      use_graph = false;
    }
  }
  if (!use_graph)
    return forward_impl(wc, plan, d_segtab, d_token_ids, d_rows, d_out, d_ws, ws_bytes, stream);
  if (tcb_status st = validate_plan_for(wc, plan)) return st;
  // the same argument checks as forward_impl BEFORE a cache hit can replay (a graph captured
  // for an all-pad plan with NULL ids must not serve a plan that has tokens)
  if (plan->info.total_tokens > 0 && !d_token_ids)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_encoder_forward: NULL device pointer");
  tcb_weights* w = const_cast<tcb_weights*>(wc);
  const int64_t M = plan->info.num_slots;
  std::lock_guard<std::mutex> gl(w->graph_mu);
  for (auto& e : w->fwd_graphs) {
    if (e.M == M && e.rows == plan->num_rows && e.row_len == plan->row_len &&
        e.segtab == d_segtab && e.ids == d_token_ids && e.drows == d_rows && e.ws == d_ws &&
        e.dout == d_out) {
      if (ws_bytes < ws_layout(w->cfg, M).total)
        break;                                   // let forward_impl report it
      e.last_use = ++w->fwd_tick;
      cudaError_t err = cudaGraphLaunch(e.exec, s);
      if (err != cudaSuccess) return cuda_fail(err, "tcb_encoder_forward: graph launch");
      g_launches.fetch_add(e.launches, std::memory_order_relaxed);
      return TCB_OK;
    }
  }
  // miss: capture this call's launches on the private stream, instantiate, run the graph on s
  if (!w->cap_stream && cudaStreamCreateWithFlags(&w->cap_stream, cudaStreamNonBlocking) != cudaSuccess) {
    cudaGetLastError();
    w->cap_stream = nullptr;
    return forward_impl(wc, plan, d_segtab, d_token_ids, d_rows, d_out, d_ws, ws_bytes, stream);
  }
  cudaStream_t cap = w->cap_stream;
  if (cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
    cudaGetLastError();
    return forward_impl(wc, plan, d_segtab, d_token_ids, d_rows, d_out, d_ws, ws_bytes, stream);
  }
  const uint64_t c0 = g_launches.load();
  const tcb_status st = forward_impl(wc, plan, d_segtab, d_token_ids, d_rows, d_out, d_ws,
                                     ws_bytes, reinterpret_cast<tcb_stream_t>(cap));
  cudaGraph_t graph = nullptr;
  const cudaError_t ce = cudaStreamEndCapture(cap, &graph);
  if (st != TCB_OK || ce != cudaSuccess || !graph) {
    if (graph) cudaGraphDestroy(graph);
    cudaGetLastError();
    if (st != TCB_OK) return st;
    return forward_impl(wc, plan, d_segtab, d_token_ids, d_rows, d_out, d_ws, ws_bytes, stream);
  }
  cudaGraphExec_t exec = nullptr;
  const cudaError_t ie = cudaGraphInstantiate(&exec, graph, 0);
  cudaGraphDestroy(graph);
  if (ie != cudaSuccess) {
    cudaGetLastError();
    return forward_impl(wc, plan, d_segtab, d_token_ids, d_rows, d_out, d_ws, ws_bytes, stream);
  }
  if (w->fwd_graphs.size() >= 4) {               // evict the least recently used
    auto lru = std::min_element(w->fwd_graphs.begin(), w->fwd_graphs.end(),
                                [](const auto& a, const auto& b) { return a.last_use < b.last_use; });
    cudaGraphExecDestroy(lru->exec);
    w->fwd_graphs.erase(lru);
  }
  w->fwd_graphs.push_back({M, plan->num_rows, plan->row_len, d_segtab, d_token_ids, d_rows, d_ws,
                           d_out, exec, g_launches.load() - c0, ++w->fwd_tick});
  const cudaError_t le = cudaGraphLaunch(exec, s);
  if (le != cudaSuccess) return cuda_fail(le, "tcb_encoder_forward: graph launch");
  return TCB_OK;
}
}  // namespace

tcb_status tcb_encoder_forward(const tcb_weights* wc, const tcb_plan* plan,
                               const int32_t* d_segtab, const int32_t* d_token_ids,
                               void* d_rows, void* d_ws, size_t ws_bytes, tcb_stream_t stream) {
  tcb::clear_error();
  return forward_entry(wc, plan, d_segtab, d_token_ids, d_rows, nullptr, d_ws, ws_bytes, stream);
}

tcb_status tcb_encoder_forward_unpacked(const tcb_weights* wc, const tcb_plan* plan,
                                        const int32_t* d_segtab, const int32_t* d_token_ids,
                                        void* d_rows, void* d_out, void* d_ws, size_t ws_bytes,
                                        tcb_stream_t stream) {
  tcb::clear_error();
  if (plan && plan->info.total_tokens > 0 && !d_out)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_encoder_forward_unpacked: d_out is NULL");
  if (plan && plan->info.total_tokens == 0)      // nothing to write: the plain forward
    return forward_entry(wc, plan, d_segtab, d_token_ids, d_rows, nullptr, d_ws, ws_bytes, stream);
  return forward_entry(wc, plan, d_segtab, d_token_ids, d_rows, d_out, d_ws, ws_bytes, stream);
}

namespace {
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

tcb_status forward_impl(const tcb_weights* wc, const tcb_plan* plan, const int32_t* d_segtab,
                        const int32_t* d_token_ids, void* d_rows, void* d_out, void* d_ws,
                        size_t ws_bytes, tcb_stream_t stream) {
  NvtxRange nvtx_fwd("tcb_encoder_forward");
  if (tcb_status st = validate_plan_for(wc, plan)) return st;
  tcb_weights* w = const_cast<tcb_weights*>(wc);
  const tcb_model_config& c = w->cfg;
  const int64_t M = plan->info.num_slots;
  if (M == 0) return TCB_OK;
  if (!d_segtab || !d_rows || !d_ws || (plan->info.total_tokens > 0 && !d_token_ids))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_encoder_forward: NULL device pointer");
  const WsLayout L = ws_layout(c, M);
  if (ws_bytes < L.total)
    return fail(TCB_ERR_WORKSPACE_TOO_SMALL, "tcb_encoder_forward: workspace " +
                                                 std::to_string(ws_bytes) + " < " +
                                                 std::to_string(L.total) + " bytes");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  uint8_t* ws = static_cast<uint8_t*>(d_ws);
  int32_t* seg = reinterpret_cast<int32_t*>(ws + L.seg);
  void* qkv = ws + L.qkv;
  void* att = ws + L.att;
  void* z = ws + L.z;
  void* x1 = ws + L.x1;
  void* hbuf = ws + L.h;
  const int d = c.d_model, f = c.d_ff;
  const int act_epi = c.act == 0 ? TCB_EPI_BIAS_GELU : TCB_EPI_BIAS_RELU;
  const int4* segtab = reinterpret_cast<const int4*>(d_segtab);

  if (tcb_status st = embed_impl(w, plan, d_segtab, d_token_ids, d_rows, seg, nullptr, s)) return st;
  bool out_done = false;                         // d_out written by the fused last FFN2

  if (c.dtype == 1) {
    // Activation TMA descriptors: cached per weights handle for the last (rows, workspace, M)
    // and COPIED into this call's locals under the lock, so concurrent forwards with other
    // buffers (direct launches on other streams) never read a descriptor being rewritten.
    CUtensorMap aX, aAtt, aX1, aH, cQkv, cZ, cH, cX, cX1;
    {
      std::lock_guard<std::mutex> g(w->mu);
      if (w->c_rows != d_rows || w->c_ws != d_ws || w->c_M != M) {
        using namespace tcb::k;
        const bool ok = make_gemm_a_map(&w->aX, d_rows, M, d) &&
                        make_gemm_a_map(&w->aAtt, att, M, d) &&
                        make_gemm_a_map(&w->aX1, x1, M, d) &&
                        make_gemm_a_map(&w->aH, hbuf, M, f) &&
                        make_gemm_c_map(&w->cQkv, qkv, M, 3 * d) &&
                        make_gemm_c_map(&w->cZ, z, M, d) && make_gemm_c_map(&w->cH, hbuf, M, f) &&
                        make_gemm_c_map(&w->cX, d_rows, M, d) &&
                        make_gemm_c_map(&w->cX1, x1, M, d);
        if (!ok) {
          w->c_rows = w->c_ws = nullptr;         // a half-written set is never reused
          w->c_M = -1;
          return fail(TCB_ERR_CUDA, "cuTensorMapEncodeTiled failed for an activation");
        }
        w->c_rows = d_rows;
        w->c_ws = d_ws;
        w->c_M = M;
      }
      aX = w->aX; aAtt = w->aAtt; aX1 = w->aX1; aH = w->aH;
      cQkv = w->cQkv; cZ = w->cZ; cH = w->cH; cX = w->cX; cX1 = w->cX1;
    }
    // bias + residual + LayerNorm fused into the W_O / FFN2 GEMMs (d = 512, 768, 1024: a
    // cluster of d / 256 CTA pairs owns complete rows); TCB_NO_LN_FUSION=1 forces the unfused
    // kernels.
    static const bool no_fusion = std::getenv("TCB_NO_LN_FUSION") != nullptr;
    const bool fuse_ln = !no_fusion && tcb::k::linear_ln_supported(d);
    float2* lnst = L.lncnt_per_launch ? reinterpret_cast<float2*>(ws + L.lnst) : nullptr;
    auto lncnt = [&](int launch) -> int* {
      return L.lncnt_per_launch ? reinterpret_cast<int*>(ws + L.lncnt + L.lncnt_per_launch * launch)
                                : nullptr;
    };
    // LayerNorm-exchange counters and attention item counters: one reset per forward
    if (cudaMemsetAsync(ws + L.lncnt, 0, L.total - L.lncnt, s) != cudaSuccess)
      return fail(TCB_ERR_CUDA, "tcb_encoder_forward: counter reset failed");
    int* attn_cnt = reinterpret_cast<int*>(ws + L.attn_cnt);
    // Tail overlap (opt-in, TCB_XOVERLAP=1; TCB_XOVERLAP=dyn: dynamic tiles without the
    // flags): FFN1 starts on the W_O + LN1 rows that are done and the next layer's QKV on the
    // FFN2 + LN2 rows that are done, with dynamic tile order, while the LayerNorm GEMM before
    // it finishes its last tiles.  Correct (parity tests pass with it), but measured no faster:
    // C2 1383 vs 1382 us per step, C3 +1% -- the overlap gains ~25 us per C2
    // step and the dynamic tile hand-off costs about as much -- so it is off by default.
    static const char* xov_env = std::getenv("TCB_XOVERLAP");
    const bool xov_dyn = xov_env != nullptr && L.ready_per_launch > 0;
    const bool xov = xov_dyn && std::string(xov_env) != "dyn";
    int* gemm_cnt = reinterpret_cast<int*>(ws + L.gemm_cnt);
    auto ready = [&](int launch) -> int* {
      return reinterpret_cast<int*>(ws + L.ready + L.ready_per_launch * launch);
    };
    for (int l = 0; l < c.num_layers; ++l) {
      NvtxRange nvtx_layer("tcb encoder layer");
      const auto& mp = w->maps[l];
      const tcb::k::GemmMaps g_qkv{aX, mp.qkv, cQkv, cQkv};
      const tcb::k::GemmMaps g_o{aAtt, mp.o, cZ, cX};
      const tcb::k::GemmMaps g_1{aX1, mp.w1, cH, cH};
      const tcb::k::GemmMaps g_2{aH, mp.w2, cZ, cX1};
      // the previous layer's FFN2 + LN2 signals its rows when fused (xov); layer 0 reads the embedding
      const bool qkv_x = xov && fuse_ln && l > 0;
      TCB_LAUNCH(TCB_K_GEMM_QKV, s, tcb::k::launch_linear_bf16_tc(
                                        g_qkv, M, 3 * d, d, w->Lf(l, B_QKV), TCB_EPI_BIAS, s,
                                        xov_dyn ? gemm_cnt + 2 * l : nullptr,
                                        qkv_x ? ready(2 * (l - 1) + 1) : nullptr, 4 * d));
      TCB_LAUNCH(TCB_K_ATTN, s, attention_bf16(M, d, c.num_heads, qkv, seg, segtab, att, attn_cnt + l,
                                               plan->row_len, s));
      if (fuse_ln) {   // W_O + bias + residual + LN1 in one kernel -> x1
        const tcb::k::GemmMaps g_o_ln{aAtt, mp.o, cX1, cX};
        TCB_LAUNCH(TCB_K_GEMM_O, s, tcb::k::launch_linear_ln_bf16_tc(
                                        g_o_ln, M, d, d, w->Lf(l, B_O), w->Lf(l, LN1_G),
                                        w->Lf(l, LN1_B), c.ln_eps, seg, s, lnst, lncnt(2 * l),
                                        xov ? ready(2 * l) : nullptr));
      } else {
        TCB_LAUNCH(TCB_K_GEMM_O, s, tcb::k::launch_linear_bf16_tc(g_o, M, d, d, w->Lf(l, B_O),
                                                                  TCB_EPI_BIAS_RESIDUAL, s));
        TCB_LAUNCH(TCB_K_LN, s, tcb::k::launch_layernorm(1, M, d, z, w->Lf(l, LN1_G),
                                                         w->Lf(l, LN1_B), c.ln_eps, seg, x1, s));
      }
      const bool ffn1_x = xov && fuse_ln;
      TCB_LAUNCH(TCB_K_GEMM_FFN1, s, tcb::k::launch_linear_bf16_tc(
                                         g_1, M, f, d, w->Lf(l, B_1), act_epi, s,
                                         xov_dyn ? gemm_cnt + 2 * l + 1 : nullptr,
                                         ffn1_x ? ready(2 * l) : nullptr, 4 * d));
      if (fuse_ln) {   // FFN2 + bias + residual + LN2 in one kernel -> X
        tcb::k::GemmMaps g_2_ln{aH, mp.w2, cX, cX1};
        g_2_ln.w_half = mp.w2h;
        g_2_ln.has_w_half = true;
        bool scattered = false;
        if (d_out && l + 1 == c.num_layers && lnst) {
          // the unpack fused into the last FFN2 + LN2: rows go straight to d_out[token]
          ProfScope ps_(TCB_K_GEMM_FFN2, s);
          const cudaError_t e = tcb::k::launch_linear_ln_bf16_tc(
              g_2_ln, M, d, f, w->Lf(l, B_2), w->Lf(l, LN2_G), w->Lf(l, LN2_B), c.ln_eps, seg, s,
              lnst, lncnt(2 * l + 1), nullptr, d_out, segtab);
          if (e == cudaSuccess) {
            g_launches.fetch_add(1, std::memory_order_relaxed);
            scattered = out_done = true;
          } else if (e == cudaErrorNotSupported) {
            cudaGetLastError();                  // packed rows + a separate unpack below
          } else {
            return cuda_fail(e, "tcb_encoder_forward_unpacked: last FFN2");
          }
        }
        if (!scattered)
          TCB_LAUNCH(TCB_K_GEMM_FFN2, s, tcb::k::launch_linear_ln_bf16_tc(
                                             g_2_ln, M, d, f, w->Lf(l, B_2), w->Lf(l, LN2_G),
                                             w->Lf(l, LN2_B), c.ln_eps, seg, s, lnst, lncnt(2 * l + 1),
                                             (xov && l + 1 < c.num_layers) ? ready(2 * l + 1) : nullptr));
      } else {
        TCB_LAUNCH(TCB_K_GEMM_FFN2, s, tcb::k::launch_linear_bf16_tc(g_2, M, d, f, w->Lf(l, B_2),
                                                                     TCB_EPI_BIAS_RESIDUAL, s));
        TCB_LAUNCH(TCB_K_LN, s, tcb::k::launch_layernorm(1, M, d, z, w->Lf(l, LN2_G),
                                                         w->Lf(l, LN2_B), c.ln_eps, seg, d_rows, s));
      }
    }
  } else {
    float* X = static_cast<float*>(d_rows);
    for (int l = 0; l < c.num_layers; ++l) {
      TCB_LAUNCH(TCB_K_GEMM_QKV, s, tcb::k::launch_linear_f32(
                                        M, 3 * d, d, X, static_cast<const float*>(w->L(l, W_QKV)),
                                        w->Lf(l, B_QKV), nullptr, TCB_EPI_BIAS,
                                        static_cast<float*>(qkv), s));
      TCB_LAUNCH(TCB_K_ATTN, s, tcb::k::launch_attention_f32(M, d, c.num_heads,
                                                             static_cast<const float*>(qkv), seg,
                                                             segtab, static_cast<float*>(att), s));
      TCB_LAUNCH(TCB_K_GEMM_O, s, tcb::k::launch_linear_f32(
                                      M, d, d, static_cast<const float*>(att),
                                      static_cast<const float*>(w->L(l, W_O)), w->Lf(l, B_O), X,
                                      TCB_EPI_BIAS_RESIDUAL, static_cast<float*>(z), s));
      TCB_LAUNCH(TCB_K_LN, s, tcb::k::launch_layernorm(0, M, d, z, w->Lf(l, LN1_G),
                                                       w->Lf(l, LN1_B), c.ln_eps, seg, x1, s));
      TCB_LAUNCH(TCB_K_GEMM_FFN1, s, tcb::k::launch_linear_f32(
                                         M, f, d, static_cast<const float*>(x1),
                                         static_cast<const float*>(w->L(l, W_1)), w->Lf(l, B_1),
                                         nullptr, act_epi, static_cast<float*>(hbuf), s));
      TCB_LAUNCH(TCB_K_GEMM_FFN2, s, tcb::k::launch_linear_f32(
                                         M, d, f, static_cast<const float*>(hbuf),
                                         static_cast<const float*>(w->L(l, W_2)), w->Lf(l, B_2),
                                         static_cast<const float*>(x1), TCB_EPI_BIAS_RESIDUAL,
                                         static_cast<float*>(z), s));
      TCB_LAUNCH(TCB_K_LN, s, tcb::k::launch_layernorm(0, M, d, z, w->Lf(l, LN2_G),
                                                       w->Lf(l, LN2_B), c.ln_eps, seg, X, s));
    }
  }
  if (d_out && !out_done)
    TCB_LAUNCH(TCB_K_UNPACK, s, tcb::k::launch_unpack(c.dtype, segtab, plan->num_rows,
                                                      plan->row_len, c.d_model, d_rows, d_out, s));
  if (std::getenv("TCB_DEBUG_SYNC")) {
    cudaError_t e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "tcb_encoder_forward (TCB_DEBUG_SYNC)");
  }
  return TCB_OK;
}
}  // namespace

tcb_status tcb_unpack(const tcb_weights* w, const tcb_plan* plan, const int32_t* d_segtab,
                      const void* d_rows, void* d_out, tcb_stream_t stream) {
  tcb::clear_error();
  nvtxRangePushA("tcb_unpack");
  struct Pop { ~Pop() { nvtxRangePop(); } } pop_;
  if (tcb_status st = validate_plan_for(w, plan)) return st;
  const int64_t M = plan->info.num_slots;
  if (M == 0) return TCB_OK;
  if (!d_segtab || !d_rows || !d_out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_unpack: NULL");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  TCB_LAUNCH(TCB_K_UNPACK, s, tcb::k::launch_unpack(w->cfg.dtype,
                                                    reinterpret_cast<const int4*>(d_segtab),
                                                    plan->num_rows, plan->row_len,
                                                    w->cfg.d_model, d_rows, d_out, s));
  return TCB_OK;
}

// ---- host-buffer sessions --------------------------------------------------------------------
}  // extern "C"

struct tcb_session {
  const tcb_weights* w = nullptr;
  int32_t rows = 0, row_len = 0;
  int64_t max_tokens = 0, seg_words = 0;
  size_t ws_bytes = 0, out_bytes_per_token = 0;
  struct Slot {
    int32_t* d_segtab = nullptr;
    int32_t* d_ids = nullptr;
    void* d_rows = nullptr;
    void* d_ws = nullptr;
    void* d_out = nullptr;
    int32_t* h_seg = nullptr;              // pinned
    cudaEvent_t h2d_done = nullptr, computed = nullptr, d2h_done = nullptr;
    int64_t ticket = -1;                   // last call that used the slot
  } slot[2];
  int64_t calls = 0;
  cudaStream_t up = nullptr;               // uploads: ahead of the compute stream
};

namespace {
void session_free(tcb_session* s) {
  if (!s) return;
  for (auto& sl : s->slot) {
    cudaFree(sl.d_segtab);
    cudaFree(sl.d_ids);
    cudaFree(sl.d_rows);
    cudaFree(sl.d_ws);
    cudaFree(sl.d_out);
    cudaFreeHost(sl.h_seg);
    if (sl.h2d_done) cudaEventDestroy(sl.h2d_done);
    if (sl.computed) cudaEventDestroy(sl.computed);
    if (sl.d2h_done) cudaEventDestroy(sl.d2h_done);
  }
  if (s->up) cudaStreamDestroy(s->up);
  delete s;
}
}  // namespace

extern "C" {

tcb_status tcb_session_create(const tcb_weights* w, int32_t num_rows, int32_t row_len,
                              int64_t max_tokens, tcb_session** out) {
  tcb::clear_error();
  if (!out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_session_create: out is NULL");
  *out = nullptr;
  if (!w || num_rows <= 0 || row_len <= 0 || row_len % 8 != 0 || max_tokens < 0 ||
      static_cast<int64_t>(num_rows) * row_len > INT32_MAX)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_session_create: bad shape");
  if (row_len > w->cfg.max_pos)
    return fail(TCB_ERR_UNSUPPORTED, "tcb_session_create: row_len exceeds max_pos");
  if (tcb_status st = check_device()) return st;
  tcb_session* s = new (std::nothrow) tcb_session();
  if (!s) return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_session_create");
  s->w = w;
  s->rows = num_rows;
  s->row_len = row_len;
  s->max_tokens = max_tokens;
  const int64_t M = static_cast<int64_t>(num_rows) * row_len;
  // segment table of at most one segment per slot + row index + query-block order (tcb.h)
  s->seg_words = 4 * (1 + M) + (num_rows + 1 + 3) / 4 * 4 + ((M + 127) / 128 + 3) / 4 * 4;
  const size_t esz = w->cfg.dtype == 0 ? 4 : 2;
  s->out_bytes_per_token = esz * static_cast<size_t>(w->cfg.d_model);
  s->ws_bytes = ws_layout(w->cfg, M).total;
  bool ok = true;
  for (auto& sl : s->slot) {
    ok = ok && cudaMalloc(&sl.d_segtab, 4 * static_cast<size_t>(s->seg_words)) == cudaSuccess &&
         cudaMalloc(&sl.d_ids, 4 * static_cast<size_t>(std::max<int64_t>(max_tokens, 1))) == cudaSuccess &&
         cudaMalloc(&sl.d_rows, esz * static_cast<size_t>(M) * w->cfg.d_model) == cudaSuccess &&
         cudaMalloc(&sl.d_ws, s->ws_bytes) == cudaSuccess &&
         cudaMalloc(&sl.d_out, s->out_bytes_per_token * static_cast<size_t>(std::max<int64_t>(max_tokens, 1))) == cudaSuccess &&
         cudaMallocHost(&sl.h_seg, 4 * static_cast<size_t>(s->seg_words)) == cudaSuccess &&
         cudaEventCreateWithFlags(&sl.h2d_done, cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&sl.computed, cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&sl.d2h_done, cudaEventDisableTiming) == cudaSuccess;
  }
  ok = ok && cudaStreamCreateWithFlags(&s->up, cudaStreamNonBlocking) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    session_free(s);
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_session_create: device / pinned allocation failed");
  }
  *out = s;
  return TCB_OK;
}

tcb_status tcb_session_run(tcb_session* s, const tcb_plan* plan, const int32_t* h_token_ids,
                           void* h_out, tcb_stream_t stream, tcb_stream_t copy_stream,
                           int64_t* ticket) {
  tcb::clear_error();
  if (!s || !plan) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_session_run: NULL session or plan");
  if (plan->num_rows != s->rows || plan->row_len != s->row_len)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_session_run: plan shape differs from the session's");
  const int64_t T = plan->info.total_tokens;
  if (T > s->max_tokens)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_session_run: plan has more tokens than max_tokens");
  if (T > 0 && (!h_token_ids || !h_out))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_session_run: NULL host buffer");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  cudaStream_t cs = copy_stream ? reinterpret_cast<cudaStream_t>(copy_stream) : st;
  const int64_t call = s->calls++;
  tcb_session::Slot& sl = s->slot[call & 1];
  if (sl.ticket >= 0 && cudaEventSynchronize(sl.h2d_done) != cudaSuccess)   // staging reusable
    return cuda_fail(cudaGetLastError(), "tcb_session_run: wait for the slot's previous upload");
  if (tcb_status e = tcb_plan_write_segtab(plan, sl.h_seg, s->seg_words)) return e;
  const int64_t words = tcb_plan_segtab_words(plan);
  // the uploads run on the session's own stream, so they overlap the previous call's forward:
  // they only wait for the slot's previous forward to have finished reading its buffers
  cudaError_t e = cudaSuccess;
  if (sl.ticket >= 0) e = cudaStreamWaitEvent(s->up, sl.computed, 0);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(sl.d_segtab, sl.h_seg, 4 * static_cast<size_t>(words), cudaMemcpyHostToDevice, s->up);
  if (e == cudaSuccess && T > 0)
    e = cudaMemcpyAsync(sl.d_ids, h_token_ids, 4 * static_cast<size_t>(T), cudaMemcpyHostToDevice, s->up);
  if (e == cudaSuccess) e = cudaEventRecord(sl.h2d_done, s->up);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(st, sl.h2d_done, 0);
  // the slot's outputs may still be on their way to the host (previous call of the slot)
  if (e == cudaSuccess && sl.ticket >= 0) e = cudaStreamWaitEvent(st, sl.d2h_done, 0);
  if (e != cudaSuccess) return cuda_fail(e, "tcb_session_run: upload");
  // forward + unpack (fused into the last FFN2 + LN2 where the L2-exchange kernel runs)
  if (tcb_status r = tcb_encoder_forward_unpacked(s->w, plan, sl.d_segtab, sl.d_ids, sl.d_rows,
                                                  sl.d_out, sl.d_ws, s->ws_bytes, stream))
    return r;
  e = cudaEventRecord(sl.computed, st);
  if (e == cudaSuccess && cs != st) e = cudaStreamWaitEvent(cs, sl.computed, 0);
  if (e == cudaSuccess && T > 0)
    e = cudaMemcpyAsync(h_out, sl.d_out, s->out_bytes_per_token * static_cast<size_t>(T),
                        cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaEventRecord(sl.d2h_done, cs);
  if (e != cudaSuccess) return cuda_fail(e, "tcb_session_run: download");
  sl.ticket = call;
  if (ticket) *ticket = call;
  return TCB_OK;
}

tcb_status tcb_session_wait(tcb_session* s, int64_t ticket) {
  tcb::clear_error();
  if (!s || ticket < 0 || ticket >= s->calls)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_session_wait: unknown ticket");
  const tcb_session::Slot& sl = s->slot[ticket & 1];
  if (sl.ticket != ticket) return TCB_OK;              // the slot has been reused: long done
  const cudaError_t e = cudaEventSynchronize(sl.d2h_done);
  return e == cudaSuccess ? TCB_OK : cuda_fail(e, "tcb_session_wait");
}

void tcb_session_destroy(tcb_session* s) { session_free(s); }

// ---- op-level entry points (include/tcb_ops.h) ---------------------------------------------
tcb_status tcb_op_linear(int32_t dtype, int64_t M, int32_t N, int32_t K, const void* A,
                         const void* W, const float* bias, const void* R, int32_t epi, void* C,
                         tcb_stream_t stream) {
  tcb::clear_error();
  if (M < 0 || N <= 0 || K <= 0 || epi < 0 || epi > 3 || (dtype != 0 && dtype != 1))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_linear: bad shape / dtype / epilogue");
  if (M == 0) return TCB_OK;
  if (!A || !W || !bias || !C || (epi == TCB_EPI_BIAS_RESIDUAL && !R))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_linear: NULL pointer");
  if (tcb_status st = check_device()) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  if (dtype == 0) {
    TCB_LAUNCH(TCB_K_GEMM_QKV, s, tcb::k::launch_linear_f32(
                                      M, N, K, static_cast<const float*>(A),
                                      static_cast<const float*>(W), bias,
                                      static_cast<const float*>(R), epi, static_cast<float*>(C), s));
    return TCB_OK;
  }
  if (K % 64 != 0 || N % 64 != 0 || M > INT32_MAX)
    return fail(TCB_ERR_UNSUPPORTED, "tcb_op_linear (bf16): needs K % 64 == 0 and N % 64 == 0");
  tcb::k::GemmMaps maps;
  if (!tcb::k::make_gemm_a_map(&maps.a, A, M, K) || !tcb::k::make_gemm_w_map(&maps.w, W, N, K) ||
      !tcb::k::make_gemm_c_map(&maps.c, C, M, N) ||
      !tcb::k::make_gemm_c_map(&maps.r, epi == TCB_EPI_BIAS_RESIDUAL ? R : C, M, N))
    return fail(TCB_ERR_CUDA, "tcb_op_linear: cuTensorMapEncodeTiled failed (alignment?)");
  TCB_LAUNCH(TCB_K_GEMM_QKV, s, tcb::k::launch_linear_bf16_tc(maps, M, N, K, bias, epi, s));
  return TCB_OK;
}

tcb_status tcb_op_linear_ln(int64_t M, int32_t N, int32_t K, const void* A, const void* W,
                            const float* bias, const void* R, const float* gamma,
                            const float* beta, float eps, const int32_t* d_seg, void* C,
                            tcb_stream_t stream) {
  tcb::clear_error();
  if (M < 0 || N <= 0 || K <= 0) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_linear_ln: bad shape");
  if (M == 0) return TCB_OK;
  if (!A || !W || !bias || !R || !gamma || !beta || !C)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_linear_ln: NULL pointer");
  if (!tcb::k::linear_ln_supported(N) || K % 64 != 0 || M > INT32_MAX)
    return fail(TCB_ERR_UNSUPPORTED, "tcb_op_linear_ln: needs N in {512, 768, 1024} and K % 64 == 0");
  if (tcb_status st = check_device()) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  tcb::k::GemmMaps maps;
  if (!tcb::k::make_gemm_a_map(&maps.a, A, M, K) || !tcb::k::make_gemm_w_map(&maps.w, W, N, K) ||
      !tcb::k::make_gemm_w_half_map(&maps.w_half, W, N, K) ||
      !tcb::k::make_gemm_c_map(&maps.c, C, M, N) || !tcb::k::make_gemm_c_map(&maps.r, R, M, N))
    return fail(TCB_ERR_CUDA, "tcb_op_linear_ln: cuTensorMapEncodeTiled failed (alignment?)");
  maps.has_w_half = true;
  // the row-statistics scratch of the L2-exchange kernel (N = 512 / 1024 with K >= 2N, or
  // every N under TCB_LN_KERNEL=global): stream-ordered allocation per call, so calls on
  // different streams never share counters (the encoder forward uses its workspace instead)
  const size_t sb = (tcb::k::linear_ln_scratch_stats_bytes(M, N) + 255) & ~size_t(255);
  const size_t cb = tcb::k::linear_ln_scratch_cnt_bytes(M);
  void* buf = nullptr;
  if (cudaMallocAsync(&buf, sb + cb, s) != cudaSuccess) {
    cudaGetLastError();
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_op_linear_ln: scratch allocation failed");
  }
  float2* st = static_cast<float2*>(buf);
  int* cnt = reinterpret_cast<int*>(static_cast<uint8_t*>(buf) + sb);
  if (cudaMemsetAsync(cnt, 0, cb, s) != cudaSuccess) {
    cudaFreeAsync(buf, s);
    return fail(TCB_ERR_CUDA, "tcb_op_linear_ln: counter reset failed");
  }
  struct FreeAfter {                              // after the launch, in stream order
    void* p;
    cudaStream_t s;
    ~FreeAfter() { cudaFreeAsync(p, s); }
  } free_after{buf, s};
  TCB_LAUNCH(TCB_K_GEMM_O, s, tcb::k::launch_linear_ln_bf16_tc(maps, M, N, K, bias, gamma, beta,
                                                               eps, d_seg, s, st, cnt));
  return TCB_OK;
}

tcb_status tcb_op_attention(int32_t dtype, int64_t num_slots, int32_t d_model,
                            int32_t num_heads, const void* qkv, const int32_t* d_seg,
                            const int32_t* d_segtab, void* O, tcb_stream_t stream) {
  tcb::clear_error();
  if (num_slots < 0 || d_model <= 0 || num_heads <= 0 || d_model % num_heads != 0 ||
      (dtype != 0 && dtype != 1))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_attention: bad shape / dtype");
  if (num_slots == 0) return TCB_OK;
  if (!qkv || !d_seg || !d_segtab || !O) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_attention: NULL");
  const int dh = d_model / num_heads;
  if ((dtype == 1 && dh != 64) || (dtype == 0 && dh > 64))
    return fail(TCB_ERR_UNSUPPORTED, "tcb_op_attention: unsupported head dim");
  if (tcb_status st = check_device()) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const int4* segtab = reinterpret_cast<const int4*>(d_segtab);
  if (dtype == 1) {
    // the kernel's dynamic item counter: stream-ordered scratch, zeroed per call
    void* cnt = nullptr;
    if (cudaMallocAsync(&cnt, sizeof(int), s) != cudaSuccess) {
      cudaGetLastError();
      return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_op_attention: counter allocation failed");
    }
    struct FreeAfter {
      void* p;
      cudaStream_t s;
      ~FreeAfter() { cudaFreeAsync(p, s); }
    } free_after{cnt, s};
    if (cudaMemsetAsync(cnt, 0, sizeof(int), s) != cudaSuccess)
      return fail(TCB_ERR_CUDA, "tcb_op_attention: counter reset failed");
    TCB_LAUNCH(TCB_K_ATTN, s, attention_bf16(num_slots, d_model, num_heads, qkv, d_seg, segtab, O,
                                             static_cast<int*>(cnt), 0, s));
  }
  else
    TCB_LAUNCH(TCB_K_ATTN, s, tcb::k::launch_attention_f32(num_slots, d_model, num_heads,
                                                           static_cast<const float*>(qkv), d_seg,
                                                           segtab, static_cast<float*>(O), s));
  return TCB_OK;
}

tcb_status tcb_op_layernorm(int32_t dtype, int64_t rows, int32_t d, const void* Z,
                            const float* g, const float* b, float eps, const int32_t* d_seg,
                            void* Y, tcb_stream_t stream) {
  tcb::clear_error();
  if (rows < 0 || d <= 0 || (dtype != 0 && dtype != 1))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_layernorm: bad shape / dtype");
  if (rows == 0) return TCB_OK;
  if (!Z || !g || !b || !Y) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_op_layernorm: NULL");
  if (d % (dtype == 1 ? 8 : 4) != 0 || d > (dtype == 1 ? 2048 : 1024))
    return fail(TCB_ERR_UNSUPPORTED, "tcb_op_layernorm: d unsupported");
  if (tcb_status st = check_device()) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  TCB_LAUNCH(TCB_K_LN, s, tcb::k::launch_layernorm(dtype, rows, d, Z, g, b, eps, d_seg, Y, s));
  return TCB_OK;
}

}  // extern "C"

// ============================================================================================
// f4: auto-regressive decoder with early memory cleaning (include/tcb_decoder.h)
// ============================================================================================
#include <chrono>

#include "../../include/tcb_decoder.h"

struct tcb_decoder {
  const tcb_weights* enc = nullptr;
  std::vector<const void*> t;            // 20 per layer (tcb_decoder.h order)
  int32_t R = 0, T = 0;                  // max requests, max target tokens (= KV positions)
  int64_t max_slots = 0;
  std::vector<void*> bufs;               // every owned device allocation
  uint8_t* memkv = nullptr;              // S x [max_slots, 2d]  encoder memory K | V
  uint8_t* cache = nullptr;              // S x [R * T, 2d]      self-attention K | V
  void *x = nullptr, *qkv = nullptr, *att = nullptr, *x1 = nullptr, *qc = nullptr,
       *x2 = nullptr, *h = nullptr, *logits = nullptr;
  float* zero_bias = nullptr;            // [vocab] (the tied output projection has no bias)
  int32_t *act = nullptr, *out_len = nullptr, *done = nullptr, *flag = nullptr,
          *tmax = nullptr, *mem_start = nullptr, *mem_len = nullptr;
  struct LayerMaps {
    CUtensorMap qkv, o, q, kv, co, w1, w2, memkv_c;
  };
  std::vector<LayerMaps> wm;
  CUtensorMap w_logits{};
  CUtensorMap aX{}, aAtt{}, aX1{}, aX2{}, aH{};
  CUtensorMap cQkv{}, cX{}, cX1{}, cX2{}, cQc{}, cH{}, cLogits{};
  tcb_decode_stats stats{};
  int32_t last_rows = 0;
  int32_t* pin = nullptr;                // pinned host: active list [2][R], done flags [2][R]
  int32_t* tstep = nullptr;              // device step index read by the graphs' kernels
  struct StepGraph {                     // one decode step captured for a bucket of rows
    int32_t rows;
    const int32_t* tokens;
    cudaGraphExec_t exec;
    uint64_t launches;
  };
  std::vector<StepGraph> graphs;
  cudaStream_t cap_stream = nullptr;     // private stream the step graphs are captured on
  cudaEvent_t ev[2] = {nullptr, nullptr};  // done flags of a step on the host
  const void* L(int layer, int i) const { return t[20 * layer + i]; }
  const float* Lf(int layer, int i) const { return static_cast<const float*>(L(layer, i)); }
};

namespace {
enum { D_W_QKV = 0, D_B_QKV, D_W_O, D_B_O, D_LN1_G, D_LN1_B, D_W_Q, D_B_Q, D_W_KV, D_B_KV,
       D_W_CO, D_B_CO, D_LN2_G, D_LN2_B, D_W_1, D_B_1, D_W_2, D_B_2, D_LN3_G, D_LN3_B };

void free_decoder(tcb_decoder* dec) {
  for (auto& g : dec->graphs) cudaGraphExecDestroy(g.exec);
  if (dec->cap_stream) cudaStreamDestroy(dec->cap_stream);
  for (void* p : dec->bufs) cudaFree(p);
  if (dec->pin) cudaFreeHost(dec->pin);
  for (cudaEvent_t e : dec->ev)
    if (e) cudaEventDestroy(e);
  delete dec;
}

template <typename T>
bool dalloc(tcb_decoder* dec, T** p, size_t bytes) {
  void* v = nullptr;
  if (cudaMalloc(&v, bytes ? bytes : 16) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  dec->bufs.push_back(v);
  *p = static_cast<T*>(v);
  return true;
}
}  // namespace

extern "C" {

int32_t tcb_decoder_weights_count(const tcb_model_config* cfg) { return cfg ? 20 * cfg->num_layers : -1; }

tcb_status tcb_decoder_create(const tcb_weights* enc, const void* const* tensors,
                              int32_t num_tensors, int32_t max_requests, int64_t max_slots,
                              int32_t max_target, tcb_decoder** out) {
  tcb::clear_error();
  if (!out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_create: out is NULL");
  *out = nullptr;
  if (!enc) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_create: enc is NULL");
  const tcb_model_config& c = enc->cfg;
  if (c.dtype != 1 || c.pe == 2 || c.emb_ln || c.use_type_emb)
    return fail(TCB_ERR_UNSUPPORTED, "tcb_decoder_create: bf16 Transformer-family models only "
                                     "(sinusoidal PE, no embedding LN / type embedding)");
  if (c.d_model / c.num_heads != 64 || !tcb::k::linear_ln_supported(c.d_model) || c.vocab % 64)
    return fail(TCB_ERR_UNSUPPORTED, "tcb_decoder_create: needs d_head 64, d_model in "
                                     "{512, 768, 1024}, vocab % 64 == 0");
  if (!tensors || num_tensors != tcb_decoder_weights_count(&c))
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_create: expected " +
                                              std::to_string(tcb_decoder_weights_count(&c)) + " tensors");
  for (int i = 0; i < num_tensors; ++i)
    if (!tensors[i] || (reinterpret_cast<uintptr_t>(tensors[i]) & 15))
      return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_create: tensor " + std::to_string(i) +
                                                " is NULL or not 16-byte aligned");
  // (dec_attn walks any number of keys in chunks of its smem score buffer, so neither the
  // self-attention length max_target nor a request's source length is bounded by it)
  if (max_requests <= 0 || max_slots <= 0 || max_target <= 0 || max_target >= c.max_pos ||
      max_slots > INT32_MAX)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_create: bad capacities");
  if (tcb_status st = check_device()) return st;
  tcb_decoder* dec = new (std::nothrow) tcb_decoder();
  if (!dec) return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_decoder_create");
  dec->enc = enc;
  dec->t.assign(tensors, tensors + num_tensors);
  dec->R = max_requests;
  dec->T = max_target;
  dec->max_slots = max_slots;
  const int64_t d = c.d_model, f = c.d_ff, V = c.vocab, R = max_requests, S = c.num_layers;
  bool ok = dalloc(dec, &dec->memkv, sizeof(uint16_t) * S * max_slots * 2 * d) &&
            dalloc(dec, &dec->cache, sizeof(uint16_t) * S * R * max_target * 2 * d) &&
            dalloc(dec, &dec->x, 2 * R * d) && dalloc(dec, &dec->qkv, 2 * R * 3 * d) &&
            dalloc(dec, &dec->att, 2 * R * d) && dalloc(dec, &dec->x1, 2 * R * d) &&
            dalloc(dec, &dec->qc, 2 * R * d) && dalloc(dec, &dec->x2, 2 * R * d) &&
            dalloc(dec, &dec->h, 2 * R * f) && dalloc(dec, &dec->logits, 2 * R * V) &&
            dalloc(dec, &dec->zero_bias, sizeof(float) * V) &&
            dalloc(dec, &dec->act, 4 * R) && dalloc(dec, &dec->out_len, 4 * R) &&
            dalloc(dec, &dec->done, 4 * R) && dalloc(dec, &dec->flag, 4 * R) &&
            dalloc(dec, &dec->tmax, 4 * R) && dalloc(dec, &dec->mem_start, 4 * R) &&
            dalloc(dec, &dec->mem_len, 4 * R) && dalloc(dec, &dec->tstep, 16);
  ok = ok && cudaMallocHost(reinterpret_cast<void**>(&dec->pin), 16 * R) == cudaSuccess &&
       cudaEventCreateWithFlags(&dec->ev[0], cudaEventDisableTiming) == cudaSuccess &&
       cudaEventCreateWithFlags(&dec->ev[1], cudaEventDisableTiming) == cudaSuccess &&
       cudaStreamCreateWithFlags(&dec->cap_stream, cudaStreamNonBlocking) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    free_decoder(dec);
    return fail(TCB_ERR_OUT_OF_MEMORY, "tcb_decoder_create: device / pinned buffers");
  }
  if (cudaMemset(dec->zero_bias, 0, sizeof(float) * V) != cudaSuccess) {
    free_decoder(dec);
    return cuda_fail(cudaGetLastError(), "tcb_decoder_create: memset");
  }
  using namespace tcb::k;
  dec->wm.resize(S);
  for (int l = 0; l < S && ok; ++l) {
    auto& m = dec->wm[l];
    ok = make_gemm_w_map(&m.qkv, dec->L(l, D_W_QKV), 3 * d, d) &&
         make_gemm_w_map(&m.o, dec->L(l, D_W_O), d, d) &&
         make_gemm_w_map(&m.q, dec->L(l, D_W_Q), d, d) &&
         make_gemm_w_map(&m.kv, dec->L(l, D_W_KV), 2 * d, d) &&
         make_gemm_w_map(&m.co, dec->L(l, D_W_CO), d, d) &&
         make_gemm_w_map(&m.w1, dec->L(l, D_W_1), f, d) &&
         make_gemm_w_map(&m.w2, dec->L(l, D_W_2), d, f) &&
         make_gemm_c_map(&m.memkv_c, dec->memkv + sizeof(uint16_t) * l * max_slots * 2 * d,
                         max_slots, 2 * d);
  }
  ok = ok && make_gemm_w_map(&dec->w_logits, enc->tok_emb(), V, d) &&
       make_gemm_a_map(&dec->aX, dec->x, R, d) && make_gemm_a_map(&dec->aAtt, dec->att, R, d) &&
       make_gemm_a_map(&dec->aX1, dec->x1, R, d) && make_gemm_a_map(&dec->aX2, dec->x2, R, d) &&
       make_gemm_a_map(&dec->aH, dec->h, R, f) && make_gemm_c_map(&dec->cQkv, dec->qkv, R, 3 * d) &&
       make_gemm_c_map(&dec->cX, dec->x, R, d) && make_gemm_c_map(&dec->cX1, dec->x1, R, d) &&
       make_gemm_c_map(&dec->cX2, dec->x2, R, d) && make_gemm_c_map(&dec->cQc, dec->qc, R, d) &&
       make_gemm_c_map(&dec->cH, dec->h, R, f) && make_gemm_c_map(&dec->cLogits, dec->logits, R, V);
  if (!ok) {
    free_decoder(dec);
    return fail(TCB_ERR_CUDA, "tcb_decoder_create: cuTensorMapEncodeTiled failed");
  }
  *out = dec;
  return TCB_OK;
}

void tcb_decoder_destroy(tcb_decoder* dec) {
  if (dec) free_decoder(dec);
}

tcb_status tcb_decode_greedy(tcb_decoder* dec, const tcb_plan* plan, const void* d_enc_rows,
                             int32_t early_clean, int32_t* d_tokens, int32_t* h_lengths,
                             tcb_stream_t stream) {
  tcb::clear_error();
  const auto t0 = std::chrono::steady_clock::now();
  if (!dec || !plan || !h_lengths) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decode_greedy: NULL");
  const tcb_model_config& c = dec->enc->cfg;
  const int32_t n = plan->n;
  if (n > dec->R) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decode_greedy: more requests than max_requests");
  if (plan->info.num_slots > dec->max_slots)
    return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decode_greedy: plan larger than max_slots");
  if (tcb_status st = validate_plan_for(dec->enc, plan)) return st;
  for (int32_t r = 0; r < n; ++r) h_lengths[r] = 0;
  dec->stats = tcb_decode_stats{};
  if (n == 0) return TCB_OK;
  if (!d_enc_rows || !d_tokens) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decode_greedy: NULL device pointer");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const int d = c.d_model, f = c.d_ff, V = c.vocab, S = c.num_layers, T = dec->T;
  const int act_epi = c.act == 0 ? TCB_EPI_BIAS_GELU : TCB_EPI_BIAS_RELU;
  const int64_t M = plan->info.num_slots;
  // per-request host metadata: memory segment in the packed rows, generation budget (R32)
  std::vector<int32_t> act_h, tmax_h(n, 0), ms_h(n, 0), ml_h(n, 0);
  int32_t max_steps = 0;
  for (int32_t r = 0; r < n; ++r) {
    if (plan->req_row[r] < 0) continue;
    ms_h[r] = plan->req_row[r] * plan->row_len + plan->req_col[r];
    ml_h[r] = plan->lengths[r];
    tmax_h[r] = std::min(plan->lengths[r], T);
    max_steps = std::max(max_steps, tmax_h[r]);
    act_h.push_back(r);
  }
  cudaError_t e = cudaMemcpyAsync(dec->tmax, tmax_h.data(), 4 * n, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dec->mem_start, ms_h.data(), 4 * n, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dec->mem_len, ml_h.data(), 4 * n, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(dec->done, 0, 4 * n, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(dec->out_len, 0, 4 * n, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(d_tokens, 0xff, sizeof(int32_t) * n * T, s);
  if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: metadata upload");
  using namespace tcb::k;
  // encoder memory K | V of every layer over the packed rows (the request's segment is its
  // memory, R30): one GEMM per layer, M = num_slots
  {
    CUtensorMap aEnc;
    if (!make_gemm_a_map(&aEnc, d_enc_rows, M, d))
      return fail(TCB_ERR_CUDA, "tcb_decode_greedy: encoder-rows tensor map");
    for (int l = 0; l < S; ++l) {
      const GemmMaps g{aEnc, dec->wm[l].kv, dec->wm[l].memkv_c, dec->wm[l].memkv_c};
      TCB_LAUNCH(TCB_K_GEMM_QKV, s, launch_linear_bf16_tc(g, M, 2 * d, d, dec->Lf(l, D_B_KV), TCB_EPI_BIAS, s));
    }
  }
  const float scale = 1.f / 8.f;                          // 1 / sqrt(d_head = 64)
  const int64_t kv_per_pos = 2LL * d * 2 * S;             // bytes of K|V per position, all layers
  double kv_sum = 0.0;
  int32_t t = 0;
  bool act_dirty = true;
  // The host never waits for the step it has just enqueued: after enqueuing step t it reads
  // the done flags of step t-1 (pinned, double-buffered) while step t runs, and drops the
  // requests finished by then from the active set of step t+1 (early memory cleaning, R33,
  // one step late).  A request finished at step t is thus recomputed once more at step t+1;
  // the argmax kernel ignores it (its done flag is set) and no other row depends on it, so
  // the generated tokens are those of the synchronous loop.
  int32_t* act_pin[2] = {dec->pin, dec->pin + dec->R};
  int32_t* done_pin[2] = {dec->pin + 2 * dec->R, dec->pin + 3 * dec->R};
  // one decode step's kernels over `A` rows (step index t, or *d_t when d_t is set)
  auto enqueue_step = [&](int A, int t, const int32_t* d_t, cudaStream_t s) -> tcb_status {
    DecEmbedArgs ea{dec->act, d_tokens, T, t, 1, 2, d, A,
                    static_cast<const __nv_bfloat16*>(dec->enc->tok_emb()), dec->enc->pe_table,
                    c.emb_scale, static_cast<__nv_bfloat16*>(dec->x), d_t};
    TCB_LAUNCH(TCB_K_EMBED, s, launch_dec_embed(ea, s));
    for (int l = 0; l < S; ++l) {
      const auto& m = dec->wm[l];
      TCB_LAUNCH(TCB_K_GEMM_QKV, s, launch_linear_bf16_tc(GemmMaps{dec->aX, m.qkv, dec->cQkv, dec->cQkv},
                                                          A, 3 * d, d, dec->Lf(l, D_B_QKV), TCB_EPI_BIAS, s));
      DecAttnArgs sa{};
      sa.act = dec->act;
      sa.q = static_cast<const __nv_bfloat16*>(dec->qkv);
      sa.ldq = 3 * d;
      sa.qoff = 0;
      sa.kv = reinterpret_cast<__nv_bfloat16*>(dec->cache + sizeof(uint16_t) * l * dec->R * T * 2 * d);
      sa.ld_kv = 2 * d;
      sa.voff = d;
      sa.self = 1;
      sa.t = t;
      sa.t_cap = T;
      sa.d = d;
      sa.heads = c.num_heads;
      sa.rows = A;
      sa.scale = scale;
      sa.out = static_cast<__nv_bfloat16*>(dec->att);
      sa.d_t = d_t;
      TCB_LAUNCH(TCB_K_ATTN, s, launch_dec_attn(sa, s));
      TCB_LAUNCH(TCB_K_GEMM_O, s, launch_linear_ln_bf16_tc(GemmMaps{dec->aAtt, m.o, dec->cX1, dec->cX},
                                                           A, d, d, dec->Lf(l, D_B_O), dec->Lf(l, D_LN1_G),
                                                           dec->Lf(l, D_LN1_B), c.ln_eps, nullptr, s));
      TCB_LAUNCH(TCB_K_GEMM_QKV, s, launch_linear_bf16_tc(GemmMaps{dec->aX1, m.q, dec->cQc, dec->cQc},
                                                          A, d, d, dec->Lf(l, D_B_Q), TCB_EPI_BIAS, s));
      DecAttnArgs ca = sa;
      ca.q = static_cast<const __nv_bfloat16*>(dec->qc);
      ca.ldq = d;
      ca.kv = reinterpret_cast<__nv_bfloat16*>(dec->memkv + sizeof(uint16_t) * l * dec->max_slots * 2 * d);
      ca.self = 0;
      ca.mem_start = dec->mem_start;
      ca.mem_len = dec->mem_len;
      TCB_LAUNCH(TCB_K_ATTN, s, launch_dec_attn(ca, s));
      TCB_LAUNCH(TCB_K_GEMM_O, s, launch_linear_ln_bf16_tc(GemmMaps{dec->aAtt, m.co, dec->cX2, dec->cX1},
                                                           A, d, d, dec->Lf(l, D_B_CO), dec->Lf(l, D_LN2_G),
                                                           dec->Lf(l, D_LN2_B), c.ln_eps, nullptr, s));
      TCB_LAUNCH(TCB_K_GEMM_FFN1, s, launch_linear_bf16_tc(GemmMaps{dec->aX2, m.w1, dec->cH, dec->cH},
                                                           A, f, d, dec->Lf(l, D_B_1), act_epi, s));
      TCB_LAUNCH(TCB_K_GEMM_FFN2, s, launch_linear_ln_bf16_tc(GemmMaps{dec->aH, m.w2, dec->cX, dec->cX2},
                                                              A, d, f, dec->Lf(l, D_B_2), dec->Lf(l, D_LN3_G),
                                                              dec->Lf(l, D_LN3_B), c.ln_eps, nullptr, s));
    }
    // tied output projection (R31) and greedy argmax
    TCB_LAUNCH(TCB_K_GEMM_QKV, s, launch_linear_bf16_tc(GemmMaps{dec->aX, dec->w_logits, dec->cLogits, dec->cLogits},
                                                        A, V, d, dec->zero_bias, TCB_EPI_BIAS, s));
    DecArgmaxArgs ga{static_cast<const __nv_bfloat16*>(dec->logits), V, A, t, 2, T, dec->act,
                     dec->tmax, d_tokens, dec->out_len, dec->done, dec->flag, d_t};
    TCB_LAUNCH(TCB_K_UNPACK, s, launch_dec_argmax(ga, s));
    if (d_t) TCB_LAUNCH(TCB_K_UNPACK, s, launch_dec_step_advance(const_cast<int32_t*>(d_t), s));
    return TCB_OK;
  };
  // CUDA graphs per bucket of rows: on a non-default stream the caller is not capturing,
  // profiling off, TCB_NO_DEC_GRAPH unset
  bool use_graphs = std::getenv("TCB_NO_DEC_GRAPH") == nullptr;
  if (use_graphs) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    use_graphs = !g_prof_on;
  }
  if (use_graphs && s != nullptr) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone) {
      cudaGetLastError();
      use_graphs = false;
    }
  }
  auto bucket_of = [&](int A) {
    int b = 32;
    while (b < A) b *= 2;
    return std::min(b, dec->R);
  };
  int rows_up = -1;
  if (use_graphs) {
    e = cudaMemsetAsync(dec->tstep, 0, 4, s);
    if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: step index");
  }
  for (; t < max_steps && !act_h.empty(); ++t) {
    const int A = static_cast<int>(act_h.size());
    const int sl = t & 1;
    if (use_graphs) {
      // the step's kernels for a bucket of rows (the power of two >= A, at most R), captured
      // once per bucket and output buffer, replayed with the step index in device memory
      const int rows = bucket_of(A);
      tcb_decoder::StepGraph* gph = nullptr;
      for (auto& gg : dec->graphs)
        if (gg.rows == rows && gg.tokens == d_tokens) gph = &gg;
      if (!gph) {
        if (dec->graphs.size() >= 16) {        // bounded cache: start over
          for (auto& gg : dec->graphs) cudaGraphExecDestroy(gg.exec);
          dec->graphs.clear();
        }
        cudaGraph_t graph = nullptr;
        cudaStream_t cap = dec->cap_stream;
        e = cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal);
        if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: capture");
        const uint64_t c0 = g_launches.load();
        const tcb_status st = enqueue_step(rows, 0, dec->tstep, cap);
        e = cudaStreamEndCapture(cap, &graph);
        if (st != TCB_OK) { if (graph) cudaGraphDestroy(graph); return st; }
        if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: capture");
        cudaGraphExec_t exec = nullptr;
        e = cudaGraphInstantiate(&exec, graph, 0);
        cudaGraphDestroy(graph);
        if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: graph instantiate");
        dec->graphs.push_back({rows, d_tokens, exec, g_launches.load() - c0});
        g_launches.fetch_sub(dec->graphs.back().launches);   // counted when replayed
        gph = &dec->graphs.back();
      }
      if (act_dirty || rows != rows_up) {   // padded active list (rows >= A are -1)
        std::memcpy(act_pin[sl], act_h.data(), 4 * static_cast<size_t>(A));
        for (int i = A; i < rows; ++i) act_pin[sl][i] = -1;
        e = cudaMemcpyAsync(dec->act, act_pin[sl], 4 * rows, cudaMemcpyHostToDevice, s);
        if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: active set upload");
        act_dirty = false;
        rows_up = rows;
      }
      e = cudaGraphLaunch(gph->exec, s);
      if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: graph launch");
      g_launches.fetch_add(gph->launches, std::memory_order_relaxed);
    } else {
      if (act_dirty) {   // act_pin[sl]'s previous upload (step t-2) completed
        std::memcpy(act_pin[sl], act_h.data(), 4 * static_cast<size_t>(A));
        e = cudaMemcpyAsync(dec->act, act_pin[sl], 4 * A, cudaMemcpyHostToDevice, s);
        if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: active set upload");
        act_dirty = false;
      }
      if (tcb_status st = enqueue_step(A, t, nullptr, s)) return st;
    }
    e = cudaMemcpyAsync(done_pin[sl], dec->done, 4 * n, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaEventRecord(dec->ev[sl], s);
    if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: step");
    dec->last_rows = A;
    dec->stats.rows_computed += A;
    const int64_t kv_live = static_cast<int64_t>(A) * (t + 1) * kv_per_pos;
    kv_sum += static_cast<double>(kv_live);
    dec->stats.kv_bytes_peak = std::max(dec->stats.kv_bytes_peak, kv_live);
    if (t == 0) continue;
    // early memory cleaning (R33): requests finished by step t-1 leave the active set
    e = cudaEventSynchronize(dec->ev[sl ^ 1]);
    if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: step");
    const int32_t* dn = done_pin[sl ^ 1];
    std::vector<int32_t> next;
    next.reserve(A);
    for (int i = 0; i < A; ++i)
      if (!dn[act_h[i]]) next.push_back(act_h[i]);
    if (next.empty()) { ++t; break; }   // step t only recomputed finished requests
    if (early_clean && static_cast<int>(next.size()) != A) {
      act_h.swap(next);
      act_dirty = true;
    }
  }
  std::vector<int32_t> len_h(n);
  e = cudaMemcpyAsync(len_h.data(), dec->out_len, 4 * n, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(e, "tcb_decode_greedy: lengths");
  for (int32_t r = 0; r < n; ++r) {
    h_lengths[r] = len_h[r];
    dec->stats.tokens_generated += len_h[r];
  }
  dec->stats.steps = t;
  dec->stats.kv_bytes_avg = t > 0 ? kv_sum / t : 0.0;
  dec->stats.ms_total =
      std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return TCB_OK;
}

tcb_status tcb_decoder_stats(const tcb_decoder* dec, tcb_decode_stats* out) {
  tcb::clear_error();
  if (!dec || !out) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_stats: NULL");
  *out = dec->stats;
  return TCB_OK;
}

tcb_status tcb_decoder_last_logits(const tcb_decoder* dec, void* h_logits, int64_t capacity_elems,
                                   int32_t* rows) {
  tcb::clear_error();
  if (!dec || !h_logits || !rows) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_last_logits: NULL");
  const int64_t need = static_cast<int64_t>(dec->last_rows) * dec->enc->cfg.vocab;
  if (capacity_elems < need) return fail(TCB_ERR_INVALID_ARGUMENT, "tcb_decoder_last_logits: buffer too small");
  *rows = dec->last_rows;
  if (need == 0) return TCB_OK;
  cudaError_t e = cudaMemcpy(h_logits, dec->logits, 2 * need, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return cuda_fail(e, "tcb_decoder_last_logits");
  return TCB_OK;
}

}  // extern "C"
