// attention_tc.cu -- segment-masked self-attention on the 5th-generation tensor cores.
//
// Eq. (5)-(6): Att_CB(Q,K,V) = softmax(QK^T/sqrt(d) + M) V with M = 0 on the
// diagonal blocks Q_i K_i^T (Eq. (7)) and -inf elsewhere (R11).  Work item = (block of 128
// query slots, head).  The block's key interval [start of its first request, end of its
// last request) is walked in 128-key chunks; chunks outside it (other rows / other
// requests) are never loaded or computed.
//
// Two kernels: v3 (namespace v3, the default; two CTAs per SM, thread = query row, P in
// TMEM, see its header) and v1 (attn_tc_kernel below, TCB_ATTN=v1, kept for A/B: one CTA per
// SM, two softmax warps per row, P through shared memory).  v1 per chunk:
//   S = Q K^T       tcgen05.mma M=128 N=128 K=64 (Q, K K-major in smem) -> TMEM (fp32)
//   softmax         8 warps: thread = one query row (its TMEM lane) x 64 of the 128 key
//                   columns (key half h); mask = key outside the row's own request -> p = 0
//                   exactly; each key half keeps its OWN running max m_h and sum l_h (lazy
//                   rescaling: O_h is only rescaled when m_h grows by more than 2^8), so the
//                   two warps of a row never synchronise; p = 2^(s*log2e/sqrt(d) - m_h) in
//                   fp32, row sum in fp32, P rounded to bf16 into smem (K-major, 128B swizzle)
//   O_h += P_h V_h  tcgen05.mma M=128 N=64 K=64 per key half (P K-major, V MN-major in smem)
//                   into two TMEM accumulators; the epilogue merges them:
//                   O = (2^(m_0-m) O_0 + 2^(m_1-m) O_1) / (2^(m_0-m) l_0 + 2^(m_1-m) l_1)
// Roles (one CTA per SM, persistent over items): warp 0 = item metadata + Q TMA, warp 1 =
// MMA issuer (one thread), warp 2 = TMEM allocator, then K/V TMA producer, warps 4..11 =
// softmax/epilogue.  Q/K/V rings and S/P double buffers are mbarrier-guarded, so loads,
// QK^T of chunk c+1, softmax of chunk c and P V of chunk c-1 overlap.
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <string>

#include "kernels.h"

namespace tcb {
namespace k {
namespace {

constexpr int TQ = 128;                 // query slots per item (TMEM lanes)
constexpr int TK = 128;                 // keys per chunk
constexpr int DH = 64;                  // head dim
constexpr int kSmWarps = 8;             // softmax warps (2 per TMEM lane quarter)
constexpr int kEpWarps = 4;             // output epilogue warps (one per TMEM lane quarter)
constexpr int kThreads = (4 + kSmWarps + kEpWarps) * 32;
constexpr int kQStages = 3, kKVStages = 3;
constexpr int kTileBytes = 128 * DH * 2;            // 16 KB: Q, K or V tile (128 rows x 128 B)
constexpr int kPBytes = TQ * TK * 2;                // 32 KB: P tile (two 64-key K blocks)
constexpr float kRescaleLog2 = 8.f;                 // lazy-rescale threshold (log2 units)

struct ItemInfo {
  int2 rows[TQ];   // [start, end) of the request of query slot q0 + r (empty for pads)
  int kbase, nch;  // first key (8-aligned) and number of 128-key chunks
};

constexpr int kSmemBytes = 1024 + kQStages * kTileBytes + 2 * kKVStages * kTileBytes +
                           2 * kPBytes + kQStages * static_cast<int>(sizeof(ItemInfo)) + 6144;

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void tma_load(uint32_t dst, const CUtensorMap* map, uint32_t bar,
                                         int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar)
               : "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                       uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]),
        "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]),
        "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]),
        "=r"(r[31])
      : "r"(taddr)
      : "memory");
}
// Two 32-column loads AND the wait in one asm statement: the compiler must not touch the
// destination registers (e.g. spill them) before tcgen05.wait::ld has completed.
__device__ __forceinline__ void tmem_ld64_sync(uint32_t taddr, uint32_t (&r)[64]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%64];\n\t"
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,"
      "%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%65];\n\t"
      "tcgen05.wait::ld.sync.aligned;"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]),
        "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]),
        "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]),
        "=r"(r[31]), "=r"(r[32]), "=r"(r[33]), "=r"(r[34]), "=r"(r[35]), "=r"(r[36]),
        "=r"(r[37]), "=r"(r[38]), "=r"(r[39]), "=r"(r[40]), "=r"(r[41]), "=r"(r[42]),
        "=r"(r[43]), "=r"(r[44]), "=r"(r[45]), "=r"(r[46]), "=r"(r[47]), "=r"(r[48]),
        "=r"(r[49]), "=r"(r[50]), "=r"(r[51]), "=r"(r[52]), "=r"(r[53]), "=r"(r[54]),
        "=r"(r[55]), "=r"(r[56]), "=r"(r[57]), "=r"(r[58]), "=r"(r[59]), "=r"(r[60]),
        "=r"(r[61]), "=r"(r[62]), "=r"(r[63])
      : "r"(taddr), "r"(taddr + 32)
      : "memory");
}
__device__ __forceinline__ void tmem_ld32_sync(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n\t"
      "tcgen05.wait::ld.sync.aligned;"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]),
        "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]),
        "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]),
        "=r"(r[31])
      : "r"(taddr)
      : "memory");
}
// tmem_ld64_sync for two 32-key groups whose loads are skipped when the group is dead for
// the whole warp (l0 / l1 warp-uniform; the skipped registers are not read by the caller).
// One asm statement per case, each declaring all 64 outputs: nothing to preserve.
__device__ __forceinline__ void tmem_ld32x2_sync(uint32_t a0, uint32_t a1, uint32_t (&r)[64]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%64];\n\t"
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,"
      "%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%65];\n\t"
      "tcgen05.wait::ld.sync.aligned;"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]),
        "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]),
        "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]),
        "=r"(r[31]), "=r"(r[32]), "=r"(r[33]), "=r"(r[34]), "=r"(r[35]), "=r"(r[36]),
        "=r"(r[37]), "=r"(r[38]), "=r"(r[39]), "=r"(r[40]), "=r"(r[41]), "=r"(r[42]),
        "=r"(r[43]), "=r"(r[44]), "=r"(r[45]), "=r"(r[46]), "=r"(r[47]), "=r"(r[48]),
        "=r"(r[49]), "=r"(r[50]), "=r"(r[51]), "=r"(r[52]), "=r"(r[53]), "=r"(r[54]),
        "=r"(r[55]), "=r"(r[56]), "=r"(r[57]), "=r"(r[58]), "=r"(r[59]), "=r"(r[60]),
        "=r"(r[61]), "=r"(r[62]), "=r"(r[63])
      : "r"(a0), "r"(a1)
      : "memory");
}
__device__ __forceinline__ void tmem_ld64_live(uint32_t taddr, uint32_t (&r)[64], bool l0, bool l1) {
#ifdef TCB_ATTN_LOAD_DEAD
  l0 = l1 = true;
#endif
  if (l0 && l1) {
    tmem_ld32x2_sync(taddr, taddr + 32, r);
  } else if (l0) {
    tmem_ld32_sync(taddr, *reinterpret_cast<uint32_t(*)[32]>(&r[0]));
  } else if (l1) {
    tmem_ld32_sync(taddr + 32, *reinterpret_cast<uint32_t(*)[32]>(&r[32]));
  }
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]),
      "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]),
      "r"(v[15]), "r"(v[16]), "r"(v[17]), "r"(v[18]), "r"(v[19]), "r"(v[20]), "r"(v[21]),
      "r"(v[22]), "r"(v[23]), "r"(v[24]), "r"(v[25]), "r"(v[26]), "r"(v[27]), "r"(v[28]),
      "r"(v[29]), "r"(v[30]), "r"(v[31])
      : "memory");
}
__device__ __forceinline__ float fmax3(float a, float b, float c) {
  float d;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// packed fp32x2 arithmetic (sm_100 FFMA2 / FADD2: two lanes of work per issue slot)
__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
  unsigned long long r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;"
      : "=l"(r)
      : "l"(*reinterpret_cast<unsigned long long*>(&a)), "l"(*reinterpret_cast<unsigned long long*>(&b)),
        "l"(*reinterpret_cast<unsigned long long*>(&c)));
  return *reinterpret_cast<float2*>(&r);
}
__device__ __forceinline__ float2 fadd2(float2 a, float2 b) {
  unsigned long long r;
  asm("add.rn.f32x2 %0, %1, %2;"
      : "=l"(r)
      : "l"(*reinterpret_cast<unsigned long long*>(&a)), "l"(*reinterpret_cast<unsigned long long*>(&b)));
  return *reinterpret_cast<float2*>(&r);
}
// K-major operand, rows of 128 B, 128B swizzle, 8-row groups 1024 B apart (SBO).
__device__ __forceinline__ uint64_t desc_kmajor(uint32_t saddr) {
  return static_cast<uint64_t>((saddr & 0x3FFFFu) >> 4) | (static_cast<uint64_t>(1) << 16) |
         (static_cast<uint64_t>(1024 >> 4) << 32) | (static_cast<uint64_t>(1) << 46) |
         (static_cast<uint64_t>(2) << 61);
}
// MN-major operand (V as the B of P.V): each 128 B row holds the 64 N-elements of one K
// index; 8 K-rows form a 1024 B swizzle atom (SBO); a single 64-wide N block (LBO unused).
__device__ __forceinline__ uint64_t desc_mnmajor(uint32_t saddr) {
  return static_cast<uint64_t>((saddr & 0x3FFFFu) >> 4) | (static_cast<uint64_t>(1) << 16) |
         (static_cast<uint64_t>(1024 >> 4) << 32) | (static_cast<uint64_t>(1) << 46) |
         (static_cast<uint64_t>(2) << 61);
}
// kind::f16 instruction descriptors: fp32 D, bf16 A/B.
constexpr uint32_t kIdescQK = (1u << 4) | (1u << 7) | (1u << 10) | ((128u >> 3) << 17) | ((128u >> 4) << 24);
constexpr uint32_t kIdescPV = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((64u >> 3) << 17) |
                              ((128u >> 4) << 24);

__device__ void compute_info(ItemInfo* inf, const int32_t* __restrict__ seg_ids,
                             const int4* __restrict__ segtab, int64_t q0, int64_t num_slots,
                             int lane) {
  int lo = INT_MAX, hi = -1;
#pragma unroll
  for (int i = 0; i < TQ / 32; ++i) {
    const int64_t row = q0 + lane + 32 * i;
    const int sg = row < num_slots ? __ldg(&seg_ids[row]) : -1;
    int2 v = make_int2(0, 0);
    if (sg >= 0) {
      const int4 rec = __ldg(&segtab[1 + sg]);
      v = make_int2(rec.x, rec.x + rec.y);
      lo = min(lo, v.x);
      hi = max(hi, v.y);
    }
    inf->rows[lane + 32 * i] = v;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
  }
  if (lane == 0) {
    if (hi < 0) {
      inf->kbase = 0;
      inf->nch = 0;
    } else {
      const int kb = lo & ~7;
      inf->kbase = kb;
      inf->nch = (hi - kb + TK - 1) / TK;
    }
  }
  __syncwarp();
}

__global__ void __launch_bounds__(kThreads, 1)
attn_tc_kernel(const __grid_constant__ CUtensorMap tmQKV, const int32_t* __restrict__ seg_ids,
               const int4* __restrict__ segtab, __nv_bfloat16* __restrict__ O,
               int64_t num_slots, int d_model, int num_heads, int num_items, float scale_log2) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023) & ~1023u;
  const uint32_t sQ = base;                                    // [3][128 x 64]
  const uint32_t sK = sQ + kQStages * kTileBytes;              // [3][128 x 64]
  const uint32_t sV = sK + kKVStages * kTileBytes;             // [3][128 x 64]
  const uint32_t sP = sV + kKVStages * kTileBytes;             // [2][2 blocks][128 x 64]
  uint8_t* gen = smem_raw + (sP + 2 * kPBytes - raw);
  ItemInfo* infos = reinterpret_cast<ItemInfo*>(gen);          // [3]
  float* mbuf = reinterpret_cast<float*>(gen + kQStages * sizeof(ItemInfo));  // row maxima: [2 items][2 halves][128]
  float* lbuf = mbuf + 4 * TQ;                                 // row sums: [2 items][2 halves][128]
  int* meta = reinterpret_cast<int*>(lbuf + 4 * TQ);           // [2 items]: item has an O
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(meta + 4);
  const uint32_t bars = (smem_u32(tmem_slot + 4) + 7) & ~7u;
  const uint32_t q_full = bars, q_empty = q_full + 8 * kQStages;
  const uint32_t kv_full = q_empty + 8 * kQStages, kv_empty = kv_full + 8 * kKVStages;
  const uint32_t s_full = kv_empty + 8 * kKVStages, s_empty = s_full + 16;
  const uint32_t p_full = s_empty + 16, p_empty = p_full + 16;
  const uint32_t o_full = p_empty + 16, o_empty = o_full + 16;   // [2] each (O double buffer)
  const uint32_t info_full = o_empty + 16;                     // [3]
  const uint32_t l_full = info_full + 8 * kQStages, l_empty = l_full + 16;   // [2] each

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kQStages; ++i) {
      mbar_init(q_full + 8 * i, 1);
      mbar_init(q_empty + 8 * i, 1 + kSmWarps + 1);   // MMA + softmax warps + K/V producer
      mbar_init(info_full + 8 * i, 1);
    }
    for (int i = 0; i < kKVStages; ++i) { mbar_init(kv_full + 8 * i, 1); mbar_init(kv_empty + 8 * i, 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(s_full + 8 * i, 1);
      mbar_init(s_empty + 8 * i, kSmWarps);
      mbar_init(p_full + 8 * i, kSmWarps);
      mbar_init(p_empty + 8 * i, 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(o_full + 8 * i, 1);
      mbar_init(o_empty + 8 * i, kEpWarps);
      mbar_init(l_full + 8 * i, kSmWarps);
      mbar_init(l_empty + 8 * i, kEpWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)), "r"(512) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;           // S0: +0, S1: +128, O[item & 1][half]: +256 + 128 (item & 1) + 64 half
  pdl_wait();                                 // QKV / segment ids come from earlier kernels
  pdl_trigger();

  if (warp == 0) {
    // ================= item metadata + Q tile =================
    if (lane == 0) asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmQKV)) : "memory");
    int qs = 0;
    uint32_t qph = 0;
    for (int item = blockIdx.x; item < num_items; item += gridDim.x) {
      const int qb = item / num_heads, h = item % num_heads;
      const int64_t q0 = static_cast<int64_t>(qb) * TQ;
      if (lane == 0) mbar_wait(q_empty + 8 * qs, qph ^ 1);
      __syncwarp();
      ItemInfo* inf = infos + qs;
      compute_info(inf, seg_ids, segtab, q0, num_slots, lane);
      if (lane == 0) {
        mbar_arrive(info_full + 8 * qs);
        if (inf->nch == 0) {
          mbar_arrive(q_full + 8 * qs);
        } else {
          mbar_expect_tx(q_full + 8 * qs, kTileBytes);
          tma_load(sQ + qs * kTileBytes, &tmQKV, q_full + 8 * qs, h * DH, static_cast<int>(q0));
        }
      }
      if (++qs == kQStages) { qs = 0; qph ^= 1; }
    }
  } else if (warp == 2) {
    // ================= K/V chunks =================
    if (lane == 0) {
      int qs = 0, ks = 0;
      uint32_t qph = 0, kph = 0;
      for (int item = blockIdx.x; item < num_items; item += gridDim.x) {
        const int h = item % num_heads;
        mbar_wait(info_full + 8 * qs, qph);
        const int kbase = infos[qs].kbase, nch = infos[qs].nch;
        mbar_arrive(q_empty + 8 * qs);
        if (++qs == kQStages) { qs = 0; qph ^= 1; }
        for (int c = 0; c < nch; ++c) {
          mbar_wait(kv_empty + 8 * ks, kph ^ 1);
          mbar_expect_tx(kv_full + 8 * ks, 2 * kTileBytes);
          tma_load(sK + ks * kTileBytes, &tmQKV, kv_full + 8 * ks, d_model + h * DH, kbase + c * TK);
          tma_load(sV + ks * kTileBytes, &tmQKV, kv_full + 8 * ks, 2 * d_model + h * DH, kbase + c * TK);
          if (++ks == kKVStages) { ks = 0; kph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ================= MMA issuer =================
    // Flat software pipeline over all chunks of all items: S = Q K^T of chunk g is issued
    // before P V of chunk g-1 waits for its P, also across item boundaries, so the softmax
    // warps find the next S ready when they finish a chunk.
    int qs = 0, ks = 0;
    uint32_t qph = 0, kph = 0;
    uint32_t gc = 0;            // global chunk counter (S / P double buffers)
    uint32_t it = 0;            // items with at least one chunk (O double buffer)
    struct Pend {
      uint32_t gc, it;
      int stage;
      bool first, last, valid;
    } pend{0, 0, 0, false, false, false};
    auto issue_pv = [&](const Pend& pp) {
      const uint32_t b = pp.gc & 1, u = pp.gc >> 1;
      mbar_wait(p_full + 8 * b, u & 1);
      if (pp.first) mbar_wait(o_empty + 8 * (pp.it & 1), ((pp.it >> 1) & 1) ^ 1);
      tc_fence_after();
      if (lane == 0) {
        const uint32_t pa = sP + b * kPBytes, va = sV + pp.stage * kTileBytes;
#pragma unroll
        for (int k = 0; k < TK / 16; ++k) {
          const uint32_t a_addr = pa + (k >> 2) * kTileBytes + (k & 3) * 32;
          tc_mma(tmem + 256 + (pp.it & 1) * 128 + (k >> 2) * 64, desc_kmajor(a_addr),
                 desc_mnmajor(va + k * 2048), kIdescPV, (!pp.first || (k & 3) > 0) ? 1u : 0u);
        }
        tc_commit(p_empty + 8 * b);
        tc_commit(kv_empty + 8 * pp.stage);
        if (pp.last) tc_commit(o_full + 8 * (pp.it & 1));
      }
      __syncwarp();
    };
    for (int item = blockIdx.x; item < num_items; item += gridDim.x) {
      mbar_wait(q_full + 8 * qs, qph);
      const int nch = infos[qs].nch;
      const uint32_t qaddr = sQ + qs * kTileBytes;
      tc_fence_after();
      if (nch == 0) {
        // An empty item must not hold back the pending P V: the softmax warps are waiting
        // for it (deferred epilogue of the previous item) and would stop releasing Q slots,
        // so a run of more than kQStages empty items would deadlock the Q ring.
        if (pend.valid) {
          issue_pv(pend);
          pend.valid = false;
        }
        if (lane == 0) mbar_arrive(q_empty + 8 * qs);
      }
      for (int c = 0; c < nch; ++c) {
        const uint32_t b = gc & 1, u = gc >> 1;
        mbar_wait(kv_full + 8 * ks, kph);
        mbar_wait(s_empty + 8 * b, (u & 1) ^ 1);
        tc_fence_after();
        if (lane == 0) {
          const uint32_t ka = sK + ks * kTileBytes;
#pragma unroll
          for (int k = 0; k < DH / 16; ++k)
            tc_mma(tmem + b * 128, desc_kmajor(qaddr + k * 32), desc_kmajor(ka + k * 32), kIdescQK,
                   k > 0 ? 1u : 0u);
          tc_commit(s_full + 8 * b);
          if (c == nch - 1) tc_commit(q_empty + 8 * qs);
        }
        __syncwarp();
        if (pend.valid) issue_pv(pend);
        pend = Pend{gc, it, ks, c == 0, c == nch - 1, true};
        if (++ks == kKVStages) { ks = 0; kph ^= 1; }
        ++gc;
      }
      if (nch > 0) ++it;
      if (++qs == kQStages) { qs = 0; qph ^= 1; }
    }
    if (pend.valid) issue_pv(pend);
  } else if (warp >= 4 + kSmWarps) {
    // ================= output epilogue: O / l -> bf16 -> global =================
    // Per item (in order): the softmax warps hand over the row sums (and whether the item
    // had any chunk); O comes from TMEM (double-buffered); pad / empty rows are written 0.
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(q * 32) << 16;
    uint32_t oit = 0;
    int k = 0;
    for (int item = blockIdx.x; item < num_items; item += gridDim.x, ++k) {
      const int qb = item / num_heads, h = item % num_heads;
      const int lb = k & 1;
      mbar_wait(l_full + 8 * lb, (k >> 1) & 1);
      const bool has_o = meta[lb] != 0;
      // merge the two key halves: weights 2^(m_h - m) (0 for a half that saw no key)
      const float m0 = mbuf[(lb * 2) * TQ + row], m1 = mbuf[(lb * 2 + 1) * TQ + row];
      const float l0 = lbuf[(lb * 2) * TQ + row], l1 = lbuf[(lb * 2 + 1) * TQ + row];
      const float mm = fmaxf(m0, m1);
      const float w0 = m0 == -INFINITY ? 0.f : ex2((m0 - mm) * scale_log2);
      const float w1 = m1 == -INFINITY ? 0.f : ex2((m1 - mm) * scale_log2);
      const float den = w0 * l0 + w1 * l1;
      const float inv = (has_o && den > 0.f) ? 1.f / den : 0.f;
      const float a0 = w0 * inv, a1 = w1 * inv;
      const int64_t grow = static_cast<int64_t>(qb) * TQ + row;
      uint4* dst = reinterpret_cast<uint4*>(O + grow * d_model + h * DH);
      const uint32_t os = oit & 1;
      if (has_o) {
        mbar_wait(o_full + 8 * os, (oit >> 1) & 1);
        tc_fence_after();
      }
#pragma unroll 1
      for (int cq = 0; cq < 2; ++cq) {          // 32 output columns at a time
        uint32_t o[64];
        if (has_o) {
          const uint32_t ob = tmem + lane_off + 256 + os * 128 + cq * 32;
          asm volatile(
              "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
              "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
              "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%64];\n\t"
              "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
              "{%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,"
              "%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%65];\n\t"
              "tcgen05.wait::ld.sync.aligned;"
              : "=r"(o[0]), "=r"(o[1]), "=r"(o[2]), "=r"(o[3]), "=r"(o[4]), "=r"(o[5]), "=r"(o[6]),
                "=r"(o[7]), "=r"(o[8]), "=r"(o[9]), "=r"(o[10]), "=r"(o[11]), "=r"(o[12]),
                "=r"(o[13]), "=r"(o[14]), "=r"(o[15]), "=r"(o[16]), "=r"(o[17]), "=r"(o[18]),
                "=r"(o[19]), "=r"(o[20]), "=r"(o[21]), "=r"(o[22]), "=r"(o[23]), "=r"(o[24]),
                "=r"(o[25]), "=r"(o[26]), "=r"(o[27]), "=r"(o[28]), "=r"(o[29]), "=r"(o[30]),
                "=r"(o[31]), "=r"(o[32]), "=r"(o[33]), "=r"(o[34]), "=r"(o[35]), "=r"(o[36]),
                "=r"(o[37]), "=r"(o[38]), "=r"(o[39]), "=r"(o[40]), "=r"(o[41]), "=r"(o[42]),
                "=r"(o[43]), "=r"(o[44]), "=r"(o[45]), "=r"(o[46]), "=r"(o[47]), "=r"(o[48]),
                "=r"(o[49]), "=r"(o[50]), "=r"(o[51]), "=r"(o[52]), "=r"(o[53]), "=r"(o[54]),
                "=r"(o[55]), "=r"(o[56]), "=r"(o[57]), "=r"(o[58]), "=r"(o[59]), "=r"(o[60]),
                "=r"(o[61]), "=r"(o[62]), "=r"(o[63])
              : "r"(ob), "r"(ob + 64)
              : "memory");
        }
        if (cq == 1) {                          // O and the row statistics are consumed
          tc_fence_before();
          __syncwarp();
          if (lane == 0) {
            if (has_o) mbar_arrive(o_empty + 8 * os);
            mbar_arrive(l_empty + 8 * lb);
          }
        }
        if (grow < num_slots) {
#pragma unroll
          for (int t = 0; t < 4; ++t) {
            uint4 x;
            uint32_t* xp = reinterpret_cast<uint32_t*>(&x);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const int j = 8 * t + 2 * e;
              const float a = inv == 0.f ? 0.f
                                         : fmaf(__uint_as_float(o[j]), a0, __uint_as_float(o[32 + j]) * a1);
              const float bq = inv == 0.f ? 0.f
                                          : fmaf(__uint_as_float(o[j + 1]), a0, __uint_as_float(o[33 + j]) * a1);
              __nv_bfloat162 hv = __floats2bfloat162_rn(a, bq);
              xp[e] = *reinterpret_cast<uint32_t*>(&hv);
            }
            dst[cq * 4 + t] = x;
          }
        }
      }
      if (has_o) ++oit;
    }
  } else if (warp >= 4) {
    // ================= softmax =================
    const int sw = warp - 4;
    const int q = warp & 3;                 // TMEM lane quarter
    const int half = sw >> 2;               // key columns [64*half, 64*half+64) of a chunk
    const int row = q * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(q * 32) << 16;
    int qs = 0;
    uint32_t qph = 0, gc = 0, it = 0;
#ifdef TCB_ATTN_PROBE
    long long p_start = clock64(), p_sfull = 0, p_ld = 0, p_max = 0, p_pempty = 0, p_exp = 0, p_q = 0, p_fin = 0, p_resc = 0;
#endif
    int ic = 0;                             // items processed (row-sum hand-over buffers)
    for (int item = blockIdx.x; item < num_items; item += gridDim.x) {
      const int qb = item / num_heads, h = item % num_heads;
#ifdef TCB_ATTN_PROBE
      long long tq = clock64();
#endif
      mbar_wait(q_full + 8 * qs, qph);
#ifdef TCB_ATTN_PROBE
      p_q += clock64() - tq;
#endif
      const ItemInfo* inf = infos + qs;
      const int2 rr = inf->rows[row];
      const int kbase = inf->kbase, nch = inf->nch;
      __syncwarp();
      if (lane == 0) mbar_arrive(q_empty + 8 * qs);   // metadata copied to registers
      if (++qs == kQStages) { qs = 0; qph ^= 1; }
      // key interval of this warp's 32 rows: union [ulo, uhi) and intersection [ilo, ihi)
      // (a pad row empties the intersection)
      const bool real = rr.y > rr.x;
      int ulo = real ? rr.x : INT_MAX, uhi = real ? rr.y : -1;
      int ilo = real ? rr.x : INT_MAX, ihi = real ? rr.y : -1;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        ulo = min(ulo, __shfl_xor_sync(0xffffffffu, ulo, o));
        uhi = max(uhi, __shfl_xor_sync(0xffffffffu, uhi, o));
        ilo = max(ilo, __shfl_xor_sync(0xffffffffu, ilo, o));
        ihi = min(ihi, __shfl_xor_sync(0xffffffffu, ihi, o));
      }
      float m_used = -INFINITY, l = 0.f;
      for (int c = 0; c < nch; ++c) {
        const uint32_t b = gc & 1, u = gc >> 1;
#ifdef TCB_ATTN_PROBE
        long long t0 = clock64();
#endif
        mbar_wait(s_full + 8 * b, u & 1);
#ifdef TCB_ATTN_PROBE
        long long t1 = clock64();
        p_sfull += t1 - t0;
#endif
        tc_fence_after();
        uint32_t sr[64];
        tmem_ld64_sync(tmem + lane_off + b * 128 + half * 64, sr);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(s_empty + 8 * b);
#ifdef TCB_ATTN_PROBE
        long long t2 = clock64();
        p_ld += t2 - t1;
#endif
        // 32-key groups of this warp's half: dead (no key of any of its rows' requests:
        // skipped, P = 0), interior (inside every row's request: no mask) or boundary
        // (masked per element: key outside the row's own request -> -inf, R11)
        const int k0 = kbase + c * TK + 64 * half;
        const int jlo = max(rr.x - k0, 0), jhi = min(rr.y - k0, 64);
        bool live[2], inner[2];
#pragma unroll
        for (int gi = 0; gi < 2; ++gi) {
          const int gk = k0 + 32 * gi;
          live[gi] = gk < uhi && gk + 32 > ulo;
          inner[gi] = gk >= ilo && gk + 32 <= ihi;
        }
        // row max with 8 independent partial maxima (short dependency chains)
        float mxp[8];
#pragma unroll
        for (int t = 0; t < 8; ++t) mxp[t] = -INFINITY;
#pragma unroll
        for (int gi = 0; gi < 2; ++gi) {
          if (!live[gi]) continue;
          if (inner[gi]) {
#pragma unroll
            for (int j = 32 * gi; j < 32 * gi + 32; j += 2)
              mxp[(j >> 1) & 7] = fmax3(mxp[(j >> 1) & 7], __uint_as_float(sr[j]), __uint_as_float(sr[j + 1]));
          } else {
            // valid keys of this row in the group as a bit mask: one bit test per score
            const int lo = min(max(jlo - 32 * gi, 0), 32), hi = min(max(jhi - 32 * gi, 0), 32);
            const uint32_t below_hi = hi >= 32 ? 0xffffffffu : (1u << hi) - 1u;
            const uint32_t from_lo = lo >= 32 ? 0u : ~((1u << lo) - 1u);   // no shift by 32
            const uint32_t vm = below_hi & from_lo;
#pragma unroll
            for (int j = 32 * gi; j < 32 * gi + 32; j += 2) {
              const float v0 = (vm & (1u << (j - 32 * gi))) ? __uint_as_float(sr[j]) : -INFINITY;
              const float v1 = (vm & (2u << (j - 32 * gi))) ? __uint_as_float(sr[j + 1]) : -INFINITY;
              sr[j] = __float_as_uint(v0);
              sr[j + 1] = __float_as_uint(v1);
              mxp[(j >> 1) & 7] = fmax3(mxp[(j >> 1) & 7], v0, v1);
            }
          }
        }
        // this key half's row max (the other half keeps its own; merged in the epilogue)
        const float rmax = fmaxf(fmaxf(fmaxf(mxp[0], mxp[1]), fmaxf(mxp[2], mxp[3])),
                                 fmaxf(fmaxf(mxp[4], mxp[5]), fmaxf(mxp[6], mxp[7])));
#ifdef TCB_ATTN_PROBE
        long long t3 = clock64();
        p_max += t3 - t2;
#endif
        // lazy rescale: a row moves its max only when it grew by more than 2^8.  The O
        // update uses warp-collective tcgen05.ld/st, so the decision is made per warp (any
        // lane) and lanes that keep their max scale by 1.
        bool grow = false;
        if (rmax != -INFINITY) {
          if (m_used == -INFINITY) m_used = rmax;   // nothing accumulated yet for this row
          else grow = (rmax - m_used) * scale_log2 > kRescaleLog2;
        }
        if (__any_sync(0xffffffffu, grow)) {
          // O must be current before it is rescaled: wait for P V of chunk c-1
          const uint32_t pb = (gc - 1) & 1, pu = (gc - 1) >> 1;
          mbar_wait(p_empty + 8 * pb, pu & 1);
          tc_fence_after();
          const float f = grow ? ex2((m_used - rmax) * scale_log2) : 1.f;
          const uint32_t oaddr = tmem + lane_off + 256 + (it & 1) * 128 + half * 64;
#pragma unroll 1
          for (int cq = 0; cq < 2; ++cq) {
            uint32_t o[32];
            tmem_ld32_sync(oaddr + 32 * cq, o);
#pragma unroll
            for (int t = 0; t < 32; ++t) o[t] = __float_as_uint(__uint_as_float(o[t]) * f);
            tmem_st32(oaddr + 32 * cq, o);
          }
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          if (grow) {
            l *= f;
            m_used = rmax;
          }
        }
        const float off = m_used == -INFINITY ? 0.f : -m_used * scale_log2;
#ifdef TCB_ATTN_PROBE
        long long t4 = clock64();
        p_resc += t4 - t3;
#endif
        // P buffer b is free once P V of chunk gc-2 is done
        if (gc >= 2) mbar_wait(p_empty + 8 * b, (u & 1) ^ 1);
#ifdef TCB_ATTN_PROBE
        long long t5 = clock64();
        p_pempty += t5 - t4;
#endif
        const uint32_t prow = sP + b * kPBytes + half * kTileBytes + row * 128;
        // independent partial row sums, packed pairs (FFMA2 / FADD2 on sm_100)
        float2 lp[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
        const float2 sc2 = make_float2(scale_log2, scale_log2), off2 = make_float2(off, off);
#pragma unroll
        for (int cch = 0; cch < 8; ++cch) {
          uint32_t w4[4] = {0u, 0u, 0u, 0u};
          if (live[cch >> 2]) {
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const int j = cch * 8 + 2 * e;
              // masked scores are -inf: 2^-inf = 0 exactly
              const float2 x = ffma2(make_float2(__uint_as_float(sr[j]), __uint_as_float(sr[j + 1])),
                                     sc2, off2);
              const float2 pp = make_float2(ex2(x.x), ex2(x.y));
              lp[e & 1] = fadd2(lp[e & 1], pp);
              __nv_bfloat162 hv = __floats2bfloat162_rn(pp.x, pp.y);
              w4[e] = *reinterpret_cast<uint32_t*>(&hv);
            }
          }
          const uint32_t addr = prow + ((cch ^ (row & 7)) << 4);
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(w4[0]),
                       "r"(w4[1]), "r"(w4[2]), "r"(w4[3])
                       : "memory");
        }
        l += (lp[0].x + lp[0].y) + (lp[1].x + lp[1].y);
#ifdef TCB_ATTN_PROBE
        p_exp += clock64() - t5;
#endif
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(p_full + 8 * b);
        ++gc;
      }
      // hand the row sums to the epilogue warps (buffer ic & 1, free once they read item ic-2)
#ifdef TCB_ATTN_PROBE
      long long tf = clock64();
#endif
      {
        const int lb = ic & 1;
        if (ic >= 2) mbar_wait(l_empty + 8 * lb, ((ic >> 1) & 1) ^ 1);
        lbuf[(lb * 2 + half) * TQ + row] = l;
        mbuf[(lb * 2 + half) * TQ + row] = m_used;
        if (sw == 0 && lane == 0) meta[lb] = nch > 0 ? 1 : 0;
        __syncwarp();
        if (lane == 0) mbar_arrive(l_full + 8 * lb);
        ++ic;
      }
#ifdef TCB_ATTN_PROBE
      p_fin += clock64() - tf;
#endif
      if (nch > 0) ++it;
    }
#ifdef TCB_ATTN_PROBE
    if (lane == 0 && blockIdx.x == 0 && (sw == 0 || sw == 5))
      printf("tcprobe warp %d total %lld wait_q %lld wait_s %lld tmem_ld %lld max %lld rescale %lld wait_p %lld exp %lld finish %lld chunks %u\n",
             warp, clock64() - p_start, p_q, p_sfull, p_ld, p_max, p_resc, p_pempty, p_exp, p_fin, gc);
#endif
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
}

// =============================================================================================
// v3 (default): TWO CTAs per SM, thread = one query row, S consumed early.
// (r02 measurements, scripts/attn_bench.py, graph-replayed op with L2 flush, µs v1 -> v3:
// C2 44.4 -> 46.2, C3 118 -> 103, C4 143 -> 126, C5 89 -> 81.)
//
// v1 above gives each query row to two softmax warps (one per 64-key half) of ONE item per
// SM; both warps of an SM sub-partition wait for the same S and then run their exponentials
// at the same time, so the MUFU pipe idles through the max / wait / hand-over phases
// (≈3.1 K cycles per 128x128 chunk against ≈1 K of exponentials; r02a probe, ncu: XU 37%).
// Here two independent CTAs share each SM (the hardware interleaves their warps), each running
// ONE item at a time with a chain that never waits for the tensor core in steady state:
//   S = Q K^T (tcgen05, M=N=128, K=64) -> TMEM S[0,128)
//   softmax warp (one per TMEM lane quarter, thread = query row):
//     pass 1: load S_0 (keys 0-63) -> masked max; load S_1 -> masked max -> row max m
//     wait for P V of the previous chunk (usually long done), lazy rescale of O (only when a
//     row's max grew by more than 2^8), exponentials of S_1 (still in registers) -> P[32,64);
//     reload S_0 -> S is now consumed: arrive, the MMA warp issues S of the NEXT chunk (its
//     K tile is prefetched), which overlaps the rest of this chunk -> exponentials -> P[0,32)
//     P (bf16 pairs) lives in its own TMEM columns and is the A operand of O += P V
//     (tcgen05.mma [d], [a_tmem], b_desc): no shared-memory round trip for P
//   the same warps normalise O at the end of an item (no separate epilogue warps)
// K and V have separate rings (K is released by S, V only by P V), an item's last P V is
// issued as soon as its P is written (the epilogue waits for it), and the output tile is
// staged in the item's Q slot (free once its last S is done) and written by one TMA store per
// warp.  Items are handed out dynamically (an atomic counter in global memory, zeroed before
// the launch), so the 1- to 5-chunk items of a mixed-length batch balance across the 296 CTAs.
namespace v3 {
constexpr int kWarps = 6;                    // 0 producer, 1 MMA + TMEM, 2..5 softmax / epilogue
constexpr int kThreads = kWarps * 32;
constexpr int kQStages = 2, kKStages = 2, kVStages = 2;
constexpr uint32_t kTmemCols = 256;          // S [0,128), O [128,192), P [192,256)
constexpr uint32_t kOCol = 128, kPCol = 192;

#ifdef TCB_ATTN_PROBE
#define PRB(var) long long var = clock64()
#define PRB_ADD(acc, since) acc += clock64() - since
#else
#define PRB(var)
#define PRB_ADD(acc, since)
#endif

struct Info {
  int2 rows[TQ];   // [start, end) of the request of query slot q0 + r (empty for pads)
  int kbase, nch;  // first key (8-aligned), number of 128-key chunks; nch < 0: no more items
  int qb, h;       // query block, head
};
constexpr int kSmemBytes = 1024 + (kQStages + kKStages + kVStages) * kTileBytes +
                           kQStages * static_cast<int>(sizeof(Info)) + 256;

// the segment table's query-block order (tcb.h: after the records and the row index), longest
// key interval first
__device__ __forceinline__ const int32_t* qblock_order(const int4* __restrict__ segtab) {
  const int4 hd = __ldg(&segtab[0]);               // {S, num_slots, row_len, total_tokens}
  const int num_rows = hd.z > 0 ? hd.y / hd.z : 0;
  return reinterpret_cast<const int32_t*>(segtab) + 4 * (1 + hd.x) + (num_rows + 1 + 3) / 4 * 4;
}

__device__ __forceinline__ void tc_mma_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc,
                                          uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
      "r"(tmem_a), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&w)[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr),
               "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7])
               : "memory");
}

// valid-key bit mask of 32-key group [g0, g0 + 32) for a row whose keys are [jlo, jhi)
// (chunk-relative)
__device__ __forceinline__ uint32_t group_mask(int jlo, int jhi, int g0) {
  const int lo = min(max(jlo - g0, 0), 32), hi = min(max(jhi - g0, 0), 32);
  const uint32_t below_hi = hi >= 32 ? 0xffffffffu : (1u << hi) - 1u;
  const uint32_t from_lo = lo >= 32 ? 0u : ~((1u << lo) - 1u);   // no shift by 32
  return below_hi & from_lo;
}

// masked max of one 64-key half (groups 2*hh, 2*hh+1) into 8 partial maxima
__device__ __forceinline__ void half_max(const uint32_t (&sr)[64], const bool* live, const bool* inner,
                                         const uint32_t* vm, int hh, float (&mxp)[8]) {
#pragma unroll
  for (int gi = 0; gi < 2; ++gi) {
    const int g = 2 * hh + gi;
    if (!live[g]) continue;
    if (inner[g]) {
#pragma unroll
      for (int j = 32 * gi; j < 32 * gi + 32; j += 2)
        mxp[(j >> 1) & 7] = fmax3(mxp[(j >> 1) & 7], __uint_as_float(sr[j]), __uint_as_float(sr[j + 1]));
    } else {
#pragma unroll
      for (int j = 32 * gi; j < 32 * gi + 32; j += 2) {
        const float v0 = (vm[g] & (1u << (j - 32 * gi))) ? __uint_as_float(sr[j]) : -INFINITY;
        const float v1 = (vm[g] & (2u << (j - 32 * gi))) ? __uint_as_float(sr[j + 1]) : -INFINITY;
        mxp[(j >> 1) & 7] = fmax3(mxp[(j >> 1) & 7], v0, v1);
      }
    }
  }
}

// p = 2^(s * scale - m) of one 32-key group (0 outside the row's request when MASKED) -> 16
// bf16 pairs (key 2j in the low half of word j).  Straight-line code: the 32 exponentials of a
// group are independent, so their MUFU latencies overlap.
template <bool MASKED>
__device__ __forceinline__ void group_exp(const uint32_t* sr, uint32_t vm, float2 sc2, float2 off2,
                                          uint32_t (&w)[16], float2 (&lp)[2]) {
#pragma unroll
  for (int e = 0; e < 16; ++e) {
    const float2 x = ffma2(make_float2(__uint_as_float(sr[2 * e]), __uint_as_float(sr[2 * e + 1])), sc2, off2);
    float2 pp = make_float2(ex2(x.x), ex2(x.y));
    if (MASKED) {
      pp.x = (vm & (1u << (2 * e))) ? pp.x : 0.f;
      pp.y = (vm & (2u << (2 * e))) ? pp.y : 0.f;
    }
    lp[e & 1] = fadd2(lp[e & 1], pp);
    __nv_bfloat162 hv = __floats2bfloat162_rn(pp.x, pp.y);
    w[e] = *reinterpret_cast<uint32_t*>(&hv);
  }
}

// the two 32-key groups of one 64-key half -> TMEM P columns [32hh, 32hh + 32); dead groups
// (no key of the warp's rows) are written as zeros without math.  live / inner are warp-uniform.
__device__ __forceinline__ void half_exp(const uint32_t (&sr)[64], const bool* live, const bool* inner,
                                         const uint32_t* vm, int hh, float2 sc2, float2 off2,
                                         uint32_t paddr, float2 (&lp)[2]) {
#pragma unroll
  for (int gi = 0; gi < 2; ++gi) {
    const int g = 2 * hh + gi;
    uint32_t w[16];
    if (!live[g]) {
#pragma unroll
      for (int e = 0; e < 16; ++e) w[e] = 0u;
    } else if (inner[g]) {
      group_exp<false>(sr + 32 * gi, 0u, sc2, off2, w, lp);
    } else {
      group_exp<true>(sr + 32 * gi, vm[g], sc2, off2, w, lp);
    }
    const uint32_t (&w0)[8] = *reinterpret_cast<const uint32_t(*)[8]>(&w[0]);
    const uint32_t (&w1)[8] = *reinterpret_cast<const uint32_t(*)[8]>(&w[8]);
    tmem_st8(paddr + 32 * hh + 16 * gi, w0);
    tmem_st8(paddr + 32 * hh + 16 * gi + 8, w1);
  }
}

__global__ void __launch_bounds__(kThreads, 2)
attn_tc3_kernel(const __grid_constant__ CUtensorMap tmQKV, const __grid_constant__ CUtensorMap tmO,
                const int32_t* __restrict__ seg_ids,
                const int4* __restrict__ segtab, __nv_bfloat16* __restrict__ O,
                int64_t num_slots, int d_model, int num_heads, int num_items, float scale_log2,
                int* __restrict__ item_counter) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023) & ~1023u;
  const uint32_t sQ = base;                                    // [2][128 x 64]
  const uint32_t sK = sQ + kQStages * kTileBytes;              // [2][128 x 64]
  const uint32_t sV = sK + kKStages * kTileBytes;              // [2][128 x 64]
  uint8_t* gen = smem_raw + (sV + kVStages * kTileBytes - raw);
  Info* infos = reinterpret_cast<Info*>(gen);                  // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(gen + kQStages * sizeof(Info));
  const uint32_t bars = (smem_u32(tmem_slot + 2) + 7) & ~7u;
  const uint32_t q_full = bars, q_empty = q_full + 8 * kQStages;
  const uint32_t k_full = q_empty + 8 * kQStages, k_empty = k_full + 8 * kKStages;
  const uint32_t v_full = k_empty + 8 * kKStages, v_empty = v_full + 8 * kVStages;
  const uint32_t s_full = v_empty + 8 * kVStages, s_free = s_full + 8;
  const uint32_t p_full = s_free + 8, pv_done = p_full + 8;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kQStages; ++i) {
      mbar_init(q_full + 8 * i, 1);
      mbar_init(q_empty + 8 * i, 1 + 4);    // MMA (after the item's last S) + 4 softmax warps
                                            // (after their output tile left the slot)
    }
    for (int i = 0; i < kKStages; ++i) { mbar_init(k_full + 8 * i, 1); mbar_init(k_empty + 8 * i, 1); }
    for (int i = 0; i < kVStages; ++i) { mbar_init(v_full + 8 * i, 1); mbar_init(v_empty + 8 * i, 1); }
    mbar_init(s_full, 1);
    mbar_init(s_free, 4);
    mbar_init(p_full, 4);
    mbar_init(pv_done, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)), "r"(kTmemCols) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();                                 // QKV / segment ids come from earlier kernels
  pdl_trigger();

  if (warp == 0) {
    // ================= producer: next item, its metadata, Q, then its K/V chunks ==========
    if (lane == 0) asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmQKV)) : "memory");
    const int32_t* qorder = qblock_order(segtab);
    int qs = 0, ks = 0, vs = 0;
    uint32_t qph = 0, kph = 0, vph = 0;
    for (int k = 0;; ++k) {
      int item = 0;
      if (item_counter) {
        if (lane == 0) item = atomicAdd(item_counter, 1);
        item = __shfl_sync(0xffffffffu, item, 0);
      } else {
        item = blockIdx.x + k * gridDim.x;
      }
      if (lane == 0) mbar_wait(q_empty + 8 * qs, qph ^ 1);
      __syncwarp();
      Info* inf = infos + qs;
      if (item >= num_items) {
        if (lane == 0) {
          inf->nch = -1;
          mbar_arrive(q_full + 8 * qs);
        }
        break;
      }
      const int qb = __ldg(&qorder[item / num_heads]), h = item % num_heads;
      const int64_t q0 = static_cast<int64_t>(qb) * TQ;
      compute_info(reinterpret_cast<ItemInfo*>(inf), seg_ids, segtab, q0, num_slots, lane);
      const int nch = inf->nch;
      if (lane == 0) {
        inf->qb = qb;
        inf->h = h;
        if (nch == 0) {
          mbar_arrive(q_full + 8 * qs);
        } else {
          mbar_expect_tx(q_full + 8 * qs, kTileBytes);
          tma_load(sQ + qs * kTileBytes, &tmQKV, q_full + 8 * qs, h * DH, static_cast<int>(q0));
        }
        // K one chunk ahead of V (K is released by S, V only by P V)
        const int kbase = inf->kbase;
        for (int c = 0; c <= nch; ++c) {
          if (c < nch) {
            mbar_wait(k_empty + 8 * ks, kph ^ 1);
            mbar_expect_tx(k_full + 8 * ks, kTileBytes);
            tma_load(sK + ks * kTileBytes, &tmQKV, k_full + 8 * ks, d_model + h * DH, kbase + c * TK);
            if (++ks == kKStages) { ks = 0; kph ^= 1; }
          }
          if (c > 0) {
            mbar_wait(v_empty + 8 * vs, vph ^ 1);
            mbar_expect_tx(v_full + 8 * vs, kTileBytes);
            tma_load(sV + vs * kTileBytes, &tmQKV, v_full + 8 * vs, 2 * d_model + h * DH, kbase + (c - 1) * TK);
            if (++vs == kVStages) { vs = 0; vph ^= 1; }
          }
        }
      }
      __syncwarp();
      if (++qs == kQStages) { qs = 0; qph ^= 1; }
    }
  } else if (warp == 1) {
    // ================= MMA issuer ===========================================================
    // Chunk g: S(g) = Q K^T as soon as S(g-1) has been read (s_free) and K(g) is in; then
    // O += P(g-1) V(g-1) once P(g-1) is written -- S of the next chunk runs while the softmax
    // warps still work on the current one.
    int qs = 0, ks = 0, vs = 0;
    uint32_t qph = 0, kph = 0, vph = 0, g = 0;
    struct Pend {
      bool first, valid;
    } pend{false, false};
#ifdef TCB_ATTN_PROBE
    long long a_q = 0, a_kv = 0, a_sf = 0, a_p = 0, a_start = clock64();
#endif
    auto issue_pv = [&](const Pend& pp, uint32_t gp) {
      PRB(t3);
      mbar_wait(v_full + 8 * vs, vph);
      mbar_wait(p_full, gp & 1);
      PRB_ADD(a_p, t3);
      tc_fence_after();
      if (lane == 0) {
        const uint32_t va = sV + vs * kTileBytes;
#pragma unroll
        for (int k = 0; k < TK / 16; ++k)
          tc_mma_ts(tmem + kOCol, tmem + kPCol + 8 * k, desc_mnmajor(va + k * 2048), kIdescPV,
                    (!pp.first || k > 0) ? 1u : 0u);
        tc_commit(pv_done);
        tc_commit(v_empty + 8 * vs);
      }
      __syncwarp();
      if (++vs == kVStages) { vs = 0; vph ^= 1; }
    };
    for (;;) {
      PRB(t0);
      mbar_wait(q_full + 8 * qs, qph);
      PRB_ADD(a_q, t0);
      const int nch = infos[qs].nch;
      if (nch < 0) break;
      tc_fence_after();
      const uint32_t qaddr = sQ + qs * kTileBytes;
      if (nch == 0) {
        // an empty item must not hold back the pending P V: the softmax warps wait for it
        // (epilogue of the previous item) and would stop releasing Q slots -> deadlock
        if (pend.valid) {
          issue_pv(pend, g - 1);
          pend.valid = false;
        }
        if (lane == 0) mbar_arrive(q_empty + 8 * qs);
      }
      for (int c = 0; c < nch; ++c) {
        PRB(t1);
        mbar_wait(k_full + 8 * ks, kph);
        PRB_ADD(a_kv, t1);
        PRB(t2);
        if (g > 0) mbar_wait(s_free, (g - 1) & 1);
        PRB_ADD(a_sf, t2);
        tc_fence_after();
        if (lane == 0) {
          const uint32_t ka = sK + ks * kTileBytes;
#pragma unroll
          for (int k = 0; k < DH / 16; ++k)
            tc_mma(tmem, desc_kmajor(qaddr + k * 32), desc_kmajor(ka + k * 32), kIdescQK, k > 0 ? 1u : 0u);
          tc_commit(s_full);
          tc_commit(k_empty + 8 * ks);
          if (c == nch - 1) tc_commit(q_empty + 8 * qs);
        }
        __syncwarp();
        if (pend.valid) issue_pv(pend, g - 1);
        pend = Pend{c == 0, true};
        ++g;
        if (++ks == kKStages) { ks = 0; kph ^= 1; }
      }
      if (pend.valid) {                     // the item's last P V: its epilogue waits for it
        issue_pv(pend, g - 1);
        pend.valid = false;
      }
      if (++qs == kQStages) { qs = 0; qph ^= 1; }
    }
    if (pend.valid) issue_pv(pend, g - 1);
#ifdef TCB_ATTN_PROBE
    if (lane == 0 && blockIdx.x < 3)
      printf("a3probe mma cta %d total %lld wait_q %lld wait_kv %lld wait_sfree %lld wait_p %lld chunks %u\n",
             blockIdx.x, clock64() - a_start, a_q, a_kv, a_sf, a_p, g);
#endif
  } else {
    // ================= softmax + output (warps 2..5, thread = query row) ===================
    const int q = warp & 3;                 // TMEM lane quarter
    const int row = q * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(q * 32) << 16;
    const uint32_t s_addr = tmem + lane_off, o_addr = tmem + lane_off + kOCol, p_addr = tmem + lane_off + kPCol;
    int qs = 0;
    uint32_t qph = 0, g = 0;
#ifdef TCB_ATTN_PROBE
    long long b_q = 0, b_s = 0, b_p1 = 0, b_pv = 0, b_e1 = 0, b_e0 = 0, b_epi = 0, b_start = clock64();
#endif
    for (;;) {
      PRB(t0);
      mbar_wait(q_full + 8 * qs, qph);
      PRB_ADD(b_q, t0);
      const Info* inf = infos + qs;
      const int nch = inf->nch;
      if (nch < 0) break;
      const int2 rr = inf->rows[row];
      const int kbase = inf->kbase, qb = inf->qb, h = inf->h;
      const int my_qs = qs;                 // the item's Q slot stages its output tile
      if (++qs == kQStages) { qs = 0; qph ^= 1; }
      // key interval of this warp's 32 rows: union [ulo, uhi) and intersection [ilo, ihi)
      const bool real = rr.y > rr.x;
      int ulo = real ? rr.x : INT_MAX, uhi = real ? rr.y : -1;
      int ilo = real ? rr.x : INT_MAX, ihi = real ? rr.y : -1;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        ulo = min(ulo, __shfl_xor_sync(0xffffffffu, ulo, o));
        uhi = max(uhi, __shfl_xor_sync(0xffffffffu, uhi, o));
        ilo = max(ilo, __shfl_xor_sync(0xffffffffu, ilo, o));
        ihi = min(ihi, __shfl_xor_sync(0xffffffffu, ihi, o));
      }
      float m_used = -INFINITY, lsum = 0.f;
      for (int c = 0; c < nch; ++c, ++g) {
        // 32-key groups of the chunk: dead (no key of any of the warp's rows' requests: P = 0
        // without math), interior (inside every row's request: no mask) or boundary (per
        // element bit mask: key outside the row's own request -> p = 0 exactly, R11)
        const int k0 = kbase + c * TK;
        const int jlo = rr.x - k0, jhi = rr.y - k0;
        bool live[4], inner[4];
        uint32_t vm[4];
#pragma unroll
        for (int gi = 0; gi < 4; ++gi) {
          const int gk = k0 + 32 * gi;
          live[gi] = gk < uhi && gk + 32 > ulo;
          inner[gi] = gk >= ilo && gk + 32 <= ihi;
          vm[gi] = group_mask(jlo, jhi, 32 * gi);
        }
        PRB(t1);
        mbar_wait(s_full, g & 1);
        PRB_ADD(b_s, t1);
        tc_fence_after();
        PRB(t2);
        float mxp[8];
#pragma unroll
        for (int t = 0; t < 8; ++t) mxp[t] = -INFINITY;
        uint32_t sr[64];
        tmem_ld64_live(s_addr, sr, live[0], live[1]);
        half_max(sr, live, inner, vm, 0, mxp);
        tmem_ld64_live(s_addr + 64, sr, live[2], live[3]);
        half_max(sr, live, inner, vm, 1, mxp);
        const float rmax = fmaxf(fmaxf(fmaxf(mxp[0], mxp[1]), fmaxf(mxp[2], mxp[3])),
                                 fmaxf(fmaxf(mxp[4], mxp[5]), fmaxf(mxp[6], mxp[7])));
        PRB_ADD(b_p1, t2);
        // P V of the previous chunk must be done before P is overwritten (and before O is
        // rescaled); it was issued when that chunk's P was complete, so this rarely waits
        PRB(t3);
        if (g > 0) mbar_wait(pv_done, (g - 1) & 1);
        tc_fence_after();
        PRB_ADD(b_pv, t3);
        // lazy rescale: a row moves its max only when it grew by more than 2^8 (warp-collective
        // TMEM access, so the decision is per warp; lanes that keep their max scale by 1)
        bool grow = false;
        if (rmax != -INFINITY) {
          if (m_used == -INFINITY) m_used = rmax;
          else grow = (rmax - m_used) * scale_log2 > kRescaleLog2;
        }
        if (__any_sync(0xffffffffu, grow)) {
          const float f = grow ? ex2((m_used - rmax) * scale_log2) : 1.f;
#pragma unroll 1
          for (int cq = 0; cq < 2; ++cq) {
            uint32_t o[32];
            tmem_ld32_sync(o_addr + 32 * cq, o);
#pragma unroll
            for (int t = 0; t < 32; ++t) o[t] = __float_as_uint(__uint_as_float(o[t]) * f);
            tmem_st32(o_addr + 32 * cq, o);
          }
          if (grow) {
            lsum *= f;
            m_used = rmax;
          }
        }
        const float off = m_used == -INFINITY ? 0.f : -m_used * scale_log2;
        const float2 sc2 = make_float2(scale_log2, scale_log2), off2 = make_float2(off, off);
        float2 lp[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
        PRB(t4);
        half_exp(sr, live, inner, vm, 1, sc2, off2, p_addr, lp);      // keys 64-127 (in registers)
        PRB_ADD(b_e1, t4);
        PRB(t5);
        tmem_ld64_live(s_addr, sr, live[0], live[1]);                   // keys 0-63 again
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(s_free);                            // S consumed: next S may go
        half_exp(sr, live, inner, vm, 0, sc2, off2, p_addr, lp);
        lsum += (lp[0].x + lp[0].y) + (lp[1].x + lp[1].y);
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(p_full);
        PRB_ADD(b_e0, t5);
      }
      // ---- output: O / l -> bf16 -> this warp's 32 rows of the item's (now unused) Q slot,
      // 128B-swizzled, -> one TMA store (pad rows and empty items: 0; rows past M clipped) ----
      PRB(t6);
      const float inv = (nch > 0 && lsum > 0.f) ? 1.f / lsum : 0.f;
      if (nch > 0) {
        mbar_wait(pv_done, (g - 1) & 1);
        tc_fence_after();
      }
      const uint32_t stage = sQ + my_qs * kTileBytes + q * 32 * 128;
#pragma unroll 1
      for (int cq = 0; cq < 2; ++cq) {          // 32 output columns at a time
        uint32_t o[32];
        if (nch > 0) tmem_ld32_sync(o_addr + 32 * cq, o);
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          uint32_t xp[4];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const int j = 8 * t + 2 * e;
            const float a = inv == 0.f ? 0.f : __uint_as_float(o[j]) * inv;
            const float b = inv == 0.f ? 0.f : __uint_as_float(o[j + 1]) * inv;
            __nv_bfloat162 hv = __floats2bfloat162_rn(a, b);
            xp[e] = *reinterpret_cast<uint32_t*>(&hv);
          }
          const int chunk = 4 * cq + t;
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(
                           stage + lane * 128 + ((chunk ^ (lane & 7)) << 4)),
                       "r"(xp[0]), "r"(xp[1]), "r"(xp[2]), "r"(xp[3])
                       : "memory");
        }
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                         reinterpret_cast<uint64_t>(&tmO)),
                     "r"(stage), "r"(h * DH), "r"(qb * TQ + q * 32)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        mbar_arrive(q_empty + 8 * my_qs);       // the slot may take the next Q
      }
      __syncwarp();
      tc_fence_before();                        // O reads done before the next item's P V
      PRB_ADD(b_epi, t6);
    }
#ifdef TCB_ATTN_PROBE
    if (lane == 0 && blockIdx.x < 3 && warp == 2)
      printf("a3probe sm cta %d total %lld wait_q %lld wait_s %lld pass1 %lld wait_pv %lld exp1 %lld exp0 %lld epi %lld chunks %u\n",
             blockIdx.x, clock64() - b_start, b_q, b_s, b_p1, b_pv, b_e1, b_e0, b_epi, g);
#endif
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 1)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
}
}  // namespace v3

// =============================================================================================
// v3s: v3 with an item-scheduler warp, for rows of at most 128 slots (every item one chunk).
// A third control warp takes the next item from the counter and computes its metadata into a
// 2-deep ring ahead of the TMA producer (8 warps: the control warpgroup hands its registers to
// the softmax warpgroup with setmaxnreg).  With one 128 x 128 chunk per item the producer's
// metadata latency is what the softmax warps wait for: C2 (L = 128) 46.5 -> 42.3 us per launch;
// on multi-chunk items the extra look-ahead costs more than it gains (C3 101.5 -> 112), so the
// launcher uses this kernel only for row_len <= 128 (r02 A/B).
namespace v3s {
constexpr int kWarps = 8;                    // warpgroup 0: 0 TMA producer, 1 MMA + TMEM,
                                             // 2 item scheduler (metadata), 3 idle;
                                             // warpgroup 1: 4..7 softmax / epilogue
constexpr int kCtrlRegs = 56, kSoftmaxRegs = 168;   // setmaxnreg split (2 CTAs x 256 threads)
constexpr int kThreads = kWarps * 32;
constexpr int kQStages = 2, kKStages = 2, kVStages = 2, kInfoStages = 2;
constexpr uint32_t kTmemCols = 256;          // S [0,128), O [128,192), P [192,256)
constexpr uint32_t kOCol = 128, kPCol = 192;


struct Info {
  int2 rows[TQ];   // [start, end) of the request of query slot q0 + r (empty for pads)
  int kbase, nch;  // first key (8-aligned), number of 128-key chunks; nch < 0: no more items
  int qb, h;       // query block, head
};
constexpr int kSmemBytes = 1024 + (kQStages + kKStages + kVStages) * kTileBytes +
                           kInfoStages * static_cast<int>(sizeof(Info)) + 256;

// the segment table's query-block order (tcb.h: after the records and the row index), longest
// key interval first
__device__ __forceinline__ const int32_t* qblock_order(const int4* __restrict__ segtab) {
  const int4 hd = __ldg(&segtab[0]);               // {S, num_slots, row_len, total_tokens}
  const int num_rows = hd.z > 0 ? hd.y / hd.z : 0;
  return reinterpret_cast<const int32_t*>(segtab) + 4 * (1 + hd.x) + (num_rows + 1 + 3) / 4 * 4;
}

__device__ __forceinline__ void tc_mma_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc,
                                          uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
      "r"(tmem_a), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&w)[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr),
               "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7])
               : "memory");
}

// valid-key bit mask of 32-key group [g0, g0 + 32) for a row whose keys are [jlo, jhi)
// (chunk-relative)
__device__ __forceinline__ uint32_t group_mask(int jlo, int jhi, int g0) {
  const int lo = min(max(jlo - g0, 0), 32), hi = min(max(jhi - g0, 0), 32);
  const uint32_t below_hi = hi >= 32 ? 0xffffffffu : (1u << hi) - 1u;
  const uint32_t from_lo = lo >= 32 ? 0u : ~((1u << lo) - 1u);   // no shift by 32
  return below_hi & from_lo;
}

// masked max of one 64-key half (groups 2*hh, 2*hh+1) into 8 partial maxima
__device__ __forceinline__ void half_max(const uint32_t (&sr)[64], const bool* live, const bool* inner,
                                         const uint32_t* vm, int hh, float (&mxp)[8]) {
#pragma unroll
  for (int gi = 0; gi < 2; ++gi) {
    const int g = 2 * hh + gi;
    if (!live[g]) continue;
    if (inner[g]) {
#pragma unroll
      for (int j = 32 * gi; j < 32 * gi + 32; j += 2)
        mxp[(j >> 1) & 7] = fmax3(mxp[(j >> 1) & 7], __uint_as_float(sr[j]), __uint_as_float(sr[j + 1]));
    } else {
#pragma unroll
      for (int j = 32 * gi; j < 32 * gi + 32; j += 2) {
        const float v0 = (vm[g] & (1u << (j - 32 * gi))) ? __uint_as_float(sr[j]) : -INFINITY;
        const float v1 = (vm[g] & (2u << (j - 32 * gi))) ? __uint_as_float(sr[j + 1]) : -INFINITY;
        mxp[(j >> 1) & 7] = fmax3(mxp[(j >> 1) & 7], v0, v1);
      }
    }
  }
}

// p = 2^(s * scale - m) of one 32-key group (0 outside the row's request when MASKED) -> 16
// bf16 pairs (key 2j in the low half of word j).  Straight-line code: the 32 exponentials of a
// group are independent, so their MUFU latencies overlap.
template <bool MASKED>
__device__ __forceinline__ void group_exp(const uint32_t* sr, uint32_t vm, float2 sc2, float2 off2,
                                          uint32_t (&w)[16], float2 (&lp)[2]) {
#pragma unroll
  for (int e = 0; e < 16; ++e) {
    const float2 x = ffma2(make_float2(__uint_as_float(sr[2 * e]), __uint_as_float(sr[2 * e + 1])), sc2, off2);
    float2 pp = make_float2(ex2(x.x), ex2(x.y));
    if (MASKED) {
      pp.x = (vm & (1u << (2 * e))) ? pp.x : 0.f;
      pp.y = (vm & (2u << (2 * e))) ? pp.y : 0.f;
    }
    lp[e & 1] = fadd2(lp[e & 1], pp);
    __nv_bfloat162 hv = __floats2bfloat162_rn(pp.x, pp.y);
    w[e] = *reinterpret_cast<uint32_t*>(&hv);
  }
}

// the two 32-key groups of one 64-key half -> TMEM P columns [32hh, 32hh + 32); dead groups
// (no key of the warp's rows) are written as zeros without math.  live / inner are warp-uniform.
__device__ __forceinline__ void half_exp(const uint32_t (&sr)[64], const bool* live, const bool* inner,
                                         const uint32_t* vm, int hh, float2 sc2, float2 off2,
                                         uint32_t paddr, float2 (&lp)[2]) {
#pragma unroll
  for (int gi = 0; gi < 2; ++gi) {
    const int g = 2 * hh + gi;
    uint32_t w[16];
    if (!live[g]) {
#pragma unroll
      for (int e = 0; e < 16; ++e) w[e] = 0u;
    } else if (inner[g]) {
      group_exp<false>(sr + 32 * gi, 0u, sc2, off2, w, lp);
    } else {
      group_exp<true>(sr + 32 * gi, vm[g], sc2, off2, w, lp);
    }
    const uint32_t (&w0)[8] = *reinterpret_cast<const uint32_t(*)[8]>(&w[0]);
    const uint32_t (&w1)[8] = *reinterpret_cast<const uint32_t(*)[8]>(&w[8]);
    tmem_st8(paddr + 32 * hh + 16 * gi, w0);
    tmem_st8(paddr + 32 * hh + 16 * gi + 8, w1);
  }
}

__global__ void __launch_bounds__(kThreads, 2)
attn_tc3s_kernel(const __grid_constant__ CUtensorMap tmQKV, const __grid_constant__ CUtensorMap tmO,
                const int32_t* __restrict__ seg_ids,
                const int4* __restrict__ segtab, __nv_bfloat16* __restrict__ O,
                int64_t num_slots, int d_model, int num_heads, int num_items, float scale_log2,
                int* __restrict__ item_counter) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023) & ~1023u;
  const uint32_t sQ = base;                                    // [2][128 x 64]
  const uint32_t sK = sQ + kQStages * kTileBytes;              // [2][128 x 64]
  const uint32_t sV = sK + kKStages * kTileBytes;              // [2][128 x 64]
  uint8_t* gen = smem_raw + (sV + kVStages * kTileBytes - raw);
  Info* infos = reinterpret_cast<Info*>(gen);                  // [kInfoStages]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(gen + kInfoStages * sizeof(Info));
  const uint32_t bars = (smem_u32(tmem_slot + 2) + 7) & ~7u;
  const uint32_t q_full = bars, q_empty = q_full + 8 * kQStages;
  const uint32_t k_full = q_empty + 8 * kQStages, k_empty = k_full + 8 * kKStages;
  const uint32_t v_full = k_empty + 8 * kKStages, v_empty = v_full + 8 * kVStages;
  const uint32_t s_full = v_empty + 8 * kVStages, s_free = s_full + 8;
  const uint32_t p_full = s_free + 8, pv_done = p_full + 8;
  const uint32_t i_full = pv_done + 8, i_empty = i_full + 8 * kInfoStages;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kQStages; ++i) {
      mbar_init(q_full + 8 * i, 1);
      mbar_init(q_empty + 8 * i, 1 + 4);    // MMA (after the item's last S) + 4 softmax warps
                                            // (after their output tile left the slot)
    }
    for (int i = 0; i < kKStages; ++i) { mbar_init(k_full + 8 * i, 1); mbar_init(k_empty + 8 * i, 1); }
    for (int i = 0; i < kVStages; ++i) { mbar_init(v_full + 8 * i, 1); mbar_init(v_empty + 8 * i, 1); }
    mbar_init(s_full, 1);
    mbar_init(s_free, 4);
    mbar_init(p_full, 4);
    mbar_init(pv_done, 1);
    for (int i = 0; i < kInfoStages; ++i) {
      mbar_init(i_full + 8 * i, 1);
      mbar_init(i_empty + 8 * i, 1 + 1 + 4);  // TMA producer + MMA + 4 softmax warps
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)), "r"(kTmemCols) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();                                 // QKV / segment ids come from earlier kernels
  pdl_trigger();
  // registers: the control warpgroup hands most of its share to the softmax warpgroup
  if (warp < 4) {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kCtrlRegs));
  if (warp == 2) {
    // ================= item scheduler: next item -> metadata ring ==========================
    const int32_t* qorder = qblock_order(segtab);
    int is = 0;
    uint32_t iph = 0;
    for (int k = 0;; ++k) {
      int item = 0;
      if (item_counter) {
        if (lane == 0) item = atomicAdd(item_counter, 1);
        item = __shfl_sync(0xffffffffu, item, 0);
      } else {
        item = blockIdx.x + k * gridDim.x;
      }
      if (lane == 0) mbar_wait(i_empty + 8 * is, iph ^ 1);
      __syncwarp();
      Info* inf = infos + is;
      if (item >= num_items) {
        if (lane == 0) {
          inf->nch = -1;
          mbar_arrive(i_full + 8 * is);
        }
        break;
      }
      const int qb = __ldg(&qorder[item / num_heads]);
      compute_info(reinterpret_cast<ItemInfo*>(inf), seg_ids, segtab, static_cast<int64_t>(qb) * TQ,
                   num_slots, lane);
      if (lane == 0) {
        inf->qb = qb;
        inf->h = item % num_heads;
        mbar_arrive(i_full + 8 * is);
      }
      __syncwarp();
      if (++is == kInfoStages) { is = 0; iph ^= 1; }
    }
  } else if (warp == 0) {
    // ================= TMA producer: per item its Q tile, then K one chunk ahead of V =========
    if (lane == 0) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmQKV)) : "memory");
      int qs = 0, ks = 0, vs = 0, is = 0;
      uint32_t qph = 0, kph = 0, vph = 0, iph = 0;
      for (;;) {
        mbar_wait(i_full + 8 * is, iph);
        const Info* inf = infos + is;
        const int nch = inf->nch, kbase = inf->kbase, qb = inf->qb, h = inf->h;
        mbar_arrive(i_empty + 8 * is);
        if (++is == kInfoStages) { is = 0; iph ^= 1; }
        if (nch < 0) break;
        mbar_wait(q_empty + 8 * qs, qph ^ 1);  // the slot is ours (also for an empty item:
                                               // the softmax warps stage its output there)
        if (nch == 0) {
          mbar_arrive(q_full + 8 * qs);
        } else {
          mbar_expect_tx(q_full + 8 * qs, kTileBytes);
          tma_load(sQ + qs * kTileBytes, &tmQKV, q_full + 8 * qs, h * DH, qb * TQ);
        }
        // K one chunk ahead of V (K is released by S, V only by P V)
        for (int c = 0; c <= nch; ++c) {
          if (c < nch) {
            mbar_wait(k_empty + 8 * ks, kph ^ 1);
            mbar_expect_tx(k_full + 8 * ks, kTileBytes);
            tma_load(sK + ks * kTileBytes, &tmQKV, k_full + 8 * ks, d_model + h * DH, kbase + c * TK);
            if (++ks == kKStages) { ks = 0; kph ^= 1; }
          }
          if (c > 0) {
            mbar_wait(v_empty + 8 * vs, vph ^ 1);
            mbar_expect_tx(v_full + 8 * vs, kTileBytes);
            tma_load(sV + vs * kTileBytes, &tmQKV, v_full + 8 * vs, 2 * d_model + h * DH, kbase + (c - 1) * TK);
            if (++vs == kVStages) { vs = 0; vph ^= 1; }
          }
        }
        if (++qs == kQStages) { qs = 0; qph ^= 1; }
      }
    }
  } else if (warp == 1) {
    // ================= MMA issuer ===========================================================
    // Chunk g: S(g) = Q K^T as soon as S(g-1) has been read (s_free) and K(g) is in; then
    // O += P(g-1) V(g-1) once P(g-1) is written -- S of the next chunk runs while the softmax
    // warps still work on the current one.
    int qs = 0, ks = 0, vs = 0;
    uint32_t qph = 0, kph = 0, vph = 0, g = 0;
    struct Pend {
      bool first, valid;
    } pend{false, false};
#ifdef TCB_ATTN_PROBE
    long long a_q = 0, a_kv = 0, a_sf = 0, a_p = 0, a_start = clock64();
#endif
    auto issue_pv = [&](const Pend& pp, uint32_t gp) {
      PRB(t3);
      mbar_wait(v_full + 8 * vs, vph);
      mbar_wait(p_full, gp & 1);
      PRB_ADD(a_p, t3);
      tc_fence_after();
      if (lane == 0) {
        const uint32_t va = sV + vs * kTileBytes;
#pragma unroll
        for (int k = 0; k < TK / 16; ++k)
          tc_mma_ts(tmem + kOCol, tmem + kPCol + 8 * k, desc_mnmajor(va + k * 2048), kIdescPV,
                    (!pp.first || k > 0) ? 1u : 0u);
        tc_commit(pv_done);
        tc_commit(v_empty + 8 * vs);
      }
      __syncwarp();
      if (++vs == kVStages) { vs = 0; vph ^= 1; }
    };
    int is = 0;
    uint32_t iph = 0;
    for (;;) {
      PRB(t0);
      mbar_wait(i_full + 8 * is, iph);
      const int nch = infos[is].nch;
      __syncwarp();
      if (lane == 0) mbar_arrive(i_empty + 8 * is);
      if (++is == kInfoStages) { is = 0; iph ^= 1; }
      if (nch < 0) break;
      mbar_wait(q_full + 8 * qs, qph);
      PRB_ADD(a_q, t0);
      tc_fence_after();
      const uint32_t qaddr = sQ + qs * kTileBytes;
      if (nch == 0) {
        // an empty item must not hold back the pending P V: the softmax warps wait for it
        // (epilogue of the previous item) and would stop releasing Q slots -> deadlock
        if (pend.valid) {
          issue_pv(pend, g - 1);
          pend.valid = false;
        }
        if (lane == 0) mbar_arrive(q_empty + 8 * qs);
      }
      for (int c = 0; c < nch; ++c) {
        PRB(t1);
        mbar_wait(k_full + 8 * ks, kph);
        PRB_ADD(a_kv, t1);
        PRB(t2);
        if (g > 0) mbar_wait(s_free, (g - 1) & 1);
        PRB_ADD(a_sf, t2);
        tc_fence_after();
        if (lane == 0) {
          const uint32_t ka = sK + ks * kTileBytes;
#pragma unroll
          for (int k = 0; k < DH / 16; ++k)
            tc_mma(tmem, desc_kmajor(qaddr + k * 32), desc_kmajor(ka + k * 32), kIdescQK, k > 0 ? 1u : 0u);
          tc_commit(s_full);
          tc_commit(k_empty + 8 * ks);
          if (c == nch - 1) tc_commit(q_empty + 8 * qs);
        }
        __syncwarp();
        if (pend.valid) issue_pv(pend, g - 1);
        pend = Pend{c == 0, true};
        ++g;
        if (++ks == kKStages) { ks = 0; kph ^= 1; }
      }
      if (pend.valid) {                     // the item's last P V: its epilogue waits for it
        issue_pv(pend, g - 1);
        pend.valid = false;
      }
      if (++qs == kQStages) { qs = 0; qph ^= 1; }
    }
    if (pend.valid) issue_pv(pend, g - 1);
#ifdef TCB_ATTN_PROBE
    if (lane == 0 && blockIdx.x < 3)
      printf("a3probe mma cta %d total %lld wait_q %lld wait_kv %lld wait_sfree %lld wait_p %lld chunks %u\n",
             blockIdx.x, clock64() - a_start, a_q, a_kv, a_sf, a_p, g);
#endif
  }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(kSoftmaxRegs));
    // ================= softmax + output (warps 4..7, thread = query row) ===================
    const int q = warp & 3;                 // TMEM lane quarter
    const int row = q * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(q * 32) << 16;
    const uint32_t s_addr = tmem + lane_off, o_addr = tmem + lane_off + kOCol, p_addr = tmem + lane_off + kPCol;
    int qs = 0, is = 0;
    uint32_t iph = 0, g = 0;
#ifdef TCB_ATTN_PROBE
    long long b_q = 0, b_s = 0, b_p1 = 0, b_pv = 0, b_e1 = 0, b_e0 = 0, b_epi = 0, b_start = clock64();
#endif
    for (;;) {
      PRB(t0);
      mbar_wait(i_full + 8 * is, iph);
      PRB_ADD(b_q, t0);
      const Info* inf = infos + is;
      const int nch = inf->nch;
      const int2 rr = inf->rows[row];
      const int kbase = inf->kbase, qb = inf->qb, h = inf->h;
      __syncwarp();
      if (lane == 0) mbar_arrive(i_empty + 8 * is);   // metadata copied to registers
      if (++is == kInfoStages) { is = 0; iph ^= 1; }
      if (nch < 0) break;
      // the item's Q slot (acquired by the producer, read by the item's S MMAs) stages the
      // output tile; no wait needed: the epilogue runs after the item's last P V
      const int my_qs = qs;
      if (++qs == kQStages) { qs = 0; }
      // key interval of this warp's 32 rows: union [ulo, uhi) and intersection [ilo, ihi)
      const bool real = rr.y > rr.x;
      int ulo = real ? rr.x : INT_MAX, uhi = real ? rr.y : -1;
      int ilo = real ? rr.x : INT_MAX, ihi = real ? rr.y : -1;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        ulo = min(ulo, __shfl_xor_sync(0xffffffffu, ulo, o));
        uhi = max(uhi, __shfl_xor_sync(0xffffffffu, uhi, o));
        ilo = max(ilo, __shfl_xor_sync(0xffffffffu, ilo, o));
        ihi = min(ihi, __shfl_xor_sync(0xffffffffu, ihi, o));
      }
      float m_used = -INFINITY, lsum = 0.f;
      for (int c = 0; c < nch; ++c, ++g) {
        // 32-key groups of the chunk: dead (no key of any of the warp's rows' requests: P = 0
        // without math), interior (inside every row's request: no mask) or boundary (per
        // element bit mask: key outside the row's own request -> p = 0 exactly, R11)
        const int k0 = kbase + c * TK;
        const int jlo = rr.x - k0, jhi = rr.y - k0;
        bool live[4], inner[4];
        uint32_t vm[4];
#pragma unroll
        for (int gi = 0; gi < 4; ++gi) {
          const int gk = k0 + 32 * gi;
          live[gi] = gk < uhi && gk + 32 > ulo;
          inner[gi] = gk >= ilo && gk + 32 <= ihi;
          vm[gi] = group_mask(jlo, jhi, 32 * gi);
        }
        PRB(t1);
        mbar_wait(s_full, g & 1);
        PRB_ADD(b_s, t1);
        tc_fence_after();
        PRB(t2);
        float mxp[8];
#pragma unroll
        for (int t = 0; t < 8; ++t) mxp[t] = -INFINITY;
        uint32_t sr[64];
        tmem_ld64_live(s_addr, sr, live[0], live[1]);
        half_max(sr, live, inner, vm, 0, mxp);
        tmem_ld64_live(s_addr + 64, sr, live[2], live[3]);
        half_max(sr, live, inner, vm, 1, mxp);
        const float rmax = fmaxf(fmaxf(fmaxf(mxp[0], mxp[1]), fmaxf(mxp[2], mxp[3])),
                                 fmaxf(fmaxf(mxp[4], mxp[5]), fmaxf(mxp[6], mxp[7])));
        PRB_ADD(b_p1, t2);
        // P V of the previous chunk must be done before P is overwritten (and before O is
        // rescaled); it was issued when that chunk's P was complete, so this rarely waits
        PRB(t3);
        if (g > 0) mbar_wait(pv_done, (g - 1) & 1);
        tc_fence_after();
        PRB_ADD(b_pv, t3);
        // lazy rescale: a row moves its max only when it grew by more than 2^8 (warp-collective
        // TMEM access, so the decision is per warp; lanes that keep their max scale by 1)
        bool grow = false;
        if (rmax != -INFINITY) {
          if (m_used == -INFINITY) m_used = rmax;
          else grow = (rmax - m_used) * scale_log2 > kRescaleLog2;
        }
        if (__any_sync(0xffffffffu, grow)) {
          const float f = grow ? ex2((m_used - rmax) * scale_log2) : 1.f;
#pragma unroll 1
          for (int cq = 0; cq < 2; ++cq) {
            uint32_t o[32];
            tmem_ld32_sync(o_addr + 32 * cq, o);
#pragma unroll
            for (int t = 0; t < 32; ++t) o[t] = __float_as_uint(__uint_as_float(o[t]) * f);
            tmem_st32(o_addr + 32 * cq, o);
          }
          if (grow) {
            lsum *= f;
            m_used = rmax;
          }
        }
        const float off = m_used == -INFINITY ? 0.f : -m_used * scale_log2;
        const float2 sc2 = make_float2(scale_log2, scale_log2), off2 = make_float2(off, off);
        float2 lp[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
        PRB(t4);
        half_exp(sr, live, inner, vm, 1, sc2, off2, p_addr, lp);      // keys 64-127 (in registers)
        PRB_ADD(b_e1, t4);
        PRB(t5);
        tmem_ld64_live(s_addr, sr, live[0], live[1]);                   // keys 0-63 again
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(s_free);                            // S consumed: next S may go
        half_exp(sr, live, inner, vm, 0, sc2, off2, p_addr, lp);
        lsum += (lp[0].x + lp[0].y) + (lp[1].x + lp[1].y);
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(p_full);
        PRB_ADD(b_e0, t5);
      }
      // ---- output: O / l -> bf16 -> this warp's 32 rows of the item's (now unused) Q slot,
      // 128B-swizzled, -> one TMA store (pad rows and empty items: 0; rows past M clipped) ----
      PRB(t6);
      const float inv = (nch > 0 && lsum > 0.f) ? 1.f / lsum : 0.f;
      if (nch > 0) {
        mbar_wait(pv_done, (g - 1) & 1);
        tc_fence_after();
      }
      const uint32_t stage = sQ + my_qs * kTileBytes + q * 32 * 128;
#pragma unroll 1
      for (int cq = 0; cq < 2; ++cq) {          // 32 output columns at a time
        uint32_t o[32];
        if (nch > 0) tmem_ld32_sync(o_addr + 32 * cq, o);
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          uint32_t xp[4];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const int j = 8 * t + 2 * e;
            const float a = inv == 0.f ? 0.f : __uint_as_float(o[j]) * inv;
            const float b = inv == 0.f ? 0.f : __uint_as_float(o[j + 1]) * inv;
            __nv_bfloat162 hv = __floats2bfloat162_rn(a, b);
            xp[e] = *reinterpret_cast<uint32_t*>(&hv);
          }
          const int chunk = 4 * cq + t;
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(
                           stage + lane * 128 + ((chunk ^ (lane & 7)) << 4)),
                       "r"(xp[0]), "r"(xp[1]), "r"(xp[2]), "r"(xp[3])
                       : "memory");
        }
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                         reinterpret_cast<uint64_t>(&tmO)),
                     "r"(stage), "r"(h * DH), "r"(qb * TQ + q * 32)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        mbar_arrive(q_empty + 8 * my_qs);       // the slot may take the next Q
      }
      __syncwarp();
      tc_fence_before();                        // O reads done before the next item's P V
      PRB_ADD(b_epi, t6);
    }
#ifdef TCB_ATTN_PROBE
    if (lane == 0 && blockIdx.x < 3 && warp == 4)
      printf("a3probe sm cta %d total %lld wait_q %lld wait_s %lld pass1 %lld wait_pv %lld exp1 %lld exp0 %lld epi %lld chunks %u\n",
             blockIdx.x, clock64() - b_start, b_q, b_s, b_p1, b_pv, b_e1, b_e0, b_epi, g);
#endif
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 1)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
}
}  // namespace v3s


}  // namespace

cudaError_t launch_attention_bf16_tc(int64_t num_slots, int d_model, int num_heads,
                                     const void* qkv, const int32_t* seg_ids,
                                     const int4* segtab, void* O, int* item_counter,
                                     int row_len, cudaStream_t s) {
  if (num_slots == 0) return cudaSuccess;
  static const bool use_v1 = [] {              // TCB_ATTN=v1: the previous kernel (A/B only)
    const char* v = std::getenv("TCB_ATTN");
    return v && std::string(v) == "v1";
  }();
  static bool attr = false;
  static int sms = 0;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(attn_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         kSmemBytes);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(v3::attn_tc3_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               v3::kSmemBytes);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(v3s::attn_tc3s_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               v3s::kSmemBytes);

    if (e != cudaSuccess) return e;
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    attr = true;
  }
  CUtensorMap map;
  if (!make_tmap_bf16(&map, qkv, static_cast<uint64_t>(num_slots), 3ull * d_model, 128, 64, 128))
    return cudaErrorInvalidValue;
  const int64_t qblocks = (num_slots + TQ - 1) / TQ;
  const int items = static_cast<int>(qblocks * num_heads);
  const float scale_log2 = 1.4426950408889634f / sqrtf(static_cast<float>(DH));
  if (use_v1) {
    const unsigned grid = static_cast<unsigned>(items < sms ? items : sms);
    return launch_ex(attn_tc_kernel, dim3(grid), dim3(kThreads), kSmemBytes, s, 1, map, seg_ids,
                     segtab, static_cast<__nv_bfloat16*>(O), num_slots, d_model, num_heads, items,
                     scale_log2);
  }
  static const bool static_order = std::getenv("TCB_ATTN_STATIC") != nullptr;   // A/B only
  if (static_order) item_counter = nullptr;
  const int ctas = 2 * sms;                   // two CTAs per SM
  const unsigned grid = static_cast<unsigned>(items < ctas ? items : ctas);
  CUtensorMap omap;
  if (!make_tmap_bf16(&omap, O, static_cast<uint64_t>(num_slots), static_cast<uint64_t>(d_model), 32, 64, 128))
    return cudaErrorInvalidValue;
  static const int sched_env = [] {             // TCB_ATTN_SCHED=0/1 forces either (A/B)
    const char* v = std::getenv("TCB_ATTN_SCHED");
    return v ? std::atoi(v) : -1;
  }();
  const bool sched = sched_env >= 0 ? sched_env == 1 : (row_len > 0 && row_len <= TK);
  if (sched)
    return launch_ex(v3s::attn_tc3s_kernel, dim3(grid), dim3(v3s::kThreads), v3s::kSmemBytes, s, 1,
                     map, omap, seg_ids, segtab, static_cast<__nv_bfloat16*>(O), num_slots,
                     d_model, num_heads, items, scale_log2, item_counter);
  return launch_ex(v3::attn_tc3_kernel, dim3(grid), dim3(v3::kThreads), v3::kSmemBytes, s, 1, map,
                   omap, seg_ids, segtab, static_cast<__nv_bfloat16*>(O), num_slots, d_model,
                   num_heads, items, scale_log2, item_counter);
}

}  // namespace k
}  // namespace tcb
