// attention.cu -- segment-masked self-attention over packed rows (sm_100a).
//
// Eq. (5)-(6): Att_CB(Q,K,V) = softmax(QK^T/sqrt(d) + M) V with M = 0 on the
// diagonal blocks Q_i K_i^T and -inf elsewhere.  Only the diagonal blocks are useful
// (Eq. (7)), and the paper notes that computing the masked blocks
// anyway wastes memory and compute (§4.2).  This kernel therefore never
// materialises M or the score matrix: a CTA owns 128 query slots (all heads, one after the
// other); each of its 8 warps owns 16 query rows and evaluates only the 16-key sub-blocks
// that intersect the key interval of its own rows' requests, so cross-request tiles are
// skipped outright.  Inside a
// visited sub-block, pairs from different requests get exactly -inf before the softmax
// (R11), i.e. probability 0.  Softmax is the online (running max / running sum) form in the
// exp2 domain (R23), fp32 throughout; P is rounded to bf16 only as the A operand of P.V.
//
// The contraction is tiny per sub-block (16x16x64 and 16x64x16) and the kernel is HBM /
// MUFU bound for the paper's request lengths, so it uses warp-level
// mma.sync.m16n8k16 (bf16 in, fp32 accumulate) with Q/K/V staged in swizzled shared memory
// by a 3-stage cp.async ring over (head, 64-key chunk) items; one online-softmax update per
// chunk.  The fp32 variant below is the 1e-4 parity path.
#include <cuda_bf16.h>

#include <cmath>
#include <cstdio>

#include "kernels.h"

namespace tcb {
namespace k {
namespace {

constexpr int KC = 64;      // keys per staged chunk
constexpr int DH = 64;      // head dim of the bf16 path

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// [rows][64] bf16 tile, 16-byte chunk c of row r stored at chunk (c ^ (r & 7)).
__device__ __forceinline__ int swz(int row, int chunk) { return row * 64 + ((chunk ^ (row & 7)) << 3); }

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2,
                                        uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& r0, uint32_t& r1,
                                          uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void mma_bf16(float (&c)[4], const uint32_t (&a)[4], uint32_t b0,
                                         uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, "
      "{%8,%9}, {%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
// 2^x on the SFU (MUFU.EX2); flushes results below 2^-126 to 0, which only affects
// probabilities that are negligible against the row maximum's 1.
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ uint32_t pack_bf16(float lo, float hi) {
  __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&h);
}

// ---- warp-specialised persistent kernel ------------------------------------------------
// Work item = (block of AQ = 16*ACW query slots, head).  Each CTA (one per SM) walks items
// blockIdx.x, blockIdx.x + gridDim.x, ...  Warp ACW is the producer: one lane computes the
// block's key interval [clo, chi) (from the segment table) and TMA-loads the Q tile and the
// K/V 64-key chunks of that interval into mbarrier-guarded rings (128B swizzle, the layout
// swz() addresses).  Warps 0..ACW-1 are consumers: each owns 16 query rows, waits on the
// ring's full barriers, evaluates only the 16-key sub-blocks inside its own rows' request
// interval, and releases the slot -- no CTA-wide barrier anywhere in the loop.  The producer
// is two warps: A computes item metadata and loads Q tiles (runs up to kQStages items
// ahead), B streams the K/V chunks.
constexpr int ACW = 8;                       // consumer warps
constexpr int AQ = 16 * ACW;                 // query slots per item
constexpr int kKVStages = 6, kQStages = 4;
constexpr int kQTileBytes = AQ * DH * 2;     // 16 KB
constexpr int kKVTileBytes = KC * DH * 2;    // 8 KB (K or V)
constexpr int kAttnSmem = 1024 + kQStages * kQTileBytes + 2 * kKVStages * kKVTileBytes + 512 +
                          kQStages * (AQ * 8 + ACW * 16 + 16);

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
// try_wait with a suspend-time hint: a waiting warp is parked by the hardware until the
// phase completes (or ~10 us pass) instead of spinning and stealing issue slots from the
// consumer warps that share its scheduler.
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity), "r"(10000)
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

// Per-item metadata the producer computes once (in smem, one slot per Q stage):
//   rows[r] = [start, end) of the request of query slot q0+r (empty for pad slots);
//   warps[w] = {union lo, union hi, intersection lo, intersection hi} of the 16 rows of
//              consumer warp w (keys outside the union are skipped; sub-blocks inside the
//              intersection need no mask);  blk = key interval of the whole block.
struct ItemInfo {
  int2 rows[AQ];
  int4 warps[ACW];
  int2 blk;
};

__device__ void compute_item_info(ItemInfo* inf, const int32_t* __restrict__ seg_ids,
                                  const int4* __restrict__ segtab, int64_t q0,
                                  int64_t num_slots, int lane) {
  // lane handles rows lane, lane+32, lane+64, lane+96 -> warp (r / 16)
  int2 r4[AQ / 32];
#pragma unroll
  for (int i = 0; i < AQ / 32; ++i) {
    const int64_t row = q0 + lane + 32 * i;
    const int sg = row < num_slots ? __ldg(&seg_ids[row]) : -1;
    int2 v = make_int2(0, 0);
    if (sg >= 0) {
      const int4 rec = __ldg(&segtab[1 + sg]);
      v = make_int2(rec.x, rec.x + rec.y);
    }
    r4[i] = v;
    inf->rows[lane + 32 * i] = v;
  }
  int blo = INT_MAX, bhi = -1;
#pragma unroll
  for (int i = 0; i < AQ / 32; ++i) {
    // rows lane+32i belong to warp 2i (lanes 0-15) or 2i+1 (lanes 16-31)
    const bool real = r4[i].y > r4[i].x;
    int ulo = real ? r4[i].x : INT_MAX, uhi = real ? r4[i].y : -1;
    int ilo = real ? r4[i].x : INT_MIN, ihi = real ? r4[i].y : INT_MAX;
    bool any_pad = !real;
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) {   // reduce within each half-warp (16 rows)
      ulo = min(ulo, __shfl_xor_sync(0xffffffffu, ulo, o));
      uhi = max(uhi, __shfl_xor_sync(0xffffffffu, uhi, o));
      ilo = max(ilo, __shfl_xor_sync(0xffffffffu, ilo, o));
      ihi = min(ihi, __shfl_xor_sync(0xffffffffu, ihi, o));
      any_pad |= __shfl_xor_sync(0xffffffffu, any_pad ? 1 : 0, o) != 0;
    }
    if (any_pad) { ilo = 0; ihi = 0; }          // a pad row needs the mask everywhere
    if ((lane & 15) == 0) inf->warps[2 * i + (lane >> 4)] = make_int4(ulo, uhi, ilo, ihi);
    if (uhi >= 0) { blo = min(blo, ulo); bhi = max(bhi, uhi); }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    blo = min(blo, __shfl_xor_sync(0xffffffffu, blo, o));
    bhi = max(bhi, __shfl_xor_sync(0xffffffffu, bhi, o));
  }
  if (lane == 0) inf->blk = bhi < 0 ? make_int2(-1, -1) : make_int2(blo & ~7, bhi);
  __syncwarp();
}

__global__ void __launch_bounds__((ACW + 2) * 32, 1)
attn_bf16_kernel(const __grid_constant__ CUtensorMap tmQKV, const int32_t* __restrict__ seg_ids,
                 const int4* __restrict__ segtab, __nv_bfloat16* __restrict__ O,
                 int64_t num_slots, int d_model, int num_heads, int num_items, float scale_log2) {
  extern __shared__ uint8_t attn_smem_raw[];
  const uint32_t raw = smem_u32(attn_smem_raw);
  const uint32_t base = (raw + 1023) & ~1023u;
  const uint32_t sQ = base;                                        // [2][AQ x 64] bf16
  const uint32_t sK = sQ + kQStages * kQTileBytes;                 // [6][64 x 64]
  const uint32_t sV = sK + kKVStages * kKVTileBytes;               // [6][64 x 64]
  const uint32_t bars = sV + kKVStages * kKVTileBytes;
  const uint32_t kv_full = bars, kv_empty = bars + 8 * kKVStages;
  const uint32_t q_full = bars + 16 * kKVStages, q_empty = q_full + 8 * kQStages;
  const uint32_t info_full = q_empty + 8 * kQStages;
  ItemInfo* infos = reinterpret_cast<ItemInfo*>(attn_smem_raw + (info_full + 8 * kQStages + 15 - raw) / 16 * 16);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kKVStages; ++i) { mbar_init(kv_full + 8 * i, 1); mbar_init(kv_empty + 8 * i, ACW); }
    for (int i = 0; i < kQStages; ++i) {
      mbar_init(q_full + 8 * i, 1);
      mbar_init(q_empty + 8 * i, ACW + 1);      // consumers + producer B
      mbar_init(info_full + 8 * i, 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == ACW) {
    // ====================== producer A: item metadata + Q tiles ========================
    if (lane == 0) asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmQKV)) : "memory");
    int q_stage = 0;
    uint32_t q_phase = 0;
    for (int item = blockIdx.x; item < num_items; item += gridDim.x) {
      const int qb = item / num_heads, h = item % num_heads;
      const int64_t q0 = static_cast<int64_t>(qb) * AQ;
      if (lane == 0) mbar_wait(q_empty + 8 * q_stage, q_phase ^ 1);
      __syncwarp();
      ItemInfo* inf = infos + q_stage;
      compute_item_info(inf, seg_ids, segtab, q0, num_slots, lane);
      if (lane == 0) {
        mbar_arrive(info_full + 8 * q_stage);                // metadata ready for producer B
        if (inf->blk.y < 0) {
          mbar_arrive(q_full + 8 * q_stage);                 // nothing to load
        } else {
          mbar_expect_tx(q_full + 8 * q_stage, kQTileBytes);
          const uint32_t dq = sQ + q_stage * kQTileBytes;
          tma_load(dq, &tmQKV, q_full + 8 * q_stage, h * DH, static_cast<int>(q0));
          tma_load(dq + kQTileBytes / 2, &tmQKV, q_full + 8 * q_stage, h * DH,
                   static_cast<int>(q0) + AQ / 2);
        }
      }
      if (++q_stage == kQStages) { q_stage = 0; q_phase ^= 1; }
    }
    return;
  }
  if (warp == ACW + 1) {
    // ====================== producer B: K/V chunks of each item ========================
    if (lane == 0) {
      int kv_stage = 0, q_stage = 0;
      uint32_t kv_phase = 0, q_phase = 0;
      for (int item = blockIdx.x; item < num_items; item += gridDim.x) {
        const int h = item % num_heads;
        mbar_wait(info_full + 8 * q_stage, q_phase);
        const int2 iv = infos[q_stage].blk;
        mbar_arrive(q_empty + 8 * q_stage);                  // done with this info slot
        if (++q_stage == kQStages) { q_stage = 0; q_phase ^= 1; }
        if (iv.y < 0) continue;
        const int nch = (iv.y - iv.x + KC - 1) / KC;
        for (int c = 0; c < nch; ++c) {
          mbar_wait(kv_empty + 8 * kv_stage, kv_phase ^ 1);
          mbar_expect_tx(kv_full + 8 * kv_stage, 2 * kKVTileBytes);
          const int kbase = iv.x + c * KC;
          tma_load(sK + kv_stage * kKVTileBytes, &tmQKV, kv_full + 8 * kv_stage,
                   d_model + h * DH, kbase);
          tma_load(sV + kv_stage * kKVTileBytes, &tmQKV, kv_full + 8 * kv_stage,
                   2 * d_model + h * DH, kbase);
          if (++kv_stage == kKVStages) { kv_stage = 0; kv_phase ^= 1; }
        }
      }
    }
    return;
  }

  // ================================== consumers ==========================================
  const int g = lane >> 2, t4 = lane & 3;
  // byte offsets of this lane's ldmatrix rows inside a swizzled [rows][128 B] tile: the
  // XOR term only depends on (lane & 7), so they are loop invariants
  uint32_t kofs[4], vofs[4], qofs[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int mi = lane >> 3;
    kofs[i] = 2 * swz((mi >> 1) * 8 + (lane & 7), 2 * i + (mi & 1));
    vofs[i] = 2 * swz((mi & 1) * 8 + (lane & 7), 2 * i + (mi >> 1));
    qofs[i] = 2 * swz(warp * 16 + (lane & 15), 2 * i + (lane >> 4));
  }
  int kv_stage = 0, q_stage = 0;
  uint32_t kv_phase = 0, q_phase = 0;
#ifdef TCB_ATTN_PROBE
  long long p_start = clock64(), p_q = 0, p_kv = 0;
  int p_items = 0, p_chunks = 0;
#endif
  for (int item = blockIdx.x; item < num_items; item += gridDim.x) {
    const int qb = item / num_heads, h = item % num_heads;
    const int64_t rowA = static_cast<int64_t>(qb) * AQ + warp * 16 + g, rowB = rowA + 8;
#ifdef TCB_ATTN_PROBE
    long long pq0 = clock64();
#endif
    mbar_wait(q_full + 8 * q_stage, q_phase);
#ifdef TCB_ATTN_PROBE
    p_q += clock64() - pq0;
    ++p_items;
#endif
    const ItemInfo* inf = infos + q_stage;
    const int2 iv = inf->blk;
    const int4 wv = inf->warps[warp];              // union lo/hi, intersection lo/hi
    const int2 ra = inf->rows[warp * 16 + g], rb = inf->rows[warp * 16 + g + 8];
    uint32_t qf[4][4];
    if (iv.y >= 0) {
      const uint32_t q = sQ + q_stage * kQTileBytes;
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) ldsm_x4(q + qofs[ks], qf[ks][0], qf[ks][1], qf[ks][2], qf[ks][3]);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(q_empty + 8 * q_stage);
    if (++q_stage == kQStages) { q_stage = 0; q_phase ^= 1; }

    float acc[8][4];
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
    float mA = -INFINITY, mB = -INFINITY, lA = 0.f, lB = 0.f;   // raw-score running maxima
    const int nch = iv.y < 0 ? 0 : (iv.y - iv.x + KC - 1) / KC;
    for (int c = 0; c < nch; ++c) {
      const int kbase = iv.x + c * KC;
      const int lim = min(wv.y, iv.y);
      const int sb_lo = wv.x > kbase ? (wv.x - kbase) >> 4 : 0;
      const int sb_hi = lim > kbase ? min(KC / 16, (lim - kbase + 15) >> 4) : 0;
      // always observe the slot's fill before releasing it (keeps the ring's phases exact
      // even when this warp skips the whole chunk)
#ifdef TCB_ATTN_PROBE
      long long pk0 = clock64();
#endif
      mbar_wait(kv_full + 8 * kv_stage, kv_phase);
#ifdef TCB_ATTN_PROBE
      p_kv += clock64() - pk0;
      ++p_chunks;
#endif
      if (wv.y >= 0 && sb_lo < sb_hi) {
        const uint32_t kt = sK + kv_stage * kKVTileBytes, vt = sV + kv_stage * kKVTileBytes;
        float s[KC / 16][2][4];
        float bmA = -INFINITY, bmB = -INFINITY;
#pragma unroll
        for (int sb = 0; sb < KC / 16; ++sb) {
          if (sb < sb_lo || sb >= sb_hi) continue;   // cross-request sub-block: skipped
#pragma unroll
          for (int j = 0; j < 2; ++j) s[sb][j][0] = s[sb][j][1] = s[sb][j][2] = s[sb][j][3] = 0.f;
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            uint32_t k0, k1, k2, k3;
            ldsm_x4(kt + sb * 2048 + kofs[ks], k0, k1, k2, k3);
            mma_bf16(s[sb][0], qf[ks], k0, k1);
            mma_bf16(s[sb][1], qf[ks], k2, k3);
          }
          // mask M of Eq. (6): key outside the row's own request -> -inf.  Sub-blocks inside
          // every row's request (the intersection) need no test.
          const int kb = kbase + sb * 16;
          if (!(kb >= wv.z && kb + 16 <= wv.w)) {
#pragma unroll
            for (int j = 0; j < 2; ++j) {
              const int k0 = kb + j * 8 + 2 * t4;
              if (!(k0 >= ra.x && k0 < ra.y)) s[sb][j][0] = -INFINITY;
              if (!(k0 + 1 >= ra.x && k0 + 1 < ra.y)) s[sb][j][1] = -INFINITY;
              if (!(k0 >= rb.x && k0 < rb.y)) s[sb][j][2] = -INFINITY;
              if (!(k0 + 1 >= rb.x && k0 + 1 < rb.y)) s[sb][j][3] = -INFINITY;
            }
          }
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            bmA = fmaxf(bmA, fmaxf(s[sb][j][0], s[sb][j][1]));
            bmB = fmaxf(bmB, fmaxf(s[sb][j][2], s[sb][j][3]));
          }
        }
        bmA = fmaxf(bmA, __shfl_xor_sync(0xffffffffu, bmA, 1));
        bmA = fmaxf(bmA, __shfl_xor_sync(0xffffffffu, bmA, 2));
        bmB = fmaxf(bmB, __shfl_xor_sync(0xffffffffu, bmB, 1));
        bmB = fmaxf(bmB, __shfl_xor_sync(0xffffffffu, bmB, 2));
        // rescale only when a running max moved AND something was accumulated under the old
        // one (the first live chunk of a row just sets its max)
        // (quad-uniform test: m is reduced over the quad, the per-thread l is not)
        const bool growA = bmA > mA && mA != -INFINITY, growB = bmB > mB && mB != -INFINITY;
        if (growA || growB) {
          const float aA = growA ? ex2((mA - bmA) * scale_log2) : 1.f;
          const float aB = growB ? ex2((mB - bmB) * scale_log2) : 1.f;
          lA *= aA;
          lB *= aB;
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            acc[j][0] *= aA; acc[j][1] *= aA;
            acc[j][2] *= aB; acc[j][3] *= aB;
          }
        }
        mA = fmaxf(mA, bmA);
        mB = fmaxf(mB, bmB);
        // p = exp2((s - m) * log2(e)/sqrt(d)) as one FFMA + MUFU; masked -inf -> 0
        const float oA = mA == -INFINITY ? 0.f : -mA * scale_log2;
        const float oB = mB == -INFINITY ? 0.f : -mB * scale_log2;
#pragma unroll
        for (int sb = 0; sb < KC / 16; ++sb) {
          if (sb < sb_lo || sb >= sb_hi) continue;   // warp-uniform skip
          float p[2][4];
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            p[j][0] = ex2(fmaf(s[sb][j][0], scale_log2, oA));
            p[j][1] = ex2(fmaf(s[sb][j][1], scale_log2, oA));
            p[j][2] = ex2(fmaf(s[sb][j][2], scale_log2, oB));
            p[j][3] = ex2(fmaf(s[sb][j][3], scale_log2, oB));
            lA += p[j][0] + p[j][1];
            lB += p[j][2] + p[j][3];
          }
          const uint32_t pa[4] = {pack_bf16(p[0][0], p[0][1]), pack_bf16(p[0][2], p[0][3]),
                                  pack_bf16(p[1][0], p[1][1]), pack_bf16(p[1][2], p[1][3])};
          // O += P V  (16 keys x 64 dims)
#pragma unroll
          for (int jj = 0; jj < 4; ++jj) {
            uint32_t v0, v1, v2, v3;
            ldsm_x4_t(vt + sb * 2048 + vofs[jj], v0, v1, v2, v3);
            mma_bf16(acc[2 * jj], pa, v0, v1);
            mma_bf16(acc[2 * jj + 1], pa, v2, v3);
          }
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(kv_empty + 8 * kv_stage);
      if (++kv_stage == kKVStages) { kv_stage = 0; kv_phase ^= 1; }
    }
    // --- normalise and store head h of this warp's rows (pad / empty rows -> 0) ---------
    lA += __shfl_xor_sync(0xffffffffu, lA, 1);
    lA += __shfl_xor_sync(0xffffffffu, lA, 2);
    lB += __shfl_xor_sync(0xffffffffu, lB, 1);
    lB += __shfl_xor_sync(0xffffffffu, lB, 2);
    const float iA = (ra.y > ra.x && lA > 0.f) ? 1.f / lA : 0.f;
    const float iB = (rb.y > rb.x && lB > 0.f) ? 1.f / lB : 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int col = h * DH + j * 8 + 2 * t4;
      if (rowA < num_slots)
        *reinterpret_cast<uint32_t*>(O + rowA * d_model + col) = pack_bf16(acc[j][0] * iA, acc[j][1] * iA);
      if (rowB < num_slots)
        *reinterpret_cast<uint32_t*>(O + rowB * d_model + col) = pack_bf16(acc[j][2] * iB, acc[j][3] * iB);
    }
  }
#ifdef TCB_ATTN_PROBE
  if (lane == 0 && blockIdx.x < 2 && (warp == 0 || warp == 5))
    printf("attnprobe cta %d warp %d total %lld wait_q %lld wait_kv %lld items %d chunks %d\n",
           blockIdx.x, warp, clock64() - p_start, p_q, p_kv, p_items, p_chunks);
#endif
}

// fp32 path: one warp per (query slot, head); keys restricted to the query's own request
// (the only entries M leaves finite); online softmax in fp32.
__global__ void __launch_bounds__(128)
attn_f32_kernel(const float* __restrict__ qkv, const int32_t* __restrict__ seg_ids,
                const int4* __restrict__ segtab, float* __restrict__ O, int64_t num_slots,
                int d_model, int dh, float scale) {
  const int lane = threadIdx.x & 31;
  const int64_t slot = static_cast<int64_t>(blockIdx.x) * 4 + (threadIdx.x >> 5);
  const int h = blockIdx.y;
  if (slot >= num_slots) return;
  const int64_t ld = 3 * static_cast<int64_t>(d_model);
  float* o = O + slot * d_model + h * dh;
  const int seg = __ldg(&seg_ids[slot]);
  if (seg < 0) {
    for (int c = lane; c < dh; c += 32) o[c] = 0.f;
    return;
  }
  const int4 rec = __ldg(&segtab[1 + seg]);
  const float* q = qkv + slot * ld + h * dh;
  const float q0 = lane < dh ? q[lane] : 0.f;
  const float q1 = lane + 32 < dh ? q[lane + 32] : 0.f;
  float m = -INFINITY, l = 0.f, a0 = 0.f, a1 = 0.f;
  for (int j = rec.x; j < rec.x + rec.y; ++j) {
    const float* kr = qkv + static_cast<int64_t>(j) * ld + d_model + h * dh;
    float dot = (lane < dh ? q0 * kr[lane] : 0.f) + (lane + 32 < dh ? q1 * kr[lane + 32] : 0.f);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) dot += __shfl_xor_sync(0xffffffffu, dot, off);
    const float s = dot * scale;
    const float nm = fmaxf(m, s);
    const float alpha = expf(m - nm);
    const float p = expf(s - nm);
    l = l * alpha + p;
    const float* vr = kr + d_model;
    a0 = a0 * alpha + (lane < dh ? p * vr[lane] : 0.f);
    a1 = a1 * alpha + (lane + 32 < dh ? p * vr[lane + 32] : 0.f);
    m = nm;
  }
  if (lane < dh) o[lane] = a0 / l;
  if (lane + 32 < dh) o[lane + 32] = a1 / l;
}

}  // namespace

cudaError_t launch_attention_bf16(int64_t num_slots, int d_model, int num_heads,
                                  const void* qkv, const int32_t* seg_ids, const int4* segtab,
                                  void* O, cudaStream_t s) {
  if (num_slots == 0) return cudaSuccess;
  static bool attr = false;
  static int sms = 0;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(attn_bf16_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, kAttnSmem);
    if (e != cudaSuccess) return e;
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    attr = true;
  }
  CUtensorMap map;
  if (!make_tmap_bf16(&map, qkv, static_cast<uint64_t>(num_slots), 3ull * d_model, 64, 64, 128))
    return cudaErrorInvalidValue;
  const int64_t qblocks = (num_slots + AQ - 1) / AQ;
  const int items = static_cast<int>(qblocks * num_heads);
  const unsigned grid = static_cast<unsigned>(items < sms ? items : sms);
  const float scale_log2 = 1.4426950408889634f / sqrtf(static_cast<float>(DH));
  attn_bf16_kernel<<<grid, (ACW + 2) * 32, kAttnSmem, s>>>(
      map, seg_ids, segtab, static_cast<__nv_bfloat16*>(O), num_slots, d_model, num_heads,
      items, scale_log2);
  return cudaGetLastError();
}

cudaError_t launch_attention_f32(int64_t num_slots, int d_model, int num_heads,
                                 const float* qkv, const int32_t* seg_ids, const int4* segtab,
                                 float* O, cudaStream_t s) {
  if (num_slots == 0) return cudaSuccess;
  const int dh = d_model / num_heads;
  dim3 grid(static_cast<unsigned>((num_slots + 3) / 4), num_heads);
  attn_f32_kernel<<<grid, 128, 0, s>>>(qkv, seg_ids, segtab, O, num_slots, d_model, dh,
                                       1.f / sqrtf(static_cast<float>(dh)));
  return cudaGetLastError();
}

}  // namespace k
}  // namespace tcb
