// tcb_internal.h -- shared declarations of libtcb (host code + kernel launchers).
#pragma once

#include <cstdint>
#include <cstddef>
#include <string>
#include <vector>

#include "../../include/tcb.h"
#include "../../include/tcb_ops.h"

// Geometry of the tcgen05 segment-masked attention kernel (attention_tc.cu); the host plan
// uses it to report the score elements the kernel evaluates (tcb_plan_info).
constexpr int kAttnQBlock = 128;   // query slots per item (TMEM lanes of S)
constexpr int kAttnKChunk = 128;   // keys per S = QK^T tile
constexpr int kAttnSmRows = 32;    // query rows of one softmax warp
constexpr int kAttnSmKeys = 32;    // keys per liveness decision of the softmax

struct tcb_plan;

namespace tcb {

// Error reporting -------------------------------------------------------------------------
void set_error(const std::string& msg);
void clear_error();
tcb_status fail(tcb_status st, const std::string& msg);

// Plan construction (pack.cpp): init_plan sets the request arrays (all unplaced);
// finish_plan derives the segments in (row, column) order from req_row / req_col and the
// counters.  Every plan producer (tcb_pack, tcb_pack_slotted, the scheduler) uses them.
void init_plan(tcb_plan* p, const int32_t* lengths, int32_t n, int32_t row_len, int32_t max_rows,
               int32_t policy);
void finish_plan(tcb_plan* p);

// Segment-table record (16 bytes), see tcb.h "device form of a plan".
struct SegRec {
  int32_t start, len, tok, req;
};

}  // namespace tcb

struct tcb_plan {
  int32_t n = 0, row_len = 0, num_rows = 0, max_rows = 0, policy = 0;
  int32_t slot_len = 0;                  // slotted ConcatBatching slot size z, 0 = none
  std::vector<int32_t> lengths, req_row, req_col;
  std::vector<int64_t> tok_off;          // request-order offset of each request's tokens
  std::vector<int32_t> seg_req, seg_start;
  tcb_plan_info info{};
};
