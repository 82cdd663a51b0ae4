// Decode attention over the paged KV cache (C4):
// one query token per sequence at position pos, keys/values at positions [0, pos]
// (the cache holds [0, pos); the new token's k / v come from the QKV output and are
// appended to its page here).
//
// HBM-bound: every cached K and V byte is read once.  Design (B200, 148 SMs):
//  * work = (sequence, head, split); a split is a run of 32-position chunks (two
//    16-token pages of K and of V, 4 x 4 KiB at d = 128); the split count is chosen
//    per launch so that there is ~1 item per CTA slot;
//  * a persistent grid (about 2 items per SM, up to 3 CTAs resident) walks its items' chunks as one task
//    stream through an NS-stage shared-memory ring filled by cp.async.bulk (the TMA
//    bulk engine) on per-stage mbarriers: NS x 16 KiB in flight per CTA, ~192 KiB per
//    SM, enough to cover the DRAM latency at the SM's share of HBM bandwidth; the
//    first NS loads are issued before the PDL wait (the cached positions do not
//    depend on the preceding QKV kernel);
//  * inside a chunk every warp works alone: a token row is spread over d/8 lanes
//    (16 B each), the score is a shuffle reduction over those lanes, and each
//    lane group keeps an online-softmax state (running max m, sum l, acc[8]) in
//    registers -- no shared-memory scores, one __syncthreads per chunk (the stage
//    is free);
//  * at the end of an item the lane groups' states are merged in a fixed order;
//    a single-split item writes o, otherwise the split's (acc, m, l) goes to the
//    workspace and the last split of (sequence, head) to finish (acq_rel counter)
//    merges the splits in split order.  Every reduction order is fixed: the result
//    is deterministic for a given (b, heads, pos).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>

#include "../../include/liger.h"
#include "common.cuh"

namespace liger {

constexpr int KVB = LIGER_KV_BLOCK;
constexpr int DC_CH = 32;          // positions per chunk (two pages)
constexpr int DC_NS = 4;           // ring stages per CTA
constexpr int DC_THREADS = 128;      // compute threads (the producer warp comes on top)
constexpr int DC_CWARPS = DC_THREADS / 32;
constexpr int DC_CTAS_PER_SM = 3;
constexpr int DC_MAX_SPLITS = 64;  // splits per (sequence, head)

__host__ __device__ __forceinline__ int64_t kv_off(int page, int kv, int heads, int head, int tok, int D) {
  return ((((int64_t)page * 2 + kv) * heads + head) * KVB + tok) * D;
}

__device__ __forceinline__ void bf16x8_to_f32(const uint4& v, float* f) {
  const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&v);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    float2 t = __bfloat1622float2(h[i]);
    f[2 * i] = t.x;
    f[2 * i + 1] = t.y;
  }
}

struct DecAttnArgs {
  const __nv_bfloat16* qkv;   // [b, 3 * heads * D]: q (already scaled) | k | v of the new token
  __nv_bfloat16* o;           // [b, heads * D]
  __nv_bfloat16* kv_pool;     // this layer's pages
  const int32_t* page_table;  // [b, max_pages]
  int max_pages, pos, heads, b;
  int nsp;                    // splits per (sequence, head)
  int cps;                    // chunks per split
  float* ws;                  // split partials [b * heads][nsp][D + 2]
  int* counters;              // [b * heads], zero between uses
};

// Split plan of a launch: chunks per split and the split count.  Each CTA slot of a
// full persistent grid gets about one item (an item's fixed costs -- q load, lane-group
// merge, split partial + merge -- are paid once per CTA): (sequence, head) pairs are
// split only while there are fewer items than slots, never below one chunk per split.
inline void dec_attn_plan(int b, int heads, int ctx, int* cps, int* nsp) {
  const int nch = (ctx + DC_CH - 1) / DC_CH;
  // 2 items per SM: with two batches decoding on the two streams, fewer attention CTAs
  // leave more of each SM to the other batch's weight-streaming GEMM (bench capacity
  // 30.35-30.49 vs 29.86-30.06 req/s with 3 per SM; one batch alone: equal within noise,
  // profiles/r02/knob_sweeps_two_stream.txt)
  static const int slots = getenv("LIGER_ATTN_SLOTS") ? atoi(getenv("LIGER_ATTN_SLOTS")) : 148 * 2;
  int want = slots / (b * heads);
  if (want < 1) want = 1;
  if (want > nch) want = nch;
  int c = (nch + want - 1) / want;
  while ((nch + c - 1) / c > DC_MAX_SPLITS) ++c;
  *cps = c;
  *nsp = (nch + c - 1) / c;
}

}  // namespace liger
