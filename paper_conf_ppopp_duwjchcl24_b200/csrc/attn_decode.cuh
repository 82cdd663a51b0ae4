// Decode attention over the paged KV cache:
// one query token per sequence, split over the context in chunks of CH
// positions.  The arithmetic of one work item (head, sequence, chunk) lives here.
//
// A work item is run by a group of DC_THREADS = 128 threads (4 warps):
//  * issue: warp 0 stages the chunk's cached K and V page blocks (16 tokens x d
//    bf16 = 4 KiB each, contiguous in the pool) into shared memory with
//    cp.async.bulk on one mbarrier (one DRAM round trip per item);
//  * compute: the new token (position pos) comes from the qkv buffer and is
//    appended to its page by the chunk that holds it; phase 1: warp w scores
//    positions [w CH/4, (w+1) CH/4) (a token row spread over d/8 lanes, shuffle
//    dot products); two-pass softmax over the chunk; phase 2: thread (slot, vec)
//    accumulates p_t V[t] over t = slot (mod SLOTS).  Chunks of one (sequence,
//    head) are merged in chunk order by the last item to finish (acq_rel counter).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include "../../include/liger.h"
#include "common.cuh"

namespace liger {

constexpr int KVB = LIGER_KV_BLOCK;
constexpr int DC_CHUNK_MIN = 32;   // positions per item: 32 or 64, chosen per launch
constexpr int DC_THREADS = 128;
constexpr int DC_MAX_SPLITS = 64;  // chunks per (sequence, head): ctx <= 64 * CH

__host__ __device__ __forceinline__ int64_t kv_off(int page, int kv, int heads, int head, int tok, int D) {
  return ((((int64_t)page * 2 + kv) * heads + head) * KVB + tok) * D;
}

// Chunk length for a decode step of b sequences x heads at context ctx: 32-position
// chunks only when 64-position ones would leave the SMs with fewer than ~2.5 items
// each (tools/kbench_attn.py, profiles/r01/attn_chunk_sweep.txt: 64 wins at b = 4,
// ctx 300 (9.8 vs 13.5 us) and b = 2, ctx 300 (7.8 vs 8.8); 32 at b = 2, ctx 160).
inline int dec_attn_chunk(int b, int heads, int ctx) {
  const bool small = (size_t)b * heads * ((ctx + 63) / 64) * 2 < (size_t)148 * 5;
  return (small && (ctx + 31) / 32 <= DC_MAX_SPLITS) ? 32 : 64;
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
  int max_pages, pos, heads;
  float* ws;                  // chunk partials [b * heads][nsp][D + 2]
  int* counters;              // [b * heads], zero between uses
};

// Shared-memory working set of one item (sK / sV: CH x D bf16 each).
template <int D, int CH>
struct DecAttnSmem {
  static constexpr int NVEC = D / 8;
  static constexpr int SLOTS = DC_THREADS / NVEC;
  __nv_bfloat16* sK;
  __nv_bfloat16* sV;
  uint64_t* bar;   // completes when the item's cached K/V have landed
  float* sc;       // [CH]
  float* red;      // [DC_THREADS / 32]
  float* part;     // [SLOTS][D]
  float* mw;       // [DC_MAX_SPLITS]
  float* lw;       // [DC_MAX_SPLITS]
  int* last;
};

// Warp 0 of the item's group (lane = 0..31): stage cached positions [t0, min(t1, pos)).
// The caller has initialised `bar` (count 1); this arrives on it with the byte count.
// sQ (optional): also stage the item's query (d bf16) -- only when q is already
// complete when the staging is issued.
template <int D, int CH>
__device__ __forceinline__ void dec_attn_issue(const DecAttnArgs& a, int head, int bi, int sp, __nv_bfloat16* sK,
                                               __nv_bfloat16* sV, uint64_t* bar, int lane,
                                               __nv_bfloat16* sQ = nullptr) {
  const int ctx = a.pos + 1;
  const int t0 = sp * CH, t1 = min(ctx, t0 + CH);
  const int tc1 = min(t1, a.pos);
  const int npg = tc1 > t0 ? (tc1 - t0 + KVB - 1) / KVB : 0;
  const int32_t* pt = a.page_table + (int64_t)bi * a.max_pages;
  if (lane == 0) {
    mbar_arrive_expect_tx(bar, (uint32_t)npg * 2 * KVB * D * 2 + (sQ ? D * 2 : 0));
    if (sQ) bulk_load(sQ, a.qkv + (int64_t)bi * 3 * a.heads * D + head * D, D * 2, bar);
  }
  __syncwarp();
  if (lane < npg) {   // lane g stages page g (page ids loaded in parallel, not a serial chain)
    const int page = pt[(t0 >> 4) + lane];
    bulk_load(sK + lane * KVB * D, a.kv_pool + kv_off(page, 0, a.heads, head, 0, D), KVB * D * 2, bar);
    bulk_load(sV + lane * KVB * D, a.kv_pool + kv_off(page, 1, a.heads, head, 0, D), KVB * D * 2, bar);
  }
}

// The whole group (tid = 0..127) computes the item once its staging was issued.
// `sync` is the group barrier.  Returns true in the item that merged the chunks
// of its (sequence, head) (or wrote the single-chunk output).
// Phase A of an item: scores, chunk softmax, P.V.  With one chunk (nsp == 1) it
// writes the output; otherwise the chunk partial (acc[D], max, sum) into a.ws.
template <int D, int CH, class Sync>
__device__ __forceinline__ void dec_attn_partial(const DecAttnArgs& a, int head, int bi, int sp, int nsp,
                                                 const DecAttnSmem<D, CH>& sm, uint32_t parity, int tid,
                                                 Sync sync, const __nv_bfloat16* sQ = nullptr) {
  constexpr int LPT = D / 8;         // lanes per token
  constexpr int TPW = 32 / LPT;      // tokens per warp step
  constexpr int WPOS = CH / 4;       // positions per warp in phase 1
  constexpr int STEPS = WPOS / TPW;  // steps for the warp's positions
  constexpr int NVEC = D / 8;
  constexpr int SLOTS = DC_THREADS / NVEC;
  constexpr int PER = CH / SLOTS;    // positions per thread in phase 2
  const int warp = tid >> 5, lane = tid & 31;
  const int pos = a.pos, ctx = pos + 1, heads = a.heads;
  const int t0 = sp * CH, t1 = min(ctx, t0 + CH);
  const int64_t ld = (int64_t)3 * heads * D;
  const __nv_bfloat16* row = a.qkv + (int64_t)bi * ld;
  const __nv_bfloat16* qp = row + head * D;
  const __nv_bfloat16* knew = row + (int64_t)heads * D + head * D;
  const __nv_bfloat16* vnew = row + (int64_t)2 * heads * D + head * D;
  const int32_t* pt = a.page_table + (int64_t)bi * a.max_pages;
  __nv_bfloat16* sK = sm.sK;
  __nv_bfloat16* sV = sm.sV;
  float* sc = sm.sc;
  float* red = sm.red;

  float qf[8];
  if (!sQ) {
    uint4 qv = __ldcg(reinterpret_cast<const uint4*>(qp + (lane % LPT) * 8));
    bf16x8_to_f32(qv, qf);
  }
  const bool has_new = (t0 <= pos && pos < t1);
  if (has_new && tid < 2 * NVEC) {   // append the new token's K/V (position pos) to its page
    const int kv = tid / NVEC, c = (tid % NVEC) * 8;
    const int page = pt[pos / KVB];
    *reinterpret_cast<uint4*>(a.kv_pool + kv_off(page, kv, heads, head, pos % KVB, D) + c) =
        __ldcg(reinterpret_cast<const uint4*>((kv ? vnew : knew) + c));
  }
  mbar_wait(sm.bar, parity);
  if (sQ) bf16x8_to_f32(*reinterpret_cast<const uint4*>(sQ + (lane % LPT) * 8), qf);
  if (has_new && tid < 2 * NVEC) {   // ... and into the staged chunk (the bulk copy may predate it)
    const int kv = tid / NVEC, c = (tid % NVEC) * 8;
    *reinterpret_cast<uint4*>((kv ? sV : sK) + (pos - t0) * D + c) =
        __ldcg(reinterpret_cast<const uint4*>((kv ? vnew : knew) + c));
  }
  sync();

  // ---- phase 1: scores for positions [t0 + warp*WPOS, +WPOS)
  {
    const int c = (lane % LPT) * 8;
#pragma unroll
    for (int st = 0; st < STEPS; ++st) {
      const int lt = warp * WPOS + st * TPW + lane / LPT;   // local position
      float dot = 0.f;
      if (t0 + lt < t1) {
        float f[8];
        bf16x8_to_f32(*reinterpret_cast<const uint4*>(sK + lt * D + c), f);
#pragma unroll
        for (int i = 0; i < 8; ++i) dot += qf[i] * f[i];
      }
#pragma unroll
      for (int off = LPT / 2; off > 0; off >>= 1) dot += __shfl_xor_sync(0xffffffffu, dot, off);
      if (t0 + lt < t1 && (lane % LPT) == 0) sc[lt] = dot;
    }
  }
  sync();
  const int n = t1 - t0;
  float mx = (tid < n) ? sc[tid] : -INFINITY;   // n <= CH <= DC_THREADS
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, off));
  if (lane == 0) red[warp] = mx;
  sync();
  mx = fmaxf(fmaxf(red[0], red[1]), fmaxf(red[2], red[3]));
  sync();
  float p_t = 0.f;
  if (tid < n) {
    p_t = __expf(sc[tid] - mx);
    sc[tid] = p_t;
  }
  float sum = p_t;
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, off);
  if (lane == 0) red[warp] = sum;
  sync();
  const float l = red[0] + red[1] + red[2] + red[3];

  // ---- phase 2: o = sum_t p_t v_t
  const int vec = tid % NVEC, slot = tid / NVEC;
  float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#pragma unroll 4
  for (int i = 0; i < PER; ++i) {
    const int lt = slot + i * SLOTS;
    if (t0 + lt < t1) {
      const float pw = sc[lt];
      float f[8];
      bf16x8_to_f32(*reinterpret_cast<const uint4*>(sV + lt * D + vec * 8), f);
#pragma unroll
      for (int e = 0; e < 8; ++e) acc[e] += pw * f[e];
    }
  }
  float* part = sm.part;
#pragma unroll
  for (int i = 0; i < 8; ++i) part[slot * D + vec * 8 + i] = acc[i];
  sync();

  if (nsp == 1) {
    for (int e = tid; e < D; e += DC_THREADS) {
      float s2 = 0.f;
#pragma unroll
      for (int s3 = 0; s3 < SLOTS; ++s3) s2 += part[s3 * D + e];
      a.o[(int64_t)bi * heads * D + head * D + e] = __float2bfloat16_rn(s2 / l);
    }
    sync();   // smem (sc / part) is reused by the group's next item
    return;
  }
  const int64_t unit = (int64_t)bi * heads + head;
  float* wp = a.ws + (unit * nsp + sp) * (D + 2);
  for (int e = tid; e < D; e += DC_THREADS) {
    float s2 = 0.f;
#pragma unroll
    for (int s3 = 0; s3 < SLOTS; ++s3) s2 += part[s3 * D + e];
    wp[e] = s2;
  }
  if (tid == 0) {
    wp[D] = mx;
    wp[D + 1] = l;
  }
  sync();
}

// Phase B (nsp > 1): merge the nsp chunk partials of (sequence bi, head) in chunk
// order into the output.  Every load issued in parallel (one per thread, then smem).
template <int D, int CH, class Sync>
__device__ __forceinline__ void dec_attn_merge(const DecAttnArgs& a, int head, int bi, int nsp,
                                               const DecAttnSmem<D, CH>& sm, int tid, Sync sync) {
  const int heads = a.heads;
  const int64_t unit = (int64_t)bi * heads + head;
  float* mw = sm.mw;
  float* lw = sm.lw;
  for (int s2 = tid; s2 < nsp; s2 += DC_THREADS) {
    const float* w2 = a.ws + (unit * nsp + s2) * (D + 2);
    mw[s2] = __ldcg(&w2[D]);
    lw[s2] = __ldcg(&w2[D + 1]);
  }
  sync();
  float M = -INFINITY;
  for (int s2 = 0; s2 < nsp; ++s2) M = fmaxf(M, mw[s2]);
  float L = 0.f;
  for (int s2 = 0; s2 < nsp; ++s2) L += lw[s2] * __expf(mw[s2] - M);
  for (int e = tid; e < D; e += DC_THREADS) {
    float acc2 = 0.f;
    for (int z0 = 0; z0 < nsp; z0 += 8) {
      float v[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) v[i] = (z0 + i < nsp) ? __ldcg(&a.ws[(unit * nsp + z0 + i) * (D + 2) + e]) : 0.f;
#pragma unroll
      for (int i = 0; i < 8; ++i)
        if (z0 + i < nsp) acc2 += v[i] * __expf(mw[z0 + i] - M);
    }
    a.o[(int64_t)bi * heads * D + head * D + e] = __float2bfloat16_rn(acc2 / L);
  }
  sync();
}

}  // namespace liger
