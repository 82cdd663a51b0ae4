// Attention over the paged KV cache (PAPER.md P:316 KV cache).
//
// Paged pool layout: [n_pages][2 (K,V)][heads][16 tokens][d] bf16; a sequence's
// page_table row maps token position p to page page_table[p / 16].
//
//  * prefill: flash-style causal attention on the tcgen05 tensor cores (TMA-loaded
//    Q / K / V tiles, S and O accumulators in TMEM, softmax warps owning one query
//    row each; persistent CTAs over (query tile, sequence, head) items), which also
//    appends the prompt's K / V to the cache pages (attn_prefill_tc.cuh).
//  * decode: one query per sequence; persistent CTAs stream 32-position chunks of
//    the cache through a cp.async.bulk ring, online softmax per lane group in
//    registers, deterministic merge of the split partials (attn_decode.cuh).
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>

#include <algorithm>

#include "attn_decode.cuh"
#include "attn_prefill_tc.cuh"
#include "common.cuh"
#include "kernels.h"

namespace liger {

// ================================================================== prefill
// tcgen05 / TMEM / TMA kernel: attn_prefill_tc.cuh.

template <int D>
static int launch_prefill_tc(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages,
                             int b, int s, int heads, cudaStream_t stream) {
  CUtensorMap tm;
  if (gemm_act_map(&tm, qkv, b * s, 3 * heads * D, (int64_t)3 * heads * D, PT_BQ)) return LIGER_ECUDA;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_prefill_tc_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, PtSmem<D>::ALLOC);
    attr = true;
  }
  const int items = (s + PT_BQ - 1) / PT_BQ * b * heads;
  const int grid = std::min(items, sm_count());
  return launch_pdl(attn_prefill_tc_kernel<D>, dim3(grid), dim3(PT_THREADS), (size_t)PtSmem<D>::ALLOC, stream, tm,
                    (__nv_bfloat16*)o, (__nv_bfloat16*)kv_pool, page_table, max_pages, b,
                    s, heads)
             ? LIGER_ECUDA
             : 0;
}

int attn_prefill_launch(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                        int s, int heads, int d, cudaStream_t stream) {
  if (b <= 0 || s <= 0) return 0;
  if (d != 64 && d != 128) return LIGER_EINVAL;
  if ((int64_t)b * s > (int64_t)1 << 30) return LIGER_EINVAL;
  return d == 128 ? launch_prefill_tc<128>(qkv, o, kv_pool, page_table, max_pages, b, s, heads, stream)
                  : launch_prefill_tc<64>(qkv, o, kv_pool, page_table, max_pages, b, s, heads, stream);
}

// ================================================================== decode
// See attn_decode.cuh for the design.  Persistent CTAs of 128 threads; CTA c takes
// items c, c + G, ... (item = (sequence, head, split), split-major within a
// (sequence, head) so that consecutive items of a CTA are different heads) and
// streams their 32-position chunks through a DC_NS-stage ring.
// Enough for every launch with at most b sequences and context at most ctx (the split
// count depends on both), so one buffer serves all passes of a slot.
size_t attn_decode_workspace_bytes(int b, int heads, int d, int ctx) {
  size_t rows = 0;
  for (int bb = 1; bb <= b; ++bb)
    for (int c = DC_CH; c < ctx + DC_CH; c += DC_CH) {
      int cps, nsp;
      dec_attn_plan(bb, heads, std::min(c, ctx), &cps, &nsp);
      rows = std::max(rows, (size_t)bb * heads * nsp);
    }
  return ATTN_COUNTER_BYTES + rows * (d + 2) * sizeof(float);
}

template <int D>
struct DecSmem {
  __nv_bfloat16 kv[DC_NS][2][DC_CH * D];   // stage s: K rows then V rows of the chunk
  float st_acc[DC_CWARPS * (32 / (D / 8))][D];     // per lane group: acc (item merge)
  float st_m[DC_CWARPS * (32 / (D / 8))], st_l[DC_CWARPS * (32 / (D / 8))];
  float mw[DC_MAX_SPLITS], lw[DC_MAX_SPLITS];
  uint64_t full[DC_NS], empty[DC_NS];
  int last;
};

// Warps 0..DC_CWARPS-1 compute, warp DC_CWARPS (lane 0) is the producer: it walks the same task list
// (chunk j of item i = blockIdx.x + k G) and keeps DC_NS chunks in flight, refilling a
// stage as soon as the four compute warps have released it (empty[s]).
template <int D>
__global__ void __launch_bounds__(DC_THREADS + 32, DC_CTAS_PER_SM) attn_decode_kernel(const DecAttnArgs a) {
  constexpr int LPT = D / 8;          // lanes per token row (16 B each)
  constexpr int TPW = 32 / LPT;       // token rows per warp step
  constexpr int NG = DC_CWARPS * TPW; // lane groups per CTA
  constexpr int PPG = DC_CH / NG;     // positions per lane group per chunk
  const TraceStart tr0 = trace_begin();
  extern __shared__ __align__(128) uint8_t dsm[];
  DecSmem<D>& sm = *reinterpret_cast<DecSmem<D>*>(dsm);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int G = gridDim.x;
  const int pos = a.pos, ctx = pos + 1, heads = a.heads, nsp = a.nsp, cps = a.cps;
  const int nch = (ctx + DC_CH - 1) / DC_CH;
  const int n_items = a.b * heads * nsp;
  auto item_chunks = [&](int it, int* c0) {
    *c0 = (it % nsp) * cps;
    return max(0, min(nch, *c0 + cps) - *c0);
  };
  if (tid == 0) {
    for (int s = 0; s < DC_NS; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], DC_CWARPS);   // one arrive per compute warp
    }
    fence_barrier_init();
  }
  __syncthreads();
  if (warp == DC_CWARPS) {
    // ---------------- producer warp: the page ids of up to 32 pages are fetched in one
    // parallel load (no serial page-table round trips on the refill path); lane 0
    // paces the ring, lanes 0 / 1 issue the two pages of a chunk
    int k = 0;
    bool waited = false;
    for (int it = blockIdx.x; it < n_items; it += G) {
      int c0;
      const int nc = item_chunks(it, &c0);
      const int bh = it / nsp, bi = bh / heads, head = bh % heads;
      const int32_t* pt = a.page_table + (int64_t)bi * a.max_pages + c0 * (DC_CH / KVB);
      const int npages_item = (min(ctx, (c0 + nc) * DC_CH) - c0 * DC_CH + KVB - 1) / KVB;
      for (int j0 = 0; j0 < nc; j0 += 32 / (DC_CH / KVB)) {
        const int pg0 = j0 * (DC_CH / KVB);
        const int my_page = (pg0 + lane < npages_item) ? pt[pg0 + lane] : 0;
        for (int j = j0; j < min(nc, j0 + 32 / (DC_CH / KVB)); ++j, ++k) {
          const int s = k % DC_NS;
          const int t0 = (c0 + j) * DC_CH;
          const int tc1 = min(t0 + DC_CH, pos);                       // cached positions [t0, tc1)
          const int npg = tc1 > t0 ? (tc1 - t0 + KVB - 1) / KVB : 0;
          if (lane == 0) {
            if (k >= DC_NS) mbar_wait(&sm.empty[s], (uint32_t)((k / DC_NS) - 1) & 1u);
            mbar_arrive_expect_tx(&sm.full[s], (uint32_t)npg * 2 * KVB * D * 2);
          }
          __syncwarp();
          const int page = __shfl_sync(0xffffffffu, my_page, ((j - j0) * (DC_CH / KVB) + lane) & 31);
          if (lane < npg) {
            bulk_load(&sm.kv[s][0][lane * KVB * D], a.kv_pool + kv_off(page, 0, heads, head, 0, D), KVB * D * 2,
                      &sm.full[s]);
            bulk_load(&sm.kv[s][1][lane * KVB * D], a.kv_pool + kv_off(page, 1, heads, head, 0, D), KVB * D * 2,
                      &sm.full[s]);
          }
          // The cached positions were written by earlier passes and the page table at
          // admission: the first stages are requested before the PDL wait.
          if (k == DC_NS - 1) {
            grid_dependency_wait();
            waited = true;
          }
        }
      }
    }
    if (!waited) grid_dependency_wait();
    grid_dependency_trigger();   // after the wait ("trigger after wait", common.cuh)
    return;
  }
  // ---------------- compute warps 0..3
  const int grp = warp * TPW + lane / LPT;   // lane group 0..NG-1
  const int gl = lane % LPT;                 // lane within the group: dims [8 gl, 8 gl + 8)
  pdl_enter();   // q and the new token's k / v come from the QKV kernel
  const uint64_t tr1 = trace_now();
  const int64_t ld = (int64_t)3 * heads * D;
  int k = 0;
  bool merged_any = false;
  // q of the CTA's next item is loaded one item ahead (its latency hides behind the ring)
  auto load_q = [&](int it) {
    const int bh = it / nsp, bi = bh / heads, head = bh % heads;
    return __ldcg(reinterpret_cast<const uint4*>(a.qkv + (int64_t)bi * ld + head * D + gl * 8));
  };
  uint4 q_next = blockIdx.x < n_items ? load_q(blockIdx.x) : make_uint4(0, 0, 0, 0);
  for (int it = blockIdx.x; it < n_items; it += G) {
    int c0;
    const int nc = item_chunks(it, &c0);
    const int sp = it % nsp, bh = it / nsp, bi = bh / heads, head = bh % heads;
    const __nv_bfloat16* row = a.qkv + (int64_t)bi * ld;
    float q[8], kn[8], vn[8];
    bf16x8_to_f32(q_next, q);
    if (it + G < n_items) q_next = load_q(it + G);
    const bool has_new = (c0 + nc) * DC_CH > pos && c0 * DC_CH <= pos;
    if (has_new) {   // the new token (position pos): from the QKV output, appended to its page
      const uint4 kv4 = __ldcg(reinterpret_cast<const uint4*>(row + (int64_t)heads * D + head * D + gl * 8));
      const uint4 vv4 = __ldcg(reinterpret_cast<const uint4*>(row + (int64_t)2 * heads * D + head * D + gl * 8));
      bf16x8_to_f32(kv4, kn);
      bf16x8_to_f32(vv4, vn);
      if (grp == 0) {
        const int page = a.page_table[(int64_t)bi * a.max_pages + pos / KVB];
        *reinterpret_cast<uint4*>(a.kv_pool + kv_off(page, 0, heads, head, pos % KVB, D) + gl * 8) = kv4;
        *reinterpret_cast<uint4*>(a.kv_pool + kv_off(page, 1, heads, head, pos % KVB, D) + gl * 8) = vv4;
      }
    }
    float m = -INFINITY, l = 0.f;
    float2 acc2[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
    float2 q2[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) q2[e] = make_float2(q[2 * e], q[2 * e + 1]);
    for (int j = 0; j < nc; ++j, ++k) {
      const int s = k % DC_NS;
      mbar_wait(&sm.full[s], (uint32_t)(k / DC_NS) & 1u);
      const int t0 = (c0 + j) * DC_CH;
      const __nv_bfloat16* sK = sm.kv[s][0];
      const __nv_bfloat16* sV = sm.kv[s][1];
      // scores of this lane group's PPG positions (independent chains), then one
      // online-softmax update for all of them
      // packed fp32x2 arithmetic (FFMA2 / FMUL2): a K or V row slice of 8 bf16 is 4 bf16x2
      // words, unpacked to 4 float2 (element 2i in the low half of word i)
      float sc[PPG];
      float2 vf[PPG][4];
      const bool full_chunk = t0 + DC_CH <= pos;   // every position cached (block-uniform)
#pragma unroll
      for (int r = 0; r < PPG; ++r) {
        const int lt = r * NG + grp;
        const int t = t0 + lt;
        float2 kf[4];
        if (full_chunk || t < pos) {
          const uint4 kw = *reinterpret_cast<const uint4*>(sK + lt * D + gl * 8);
          const uint4 vw = *reinterpret_cast<const uint4*>(sV + lt * D + gl * 8);
          const uint32_t kk[4] = {kw.x, kw.y, kw.z, kw.w}, vv[4] = {vw.x, vw.y, vw.z, vw.w};
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            kf[e] = make_float2(__uint_as_float(kk[e] << 16), __uint_as_float(kk[e] & 0xFFFF0000u));
            vf[r][e] = make_float2(__uint_as_float(vv[e] << 16), __uint_as_float(vv[e] & 0xFFFF0000u));
          }
        } else {
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            kf[e] = make_float2(kn[2 * e], kn[2 * e + 1]);
            vf[r][e] = make_float2(vn[2 * e], vn[2 * e + 1]);
          }
        }
        float2 d2 = __fmul2_rn(q2[0], kf[0]);
#pragma unroll
        for (int e = 1; e < 4; ++e) d2 = __ffma2_rn(q2[e], kf[e], d2);
        sc[r] = d2.x + d2.y;
      }
#pragma unroll
      for (int off = LPT / 2; off > 0; off >>= 1)
#pragma unroll
        for (int r = 0; r < PPG; ++r) sc[r] += __shfl_xor_sync(0xffffffffu, sc[r], off);
      __syncwarp();
      if (lane == 0) mbar_arrive(&sm.empty[s]);   // this warp is done with stage s (values in registers)
      float mn = m;
#pragma unroll
      for (int r = 0; r < PPG; ++r)
        if (full_chunk || t0 + r * NG + grp <= pos) mn = fmaxf(mn, sc[r]);
      if (mn != -INFINITY) {   // group-uniform: at least one valid position so far
        const float scale = __expf(m - mn);
        l *= scale;
        const float2 sc2 = make_float2(scale, scale);
#pragma unroll
        for (int e = 0; e < 4; ++e) acc2[e] = __fmul2_rn(acc2[e], sc2);
#pragma unroll
        for (int r = 0; r < PPG; ++r) {
          if (full_chunk || t0 + r * NG + grp <= pos) {
            const float p = __expf(sc[r] - mn);
            l += p;
            const float2 p2 = make_float2(p, p);
#pragma unroll
            for (int e = 0; e < 4; ++e) acc2[e] = __ffma2_rn(p2, vf[r][e], acc2[e]);
          }
        }
        m = mn;
      }
    }
    // ---- merge the lane groups' states (fixed order), then the item's result
    if (gl == 0) {
      sm.st_m[grp] = m;
      sm.st_l[grp] = l;
    }
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      sm.st_acc[grp][gl * 8 + 2 * e] = acc2[e].x;
      sm.st_acc[grp][gl * 8 + 2 * e + 1] = acc2[e].y;
    }
    named_bar_sync(1, DC_THREADS);
    float M = -INFINITY;
#pragma unroll
    for (int g = 0; g < NG; ++g) M = fmaxf(M, sm.st_m[g]);
    float L = 0.f;
#pragma unroll
    for (int g = 0; g < NG; ++g) L += sm.st_m[g] == -INFINITY ? 0.f : sm.st_l[g] * __expf(sm.st_m[g] - M);
    const int64_t unit = (int64_t)bi * heads + head;
    if (nsp == 1) {
      for (int e = tid; e < D; e += DC_THREADS) {
        float v = 0.f;
#pragma unroll
        for (int g = 0; g < NG; ++g) v += sm.st_m[g] == -INFINITY ? 0.f : sm.st_acc[g][e] * __expf(sm.st_m[g] - M);
        a.o[(int64_t)bi * heads * D + head * D + e] = __float2bfloat16_rn(v / L);
      }
      named_bar_sync(1, DC_THREADS);
      continue;
    }
    float* wp = a.ws + (unit * nsp + sp) * (D + 2);
    for (int e = tid; e < D; e += DC_THREADS) {
      float v = 0.f;
#pragma unroll
      for (int g = 0; g < NG; ++g) v += sm.st_m[g] == -INFINITY ? 0.f : sm.st_acc[g][e] * __expf(sm.st_m[g] - M);
      wp[e] = v;
    }
    if (tid == 0) {
      wp[D] = M;
      wp[D + 1] = L;
    }
    named_bar_sync(1, DC_THREADS);   // the CTA's partial is written (CTA scope) ...
    if (tid == 0) {
      __threadfence();               // ... and made visible device-wide by one cumulative fence
      int prev;
      asm volatile("atom.add.acq_rel.gpu.global.s32 %0, [%1], 1;" : "=r"(prev) : "l"(&a.counters[unit]) : "memory");
      sm.last = (prev == nsp - 1);
    }
    named_bar_sync(1, DC_THREADS);
    if (sm.last) {   // the last split of (sequence, head): merge the splits in split order
      for (int z = tid; z < nsp; z += DC_THREADS) {
        const float* w2 = a.ws + (unit * nsp + z) * (D + 2);
        sm.mw[z] = __ldcg(&w2[D]);
        sm.lw[z] = __ldcg(&w2[D + 1]);
      }
      named_bar_sync(1, DC_THREADS);
      float MM = -INFINITY;
      for (int z = 0; z < nsp; ++z) MM = fmaxf(MM, sm.mw[z]);
      float LL = 0.f;
      for (int z = 0; z < nsp; ++z) LL += sm.lw[z] * __expf(sm.mw[z] - MM);
      for (int e = tid; e < D; e += DC_THREADS) {
        float v = 0.f;
        for (int z0 = 0; z0 < nsp; z0 += 8) {
          float w8[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) w8[i] = (z0 + i < nsp) ? __ldcg(&a.ws[(unit * nsp + z0 + i) * (D + 2) + e]) : 0.f;
#pragma unroll
          for (int i = 0; i < 8; ++i)
            if (z0 + i < nsp) v += w8[i] * __expf(sm.mw[z0 + i] - MM);
        }
        a.o[(int64_t)bi * heads * D + head * D + e] = __float2bfloat16_rn(v / LL);
      }
      if (tid == 0) a.counters[unit] = 0;
      merged_any = true;
    }
    named_bar_sync(1, DC_THREADS);
  }
  if (tid == 0) trace_write(merged_any ? (TK_ATTN_DEC | 0x100) : TK_ATTN_DEC, tr0, tr1);
}

template <int D>
static int launch_decode(const DecAttnArgs& a, cudaStream_t stream) {
  const size_t dsmem = sizeof(DecSmem<D>) + 128;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_decode_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem);
    attr = true;
  }
  const int items = a.b * a.heads * a.nsp;
  const int grid = std::min(items, 148 * DC_CTAS_PER_SM);
  return launch_pdl(attn_decode_kernel<D>, dim3(grid), dim3(DC_THREADS + 32), dsmem, stream, a);
}

int attn_decode_launch(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                       int pos, int heads, int d, void* workspace, size_t ws_bytes, cudaStream_t stream) {
  if (b <= 0) return 0;
  const int ctx = pos + 1;
  DecAttnArgs a;
  dec_attn_plan(b, heads, ctx, &a.cps, &a.nsp);
  // the page table row must hold position pos (the new token's page)
  if (a.nsp > DC_MAX_SPLITS || (d != 64 && d != 128) || pos < 0 || pos >= max_pages * KVB) return LIGER_EINVAL;
  if (a.nsp > 1) {
    if (!workspace || ws_bytes < attn_decode_workspace_bytes(b, heads, d, ctx) ||
        (size_t)b * heads * 4 > ATTN_COUNTER_BYTES)
      return LIGER_EINVAL;
  }
  a.qkv = (const __nv_bfloat16*)qkv;
  a.o = (__nv_bfloat16*)o;
  a.kv_pool = (__nv_bfloat16*)kv_pool;
  a.page_table = page_table;
  a.max_pages = max_pages;
  a.pos = pos;
  a.heads = heads;
  a.b = b;
  a.counters = (int*)workspace;
  a.ws = workspace ? (float*)((char*)workspace + ATTN_COUNTER_BYTES) : nullptr;
  const int rc = d == 128 ? launch_decode<128>(a, stream) : launch_decode<64>(a, stream);
  return rc ? LIGER_ECUDA : 0;
}

void preload_attention_kernels() {
  preload_kernel(attn_prefill_tc_kernel<64>);
  preload_kernel(attn_prefill_tc_kernel<128>);
  preload_kernel(attn_decode_kernel<64>);
  preload_kernel(attn_decode_kernel<128>);
}

LIGER_TRACE_SETTER(attention)

}  // namespace liger
