// Attention over the paged KV cache (PAPER.md P:316 KV cache).
//
// Paged pool layout: [n_pages][2 (K,V)][heads][16 tokens][d] bf16; a sequence's
// page_table row maps token position p to page page_table[p / 16].
//
//  * prefill: flash-style causal attention with bf16 tensor-core mma.sync
//    (m16n8k16, fp32 accumulate), 64 queries x 64 keys per step, online
//    softmax in registers; the CTA on the diagonal tile also writes that key
//    tile's K/V into the cache pages.
//  * decode: one query per sequence; persistent CTAs stream 32-position chunks of
//    the cache through a cp.async.bulk ring, online softmax per lane group in
//    registers, deterministic merge of the split partials (attn_decode.cuh).
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>

#include <algorithm>

#include "attn_decode.cuh"
#include "common.cuh"
#include "kernels.h"

namespace liger {

// ================================================================== prefill
constexpr int PF_BQ = 128, PF_BK = 64;

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void mma_bf16_16816(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                               uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t pack_bf16(float lo, float hi) {
  __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&v);
}

__device__ __forceinline__ void cp_async16(void* smem_dst, const void* gsrc, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(smem_dst)), "l"(gsrc),
               "r"(valid ? 16 : 0)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// Prefill causal attention, flash-style: CTA = (128-query tile, head, sequence),
// 8 warps x 16 query rows; 64-key tiles of K and V double-buffered in shared
// memory with cp.async (the next tile loads while the current one is
// computed); S = Q K^T and O += P V on bf16 tensor cores (mma.sync m16n8k16,
// fp32 accumulate); online softmax in registers.  The CTA whose query range
// contains a key tile also writes that tile's K/V into the paged cache.
constexpr int PF_THREADS = 256;
template <int D>
__global__ void __launch_bounds__(PF_THREADS) attn_prefill_kernel(const __nv_bfloat16* __restrict__ qkv,
                                                                  __nv_bfloat16* __restrict__ o,
                                                                  __nv_bfloat16* __restrict__ kv_pool,
                                                                  const int32_t* __restrict__ page_table,
                                                                  int max_pages, int s, int heads) {
  constexpr int LDS = D + 8;   // padded smem row (bank-conflict-free ldmatrix)
  constexpr int NV = D / 8;    // 16-byte vectors per row
  extern __shared__ __align__(16) uint8_t pf_smem[];
  __nv_bfloat16* sQ = reinterpret_cast<__nv_bfloat16*>(pf_smem);       // [PF_BQ][LDS]
  __nv_bfloat16* sK = sQ + PF_BQ * LDS;                                  // [2][PF_BK][LDS]
  __nv_bfloat16* sV = sK + 2 * PF_BK * LDS;                              // [2][PF_BK][LDS]

  const int nqt = gridDim.x;
  const int qt = nqt - 1 - blockIdx.x;   // longest (most key tiles) first
  const int head = blockIdx.y, bi = blockIdx.z;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int64_t ld = (int64_t)3 * heads * D;
  const __nv_bfloat16* base = qkv + (int64_t)bi * s * ld;
  const int q0 = qt * PF_BQ;
  const int q_hi = min(s, q0 + PF_BQ);            // rows [q0, q_hi)
  const int nkt = (q_hi - 1) / PF_BK + 1;         // key tiles with k0 <= last row
  pdl_enter();

  auto load_kv = [&](int kt, int buf) {
    const int k0 = kt * PF_BK;
    for (int i = tid; i < PF_BK * NV; i += PF_THREADS) {
      const int r = i / NV, c = (i % NV) * 8;
      const bool ok = k0 + r < s;
      const __nv_bfloat16* rowp = base + (int64_t)(ok ? k0 + r : 0) * ld;
      cp_async16(&sK[(buf * PF_BK + r) * LDS + c], rowp + (int64_t)heads * D + head * D + c, ok);
      cp_async16(&sV[(buf * PF_BK + r) * LDS + c], rowp + (int64_t)2 * heads * D + head * D + c, ok);
    }
  };
  for (int i = tid; i < PF_BQ * NV; i += PF_THREADS) {
    const int r = i / NV, c = (i % NV) * 8;
    const bool ok = q0 + r < s;
    cp_async16(&sQ[r * LDS + c], base + (int64_t)(ok ? q0 + r : 0) * ld + head * D + c, ok);
  }
  load_kv(0, 0);
  cp_async_commit();

  const int g = lane >> 2, tig = lane & 3;
  float m_r[2] = {-INFINITY, -INFINITY}, l_r[2] = {0.f, 0.f};
  float acc[D / 8][4];
#pragma unroll
  for (int j = 0; j < D / 8; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
  const float L2E = 1.4426950408889634f;
  const int wrow0 = q0 + warp * 16;        // this warp's rows [wrow0, wrow0 + 16)
  const int row0 = wrow0 + g;              // this thread's rows: row0, row0 + 8

  for (int kt = 0; kt < nkt; ++kt) {
    const int buf = kt & 1;
    const int k0 = kt * PF_BK;
    if (kt + 1 < nkt) load_kv(kt + 1, buf ^ 1);
    cp_async_commit();
    cp_async_wait<1>();   // tile kt (and Q) landed
    __syncthreads();
    const __nv_bfloat16* cK = sK + buf * PF_BK * LDS;
    const __nv_bfloat16* cV = sV + buf * PF_BK * LDS;
    if (k0 >= q0 && k0 < q0 + PF_BQ) {   // this CTA appends key tile kt to the paged cache
      for (int i = tid; i < PF_BK * NV; i += PF_THREADS) {
        const int r = i / NV, c = (i % NV) * 8;
        const int p = k0 + r;
        if (p < s) {
          const int page = page_table[(int64_t)bi * max_pages + p / KVB];
          *reinterpret_cast<uint4*>(kv_pool + kv_off(page, 0, heads, head, p % KVB, D) + c) =
              *reinterpret_cast<const uint4*>(&cK[r * LDS + c]);
          *reinterpret_cast<uint4*>(kv_pool + kv_off(page, 1, heads, head, p % KVB, D) + c) =
              *reinterpret_cast<const uint4*>(&cV[r * LDS + c]);
        }
      }
    }
    if (k0 <= wrow0 + 15 && wrow0 < s) {   // warp-uniform: some key of this tile is visible to the warp
      float sc[8][4];
#pragma unroll
      for (int j = 0; j < 8; ++j) sc[j][0] = sc[j][1] = sc[j][2] = sc[j][3] = 0.f;
#pragma unroll
      for (int kc = 0; kc < D; kc += 16) {
        uint32_t a0, a1, a2, a3;
        const int ar = warp * 16 + (lane % 8) + ((lane / 8) % 2) * 8;
        const int ac = kc + (lane / 16) * 8;
        ldsm_x4(smem_u32(&sQ[ar * LDS + ac]), a0, a1, a2, a3);
#pragma unroll
        for (int nb = 0; nb < 8; nb += 2) {
          uint32_t b0, b1, b2, b3;
          const int br = nb * 8 + (lane % 8) + (lane / 16) * 8;
          const int bc = kc + ((lane / 8) % 2) * 8;
          ldsm_x4(smem_u32(&cK[br * LDS + bc]), b0, b1, b2, b3);
          mma_bf16_16816(sc[nb], a0, a1, a2, a3, b0, b1);
          mma_bf16_16816(sc[nb + 1], a0, a1, a2, a3, b2, b3);
        }
      }
      if (k0 + PF_BK - 1 > wrow0 || k0 + PF_BK > s) {   // diagonal / ragged tile: mask
#pragma unroll
        for (int nb = 0; nb < 8; ++nb) {
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const int key = k0 + nb * 8 + tig * 2 + (e & 1);
            const int row = row0 + (e >> 1) * 8;
            if (key > row || key >= s) sc[nb][e] = -INFINITY;
          }
        }
      }
#pragma unroll
      for (int h2 = 0; h2 < 2; ++h2) {
        float mx = -INFINITY;
#pragma unroll
        for (int nb = 0; nb < 8; ++nb) mx = fmaxf(mx, fmaxf(sc[nb][2 * h2], sc[nb][2 * h2 + 1]));
        mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 1));
        mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 2));
        const float m_new = fmaxf(m_r[h2], mx);
        const float corr = (m_new == -INFINITY) ? 1.f : exp2f((m_r[h2] - m_new) * L2E);
        float sum = 0.f;
#pragma unroll
        for (int nb = 0; nb < 8; ++nb) {
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const float v = sc[nb][2 * h2 + e];
            const float pv = (v == -INFINITY) ? 0.f : exp2f((v - m_new) * L2E);
            sc[nb][2 * h2 + e] = pv;
            sum += pv;
          }
        }
        sum += __shfl_xor_sync(0xffffffffu, sum, 1);
        sum += __shfl_xor_sync(0xffffffffu, sum, 2);
        l_r[h2] = l_r[h2] * corr + sum;
        m_r[h2] = m_new;
#pragma unroll
        for (int j = 0; j < D / 8; ++j) {
          acc[j][2 * h2] *= corr;
          acc[j][2 * h2 + 1] *= corr;
        }
      }
#pragma unroll
      for (int kc = 0; kc < 4; ++kc) {   // 16 keys per step
        const uint32_t a0 = pack_bf16(sc[2 * kc][0], sc[2 * kc][1]);
        const uint32_t a1 = pack_bf16(sc[2 * kc][2], sc[2 * kc][3]);
        const uint32_t a2 = pack_bf16(sc[2 * kc + 1][0], sc[2 * kc + 1][1]);
        const uint32_t a3 = pack_bf16(sc[2 * kc + 1][2], sc[2 * kc + 1][3]);
#pragma unroll
        for (int nb = 0; nb < D / 8; nb += 2) {
          uint32_t b0, b1, b2, b3;
          const int vr = kc * 16 + (lane % 8) + ((lane / 8) % 2) * 8;
          const int vc = nb * 8 + (lane / 16) * 8;
          ldsm_x4_t(smem_u32(&cV[vr * LDS + vc]), b0, b1, b2, b3);
          mma_bf16_16816(acc[nb], a0, a1, a2, a3, b0, b1);
          mma_bf16_16816(acc[nb + 1], a0, a1, a2, a3, b2, b3);
        }
      }
    }
    __syncthreads();   // buffer `buf` is refilled at iteration kt + 2
  }
  cp_async_wait<0>();
#pragma unroll
  for (int h2 = 0; h2 < 2; ++h2) {
    const int row = row0 + h2 * 8;
    if (row < s) {
      const float inv = 1.0f / l_r[h2];
      __nv_bfloat16* orow = o + ((int64_t)bi * s + row) * ((int64_t)heads * D) + head * D;
#pragma unroll
      for (int nb = 0; nb < D / 8; ++nb) {
        const int c = nb * 8 + tig * 2;
        *reinterpret_cast<__nv_bfloat162*>(orow + c) =
            __floats2bfloat162_rn(acc[nb][2 * h2] * inv, acc[nb][2 * h2 + 1] * inv);
      }
    }
  }
}

int attn_prefill_launch(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                        int s, int heads, int d, cudaStream_t stream) {
  if (b <= 0 || s <= 0) return 0;
  dim3 grid((s + PF_BQ - 1) / PF_BQ, heads, b);
  const size_t smem = (size_t)(PF_BQ + 4 * PF_BK) * (d + 8) * 2;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_prefill_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (PF_BQ + 4 * PF_BK) * (128 + 8) * 2);
    cudaFuncSetAttribute(attn_prefill_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (PF_BQ + 4 * PF_BK) * (64 + 8) * 2);
    attr = true;
  }
  int rc;
  if (d == 128)
    rc = launch_pdl(attn_prefill_kernel<128>, grid, dim3(PF_THREADS), smem, stream, (const __nv_bfloat16*)qkv,
                    (__nv_bfloat16*)o, (__nv_bfloat16*)kv_pool, page_table, max_pages, s, heads);
  else if (d == 64)
    rc = launch_pdl(attn_prefill_kernel<64>, grid, dim3(PF_THREADS), smem, stream, (const __nv_bfloat16*)qkv,
                    (__nv_bfloat16*)o, (__nv_bfloat16*)kv_pool, page_table, max_pages, s, heads);
  else
    return LIGER_EINVAL;
  return rc ? LIGER_ECUDA : 0;
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
  float st_acc[4 * (32 / (D / 8))][D];     // per lane group: acc (item merge)
  float st_m[4 * (32 / (D / 8))], st_l[4 * (32 / (D / 8))];
  float mw[DC_MAX_SPLITS], lw[DC_MAX_SPLITS];
  uint64_t full[DC_NS], empty[DC_NS];
  int last;
};

// Warps 0..3 compute, warp 4 (lane 0) is the producer: it walks the same task list
// (chunk j of item i = blockIdx.x + k G) and keeps DC_NS chunks in flight, refilling a
// stage as soon as the four compute warps have released it (empty[s]).
template <int D>
__global__ void __launch_bounds__(DC_THREADS + 32) attn_decode_kernel(const DecAttnArgs a) {
  constexpr int LPT = D / 8;          // lanes per token row (16 B each)
  constexpr int TPW = 32 / LPT;       // token rows per warp step
  constexpr int NG = 4 * TPW;         // lane groups per CTA
  constexpr int PPG = DC_CH / NG;     // positions per lane group per chunk
  const uint64_t tr0 = trace_now();
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
      mbar_init(&sm.empty[s], 4);   // one arrive per compute warp
    }
    fence_barrier_init();
  }
  __syncthreads();
  if (warp == 4) {
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
  preload_kernel(attn_prefill_kernel<64>);
  preload_kernel(attn_prefill_kernel<128>);
  preload_kernel(attn_decode_kernel<64>);
  preload_kernel(attn_decode_kernel<128>);
}

LIGER_TRACE_SETTER(attention)

}  // namespace liger
