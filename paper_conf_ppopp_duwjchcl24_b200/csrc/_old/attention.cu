// Attention over the paged KV cache (PAPER.md P:316 KV cache).
//
// Paged pool layout: [n_pages][2 (K,V)][heads][16 tokens][d] bf16; a sequence's
// page_table row maps token position p to page page_table[p / 16].
//
//  * prefill: flash-style causal attention with bf16 tensor-core mma.sync
//    (m16n8k16, fp32 accumulate), 64 queries x 64 keys per step, online
//    softmax in registers; the CTA on the diagonal tile also writes that key
//    tile's K/V into the cache pages.
//  * decode: one query per sequence; split over the context in fixed chunks
//    of 256 positions (a function of ctx only), two-pass softmax per chunk
//    with warp-shuffle dot products, deterministic merge of the chunk partials
//    in chunk order by the last CTA to finish.
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>

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
// CTA = (head, sequence, chunk of DC_CHUNK positions), 128 threads.  Thread 0
// stages the chunk's K and V page blocks (16 tokens x d bf16 = 4 KiB each,
// contiguous in the paged pool) into shared memory with cp.async.bulk (TMA bulk
// engine), all issued at once on one mbarrier, so a CTA pays one DRAM round
// trip.  The new token (position pos) is taken from the qkv buffer (and
// appended to its page by the last chunk's CTA).  Phase 1: warp w scores
// positions [32w, 32w+32) (a token row spread over d/8 lanes, shuffle dot
// products); two-pass softmax over the chunk; phase 2: thread (slot, vec)
// accumulates p_t V[t] over positions t = slot (mod SLOTS).  Chunks of one
// (sequence, head) are merged in chunk order by the last CTA (deterministic).
size_t attn_decode_workspace_bytes(int b, int heads, int d, int ctx) {
  const int ns = (ctx + DC_CHUNK_MIN - 1) / DC_CHUNK_MIN;   // worst case (32-position chunks)
  return ATTN_COUNTER_BYTES + (size_t)b * heads * ns * (d + 2) * sizeof(float);
}

struct CtaSync {
  __device__ __forceinline__ void operator()() const { __syncthreads(); }
};

// One CTA per work item (head, sequence, chunk); see attn_decode.cuh.
template <int D, int DC_CHUNK>
__global__ void __launch_bounds__(DC_THREADS) attn_decode_kernel(const DecAttnArgs a) {
  constexpr int SLOTS = DecAttnSmem<D, DC_CHUNK>::SLOTS;
  const uint64_t tr0 = trace_now();
  extern __shared__ __align__(128) uint8_t dsm[];
  __shared__ float sc[DC_CHUNK];
  __shared__ float red[DC_THREADS / 32];
  __shared__ float part[SLOTS * D];
  __shared__ float mw[DC_MAX_SPLITS], lw[DC_MAX_SPLITS];
  __shared__ __align__(8) uint64_t bar;
  __shared__ int last;
  DecAttnSmem<D, DC_CHUNK> sm;
  sm.sK = reinterpret_cast<__nv_bfloat16*>(dsm);
  sm.sV = sm.sK + DC_CHUNK * D;
  sm.bar = &bar;
  sm.sc = sc;
  sm.red = red;
  sm.part = part;
  sm.mw = mw;
  sm.lw = lw;
  sm.last = &last;
  const int head = blockIdx.x, bi = blockIdx.y, sp = blockIdx.z, nsp = gridDim.z;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    fence_barrier_init();
  }
  __syncthreads();
  // The cached positions (< pos) were written by earlier passes, and the page
  // table at admission: staging them does not depend on the preceding kernel
  // (QKV), so it is issued before griddepcontrol.wait.
  if (threadIdx.x < 32) dec_attn_issue<D, DC_CHUNK>(a, head, bi, sp, sm.sK, sm.sV, &bar, threadIdx.x);
  pdl_enter();   // q and the new token's k / v come from the QKV kernel
  const uint64_t tr1 = trace_now();
  dec_attn_partial<D, DC_CHUNK>(a, head, bi, sp, nsp, sm, 0, threadIdx.x, CtaSync{});
  bool merged = false;
  if (nsp > 1) {   // the last chunk of (sequence, head) to finish merges (acq_rel counter)
    const int64_t unit = (int64_t)bi * a.heads + head;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) {
      int prev;
      asm volatile("atom.add.acq_rel.gpu.global.s32 %0, [%1], 1;" : "=r"(prev) : "l"(&a.counters[unit]) : "memory");
      last = (prev == nsp - 1);
    }
    __syncthreads();
    if (last) {
      dec_attn_merge<D, DC_CHUNK>(a, head, bi, nsp, sm, threadIdx.x, CtaSync{});
      if (threadIdx.x == 0) a.counters[unit] = 0;
      merged = true;
    }
  }
  if (threadIdx.x == 0) trace_write(merged ? (TK_ATTN_DEC | 0x100) : TK_ATTN_DEC, tr0, tr1);
}

template <int D, int CH>
static int launch_decode(const DecAttnArgs& a, int b, cudaStream_t stream) {
  const int ns = (a.pos + 1 + CH - 1) / CH;
  const size_t dsmem = (size_t)2 * CH * D * 2;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_decode_kernel<D, CH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem);
    attr = true;
  }
  return launch_pdl(attn_decode_kernel<D, CH>, dim3(a.heads, b, ns), dim3(DC_THREADS), dsmem, stream, a);
}

int attn_decode_launch(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                       int pos, int heads, int d, void* workspace, size_t ws_bytes, cudaStream_t stream) {
  if (b <= 0) return 0;
  const int ctx = pos + 1;
  int CH = dec_attn_chunk(b, heads, ctx);
  static const int ch_env = getenv("LIGER_ATTN_CHUNK") ? atoi(getenv("LIGER_ATTN_CHUNK")) : 0;   // experiments
  if ((ch_env == 32 || ch_env == 64 || ch_env == 128) && (ctx + ch_env - 1) / ch_env <= DC_MAX_SPLITS) CH = ch_env;
  const int ns = (ctx + CH - 1) / CH;
  if (ns > DC_MAX_SPLITS) return LIGER_EINVAL;   // context longer than 4096 positions
  if (ns > 1) {
    if (!workspace || ws_bytes < attn_decode_workspace_bytes(b, heads, d, ctx) ||
        (size_t)b * heads * 4 > ATTN_COUNTER_BYTES)
      return LIGER_EINVAL;
  }
  DecAttnArgs a;
  a.qkv = (const __nv_bfloat16*)qkv;
  a.o = (__nv_bfloat16*)o;
  a.kv_pool = (__nv_bfloat16*)kv_pool;
  a.page_table = page_table;
  a.max_pages = max_pages;
  a.pos = pos;
  a.heads = heads;
  a.counters = (int*)workspace;
  a.ws = workspace ? (float*)((char*)workspace + ATTN_COUNTER_BYTES) : nullptr;
  int rc;
  if (d == 128)
    rc = CH == 32 ? launch_decode<128, 32>(a, b, stream)
                  : CH == 64 ? launch_decode<128, 64>(a, b, stream) : launch_decode<128, 128>(a, b, stream);
  else if (d == 64)
    rc = CH == 32 ? launch_decode<64, 32>(a, b, stream)
                  : CH == 64 ? launch_decode<64, 64>(a, b, stream) : launch_decode<64, 128>(a, b, stream);
  else
    return LIGER_EINVAL;
  return rc ? LIGER_ECUDA : 0;
}

LIGER_TRACE_SETTER(attention)

}  // namespace liger
