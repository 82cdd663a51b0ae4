// Prefill causal attention on the 5th-generation tensor cores (
// PAPER.md P:316; PAPER's "Attention" block of Fig. 2 / the KV cache it fills).
//
// CTA = (128-query tile, head, sequence), 192 threads:
//   warp 0 (one lane) -- TMA producer: the Q tile once, then 128-key blocks of K and V
//     (two stages) straight from the QKV GEMM's output rows (a 2-D tensor map over
//     qkv [b*s, 3*heads*d], 64 x 128 boxes, 128-byte swizzle);
//   warp 1 (one lane) -- MMA issuer: S = Q K^T (M = 128 queries, N = 128 keys, K = d)
//     into TMEM columns [0, 128), then O_j = P V (M = 128, N = d, K = 128 keys; V is
//     the MN-major B operand, d contiguous) into TMEM columns [128, 128 + d);
//   warps 2..5 -- softmax: thread r owns query row r (TMEM lane r); two passes over
//     its S row (row max, then p = 2^((s - m) log2 e) written as bf16 into the
//     swizzled P tile the PV MMA reads from shared memory), online rescaling of the
//     output row kept in registers (O = alpha O + O_j), 1 / l at the end.
// While it turns the diagonal block (key block == query tile) into P, the softmax
// group also appends those keys' K / V rows from shared memory to the paged cache.  q is pre-scaled by 1 / sqrt(d) (the QKV
// GEMM epilogue); causal mask key <= query, keys >= s masked.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include "attn_decode.cuh"
#include "common.cuh"

namespace liger {

constexpr int PT_BQ = 128, PT_BK = 128, PT_THREADS = 192;

template <int D>
struct PtSmem {
  static constexpr int BOX = 128 * 64 * 2;           // one 64-column box of 128 rows (16 KiB)
  static constexpr int NB = D / 64;                   // boxes per row block
  static constexpr int Q0 = 0;                        // Q buffer q at Q0 + q * NB * BOX (two)
  static constexpr int K0 = Q0 + 2 * NB * BOX;        // K stage s at K0 + s * NB * BOX
  static constexpr int V0 = K0 + 2 * NB * BOX;
  static constexpr int P = V0 + 2 * NB * BOX;         // 128 x 128 bf16 = 2 boxes
  static constexpr int BARS = P + 2 * BOX;
  static constexpr int BYTES = BARS + 128;            // + barriers / TMEM slot
  static constexpr int ALLOC = BYTES + 1024;          // 1024-B alignment slack
};

LIGER_DEV void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
LIGER_DEV float ex2_approx(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// 32 lanes x 32 bit, 16 consecutive columns per thread, TMEM <- registers.
LIGER_DEV void tmem_st_32x32b_x16(uint32_t taddr, const uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
          taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
      : "memory");
}
LIGER_DEV void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// UMMA descriptor, 128-byte swizzle, MN-major operand (the contiguous dimension is
// N): lbo = bytes between 64-element column blocks, sbo = bytes between 8-row groups.
LIGER_DEV uint64_t umma_desc_sw128_mn(uint32_t smem_addr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((smem_addr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

template <int D>
__global__ void __launch_bounds__(PT_THREADS, 1)
    attn_prefill_tc_kernel(const __grid_constant__ CUtensorMap tm, __nv_bfloat16* __restrict__ o,
                           __nv_bfloat16* __restrict__ kv_pool,
                           const int32_t* __restrict__ page_table, int max_pages, int b, int s, int heads) {
  using L = PtSmem<D>;
  const TraceStart tr0 = trace_begin();
  extern __shared__ uint8_t pt_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(pt_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + L::BARS);
  uint64_t* q_full = bars + 0;     // [2]
  uint64_t* q_empty = bars + 2;    // [2]
  uint64_t* kv_full = bars + 4;    // [2]
  uint64_t* kv_empty = bars + 6;   // [2]
  uint64_t* s_full = bars + 8;
  uint64_t* s_free = bars + 9;
  uint64_t* p_full = bars + 10;
  uint64_t* o_full = bars + 11;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 12);

  // Persistent: item i = (query tile, sequence, head), longest query tiles first;
  // CTA c takes items c, c + G, ...  The producer runs up to two items ahead (Q
  // double-buffered), so an item's loads and the next item's S = Q K^T overlap the
  // previous item's softmax tail and output stores.
  const int nqt = (s + PT_BQ - 1) / PT_BQ;
  const int n_items = nqt * b * heads;
  const int G = gridDim.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  auto item_of = [&](int i, int* qt, int* bi, int* head) {
    *head = i % heads;
    *bi = (i / heads) % b;
    *qt = nqt - 1 - i / (heads * b);
  };

  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&q_full[i], 1);
      mbar_init(&q_empty[i], 1);
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
    }
    mbar_init(s_full, 1);
    mbar_init(s_free, 128);
    mbar_init(p_full, 128);
    mbar_init(o_full, 1);
    fence_barrier_init();
  }
  if (warp == 0 && lane == 0) tma_prefetch_desc(&tm);
  if (warp == 1) tmem_alloc(tmem_slot, 256);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t tS = tmem, tO = tmem + 128;
  pdl_enter();   // Q / K / V come from the QKV GEMM
  const uint64_t tr1 = trace_now();

  if (warp == 0) {
    if (lane == 0) {
      int g = 0, it = 0;
      for (int i = blockIdx.x; i < n_items; i += G, ++it) {
        int qt, bi, head;
        item_of(i, &qt, &bi, &head);
        const int row_base = bi * s;
        const int cq = head * D, ck = heads * D + head * D, cv = 2 * heads * D + head * D;
        const int qb = it & 1;
        if (it >= 2) mbar_wait(&q_empty[qb], ((it >> 1) - 1) & 1);
        mbar_arrive_expect_tx(&q_full[qb], L::NB * L::BOX);
        for (int c = 0; c < L::NB; ++c)
          tma_load_2d(sm + L::Q0 + (qb * L::NB + c) * L::BOX, &tm, &q_full[qb], cq + c * 64, row_base + qt * PT_BQ);
        for (int j = 0; j <= qt; ++j, ++g) {
          const int st = g & 1;
          if (g >= 2) mbar_wait(&kv_empty[st], ((g >> 1) - 1) & 1);
          mbar_arrive_expect_tx(&kv_full[st], 2 * L::NB * L::BOX);
          for (int c = 0; c < L::NB; ++c) {
            tma_load_2d(sm + L::K0 + (st * L::NB + c) * L::BOX, &tm, &kv_full[st], ck + c * 64, row_base + j * PT_BK);
            tma_load_2d(sm + L::V0 + (st * L::NB + c) * L::BOX, &tm, &kv_full[st], cv + c * 64, row_base + j * PT_BK);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // kind::f16, D = f32, A = B = bf16, M = 128; S: N = 128, both K-major;
      // PV: N = D, B (V) MN-major (bit 16).  Order S_0, S_1, PV_0, S_2, PV_1, ...: the
      // next block's S = Q K^T runs while the softmax warps turn this block's S into P.
      const uint32_t id_s = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(PT_BK >> 3) << 17) | ((128u >> 4) << 24);
      const uint32_t id_pv =
          (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(D >> 3) << 17) | ((128u >> 4) << 24);
      const uint32_t sP = smem_u32(sm + L::P);
      int g = 0, it = 0;
      bool prev_first = false;
      auto issue_pv = [&](int gp, bool first) {   // O (+)= P V of block gp
        const int st = gp & 1;
        const uint32_t sV = smem_u32(sm + L::V0 + st * L::NB * L::BOX);
        mbar_wait(p_full, gp & 1);
        tc_fence_after();
#pragma unroll
        for (int k = 0; k < PT_BK / 16; ++k) {
          const uint64_t pd = umma_desc_sw128(sP + (k >> 2) * L::BOX + (k & 3) * 32);
          const uint64_t vd = umma_desc_sw128_mn(sV + k * 16 * 128, L::BOX, 1024);
          umma_bf16(tO, pd, vd, id_pv, (!first || k > 0) ? 1u : 0u);
        }
        umma_commit(o_full);
        umma_commit(&kv_empty[st]);
      };
      for (int i = blockIdx.x; i < n_items; i += G, ++it) {
        int qt, bi, head;
        item_of(i, &qt, &bi, &head);
        const int qb = it & 1;
        const uint32_t sQ = smem_u32(sm + L::Q0 + qb * L::NB * L::BOX);
        mbar_wait(&q_full[qb], (it >> 1) & 1);
        for (int j = 0; j <= qt; ++j, ++g) {
          const int st = g & 1;
          mbar_wait(&kv_full[st], (g >> 1) & 1);
          if (g >= 1) mbar_wait(s_free, (g - 1) & 1);   // softmax has read the previous S
          tc_fence_after();
          const uint32_t sK = smem_u32(sm + L::K0 + st * L::NB * L::BOX);
#pragma unroll
          for (int k = 0; k < D / 16; ++k) {
            const uint32_t off = (k >> 2) * L::BOX + (k & 3) * 32;
            umma_bf16(tS, umma_desc_sw128(sQ + off), umma_desc_sw128(sK + off), id_s, k > 0);
          }
          umma_commit(s_full);
          if (j == qt) umma_commit(&q_empty[qb]);   // the item's last read of its Q tile
          if (g >= 1) issue_pv(g - 1, prev_first);
          prev_first = j == 0;
        }
      }
      if (g >= 1) issue_pv(g - 1, prev_first);
    }
  } else {
    // ---------------- softmax warps: TMEM lane quadrant = warp % 4.  The output row
    // accumulates in TMEM (PV MMAs with accumulate); it is rescaled only when the row
    // max grows by more than 2^8 (p = 2^((s - m) log2 e) <= 256 otherwise: exact in
    // fp32, the same normaliser l divides it at the end).
    const int row = (warp & 3) * 32 + lane;
    const uint32_t lane_off = (uint32_t)((warp & 3) * 32) << 16;
    const float L2E = 1.4426950408889634f;
    uint8_t* prow = sm + L::P + row * 128;
    int g = 0;
    for (int i = blockIdx.x; i < n_items; i += G) {
      int qt, bi, head;
      item_of(i, &qt, &bi, &head);
      const int row_base = bi * s;
      const int qrow = qt * PT_BQ + row;
      float mu = -INFINITY, l = 0.f;   // mu: the max the exponents are taken against
      for (int j = 0; j <= qt; ++j, ++g) {
        const int kmax = min(qrow, s - 1) - j * PT_BK;   // keys j*128 + c, c <= kmax, are visible
        mbar_wait(s_full, g & 1);
        tc_fence_after();
        uint32_t r[PT_BK];
#pragma unroll
        for (int c0 = 0; c0 < PT_BK; c0 += 16) tmem_ld_32x32b_x16(tS + lane_off + c0, *reinterpret_cast<uint32_t(*)[16]>(&r[c0]));
        tmem_ld_wait();
        tc_fence_before();
        mbar_arrive(s_free);   // S may be overwritten by the next block's Q K^T
        if (j == qt) {
          // diagonal block: append its keys (this tile's positions) to the paged cache
          // from the K / V stage, which stays loaded until this block's PV completes
          // (16-byte chunk c of row r in a 64-column box at (c ^ (r % 8)) * 16)
          constexpr int CH = D / 8, RPI = 128 / CH;
          const uint8_t* sK = sm + L::K0 + (g & 1) * L::NB * L::BOX;
          const uint8_t* sV = sm + L::V0 + (g & 1) * L::NB * L::BOX;
#pragma unroll 4
          for (int it2 = 0; it2 < CH; ++it2) {
            const int r = it2 * RPI + row / CH, c = row % CH;
            const int qr = qt * PT_BQ + r;
            if (qr < s) {
              const int page = page_table[(int64_t)bi * max_pages + qr / KVB];
              const int so = (c >> 3) * L::BOX + r * 128 + (((c & 7) ^ (r & 7)) << 4);
              reinterpret_cast<uint4*>(kv_pool + kv_off(page, 0, heads, head, qr % KVB, D))[c] =
                  *reinterpret_cast<const uint4*>(sK + so);
              reinterpret_cast<uint4*>(kv_pool + kv_off(page, 1, heads, head, qr % KVB, D))[c] =
                  *reinterpret_cast<const uint4*>(sV + so);
            }
          }
        }
        float mx = -INFINITY;
#pragma unroll
        for (int e = 0; e < PT_BK; ++e)
          if (e <= kmax) mx = fmaxf(mx, __uint_as_float(r[e]));
        float alpha = 1.f;
        bool rescale = false;   // warp-uniform: tcgen05.ld / st are warp-collective
        if (j == 0) {
          mu = mx;
        } else if (__any_sync(0xffffffffu, (mx - mu) * L2E > 8.f)) {
          if (mx > mu) {
            alpha = ex2_approx((mu - mx) * L2E);
            mu = mx;
          }
          rescale = true;
        }
        if (g >= 1) {   // the previous block's PV is done: P is free, O is current
          mbar_wait(o_full, (g - 1) & 1);
          tc_fence_after();
        }
        if (rescale) {
#pragma unroll
          for (int c0 = 0; c0 < D; c0 += 16) {
            uint32_t t[16];
            tmem_ld_32x32b_x16(tO + lane_off + c0, t);
            tmem_ld_wait();
#pragma unroll
            for (int e = 0; e < 16; ++e) t[e] = __float_as_uint(__uint_as_float(t[e]) * alpha);
            tmem_st_32x32b_x16(tO + lane_off + c0, t);
          }
          tmem_st_wait();
        }
        const float mb = mu * L2E;
        float sum = 0.f;
#pragma unroll
        for (int c0 = 0; c0 < PT_BK; c0 += 8) {
          uint32_t pk[4];
#pragma unroll
          for (int e = 0; e < 8; e += 2) {
            const float p0 = (c0 + e <= kmax) ? ex2_approx(fmaf(__uint_as_float(r[c0 + e]), L2E, -mb)) : 0.f;
            const float p1 = (c0 + e + 1 <= kmax) ? ex2_approx(fmaf(__uint_as_float(r[c0 + e + 1]), L2E, -mb)) : 0.f;
            sum += p0 + p1;
            __nv_bfloat162 h2 = __floats2bfloat162_rn(p0, p1);
            pk[e >> 1] = *reinterpret_cast<uint32_t*>(&h2);
          }
          // chunk c of 8 keys in a 64-key box lives at (c ^ (row & 7)) * 16 (128-B swizzle)
          const int box = c0 >> 6, chunk = (c0 & 63) >> 3;
          *reinterpret_cast<uint4*>(prow + box * L::BOX + ((chunk ^ (row & 7)) << 4)) =
              make_uint4(pk[0], pk[1], pk[2], pk[3]);
        }
        l = l * alpha + sum;
        tc_fence_before();
        fence_proxy_async_smem();   // P (generic stores) -> the PV MMA (async proxy)
        mbar_arrive(p_full);
      }
      // the item's output row: O / l once its last PV is done, staged through the (now
      // free) P tile as bf16 rows (16-byte chunk c of row r at c ^ (r % 16)), then
      // written out row-contiguously by the 128 threads together
      mbar_wait(o_full, (g - 1) & 1);
      tc_fence_after();
      constexpr int CH = D / 8;           // 16-byte chunks per row
      constexpr int RPI = 128 / CH;       // rows per pass of the 128 threads
      uint8_t* stage = sm + L::P;
      const float inv = 1.0f / l;
#pragma unroll
      for (int c0 = 0; c0 < D; c0 += 16) {
        uint32_t t[16];
        tmem_ld_32x32b_x16(tO + lane_off + c0, t);
        tmem_ld_wait();
#pragma unroll
        for (int hc = 0; hc < 2; ++hc) {
          __nv_bfloat162 h[4];
#pragma unroll
          for (int e = 0; e < 4; ++e)
            h[e] = __floats2bfloat162_rn(__uint_as_float(t[8 * hc + 2 * e]) * inv,
                                         __uint_as_float(t[8 * hc + 2 * e + 1]) * inv);
          const int c = (c0 >> 3) + hc;
          *reinterpret_cast<uint4*>(stage + row * (D * 2) + ((c ^ (row & 15) & (CH - 1)) << 4)) =
              *reinterpret_cast<uint4*>(h);
        }
      }
      tc_fence_before();
      named_bar_sync(1, 128);
      const int tid = row;                 // 0..127 within the softmax warps
      const int q0 = qt * PT_BQ;
#pragma unroll 4
      for (int it2 = 0; it2 < CH; ++it2) {
        const int r = it2 * RPI + tid / CH, c = tid % CH;
        const int qr = q0 + r;
        if (qr < s) {
          const int64_t grow = (int64_t)row_base + qr;
          reinterpret_cast<uint4*>(o + grow * ((int64_t)heads * D) + head * D)[c] =
              *reinterpret_cast<const uint4*>(stage + r * (D * 2) + ((c ^ (r & 15) & (CH - 1)) << 4));
        }
      }
      named_bar_sync(1, 128);   // the staging tile is the next item's P
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, 256);
  }
  if (threadIdx.x == 0) trace_write(TK_ATTN_PRE, tr0, tr1);
}

}  // namespace liger
