// Fused decode pass: every decoder layer of one decode step of one batch in ONE
// persistent kernel (sm_100a).  SURVEY §8(a) rows a2-a11 for M = b <= 32 tokens at
// t = 1 (no all-reduce between the compute runs; PAPER.md P:149 -- with one
// device the interleaving scheduler degenerates to the serial order, so a whole
// decode pass is a single compute run).
//
// Why: a decode layer streams 12 h^2 / t bf16 weights from HBM and does almost
// nothing else.  As separate kernels (LN1, QKV, attention, out-proj, split-K
// fixup, LN2, FC1, fixup, FC2, fixup) each hand-off costs ~1.3 us of grid drain +
// PDL release and each small kernel 2-5 us of pure latency; the in-kernel
// %globaltimer trace of an OPT-13B layer (b = 2) showed ~40 of 136 us lost that
// way while the GEMMs themselves streamed at 6.8 TB/s.  Here the weight stream
// never stops: a producer warp keeps TMA-loading the next GEMM's weight blocks
// into the shared-memory ring while the other warps run the latency-bound phases.
//
// Phases of layer l (global phase index k = 7 l + p):
//   p0 LN1   x = x + part + b_2(l-1) (nothing at the range's first layer); y = LN(x)
//   p1 QKV   qkv = y W_qkv^T + b_qkv, q columns * d^-1/2
//   p2 ATTN  attn = softmax(q K^T) V over the paged cache (+ append k, v of pos)
//   p3 OUT   part = attn W_o^T
//   p4 LN2   x = x + part + b_o; y = LN(x)
//   p5 FC1   hbuf = act(y W_1^T + b_1)
//   p6 FC2   part = hbuf W_2^T           (b_2 and the residual: next layer's p0 / the LM head)
//
// Grid = one CTA per SM (persistent).  Warp roles (256 threads):
//   warp 0  weight producer: TMA of W blocks into the ring, never waits on data
//   warp 1  TMEM allocator + single-thread tcgen05.mma issuer
//   warp 2  activation producer: waits for phase k-1, then TMA of the X blocks
//   warp 3  idle
//   warps 4-7 workers: GEMM epilogues (tcgen05.ld; fp32 split partials, the last
//           split of a tile to arrive reduces it in z order), LayerNorm rows,
//           attention items (double-buffered cp.async.bulk KV staging).
// Cross-CTA ordering: one 64-bit counter; a CTA's workers add 1 (release) after
// each phase, and only once the counter shows every phase before it complete, so
// counter >= base + G k  <=>  phases 0..k-1 are complete everywhere.
//
// Bit-exactness: the split plan (gemm_plan), the MMA K order, the z-order split
// reduction and epilogue, the LayerNorm reduction tree (emulating add_ln_kernel's
// NT-thread tree with 128 threads) and the attention item code (attn_decode.cuh)
// are those of the per-kernel path, so the fused pass reproduces its bits (tested).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>

#include <vector>

#include "attn_decode.cuh"
#include "common.cuh"
#include "kernels.h"

namespace liger {

namespace {

constexpr int FD_THREADS = 256;
constexpr int FD_BM = 128, FD_BK = 64;
constexpr int FD_A_BYTES = FD_BM * FD_BK * 2;
constexpr int FD_ACC_COLS = 32;   // TMEM columns per accumulator stage (bn <= 32)
constexpr int FD_TS = 4;          // accumulator stages
constexpr int FD_MAX_TILES = 2048;   // tile counters in the workspace's counter region
constexpr int FD_PHASES = 7;
constexpr int FD_MAX_SMEM = 227 * 1024;
constexpr int FD_MAX_LAYERS = 96;   // layers per launch: their weight descriptors live in constant memory

// Weight TMA descriptors [layer][QKV, OUT, FC1, FC2].  Constant (or param) space:
// with the descriptors in global memory every TMA load paid a descriptor fetch
// (~1 us per 16 KiB block, measured), i.e. no pipelining at all.
__constant__ CUtensorMap c_wmap[FD_MAX_LAYERS * 4];

struct FGemm {
  int N, K, splits, kcb, tiles, units, nkb;
  int scale_cols, act;
  float scale;
  void* out;
  int64_t ldo;
};

struct FLayer {
  const __nv_bfloat16 *b_qkv, *b_o, *b_1, *b_2, *g1, *be1, *g2, *be2;
};

struct FParams {
  int L, M, h, heads, d, bn, S, G, pos, nsp, first_no_add;
  int ln_nt;           // add_ln_kernel's thread count for this h (its reduction tree)
  int stage_bytes;     // KV / LayerNorm staging region (bytes)
  int nbuf;            // attention items staged ahead (KV buffers)
  float eps;
  FGemm gm[4];         // QKV, OUT, FC1, FC2
  int units_layer;     // sum of the four GEMMs' units
  const FLayer* layers;      // [L]
  __nv_bfloat16 *x, *y, *part;
  __nv_bfloat16* kv;
  int64_t kv_layer_elems;
  DecAttnArgs attn;    // per-layer kv_pool is offset in the kernel
  float* ws;           // split partials
  int* tile_cnt;       // [FD_MAX_TILES]
  unsigned long long* sync;
  unsigned long long sync_base;
};

__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_release_add_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
// Spin until *p >= target (single thread): relaxed polling (an acquire per poll would
// invalidate the SM's L1 each time), one acquire fence once satisfied.  Traps after
// ~2 s instead of hanging the GPU.
__device__ __forceinline__ void wait_counter(const unsigned long long* p, unsigned long long target) {
  if (ld_relaxed_u64(p) < target) {
    const uint64_t t0 = trace_now();
    while (ld_relaxed_u64(p) < target) {
      __nanosleep(100);
      if (trace_now() - t0 > 2000000000ull) __trap();
    }
  }
  asm volatile("fence.acq_rel.gpu;" ::: "memory");
}
__device__ __forceinline__ void worker_sync() { named_bar_sync(1, 128); }
struct WorkerSync {
  __device__ __forceinline__ void operator()() const { named_bar_sync(1, 128); }
};

__device__ __forceinline__ float fd_epi(const FGemm& g, float v, int n, float bias_v) {
  v += bias_v;
  if (n < g.scale_cols) v *= g.scale;
  if (g.act == LIGER_ACT_RELU) v = fmaxf(v, 0.0f);
  else if (g.act == LIGER_ACT_GELU_TANH) v = gelu_tanh_f(v);
  return v;
}

// global phase index of GEMM g in a layer
__device__ __forceinline__ int gemm_phase(int g) { return g == 0 ? 1 : (g == 1 ? 3 : (g == 2 ? 5 : 6)); }

// first unit of GEMM g of layer l owned by CTA `cta` (units u = first, first + G, ...)
__device__ __forceinline__ int first_unit(const FParams& p, int l, int g, int cta) {
  int off = (int)(((long long)l * p.units_layer) % p.G);
  for (int i = 0; i < g; ++i) off += p.gm[i].units;
  off %= p.G;
  return ((cta - off) % p.G + p.G) % p.G;
}

// The weight blocks this CTA streams, in order: layer, GEMM, its units, K blocks.
struct WCursor {
  int l, g, u, kb, kb1;
  bool done;
  __device__ __forceinline__ void settle(const FParams& p, int cta) {
    while (true) {
      if (l >= p.L) {
        done = true;
        return;
      }
      const FGemm& gm = p.gm[g];
      if (u < gm.units) {
        kb = (u % gm.splits) * gm.kcb;
        kb1 = min(gm.nkb, kb + gm.kcb);
        return;
      }
      if (++g == 4) {
        g = 0;
        ++l;
      }
      if (l < p.L) u = first_unit(p, l, g, cta);
    }
  }
  __device__ __forceinline__ void init(const FParams& p, int cta) {
    l = 0;
    g = 0;
    done = false;
    u = first_unit(p, 0, 0, cta);
    settle(p, cta);
  }
  __device__ __forceinline__ void next(const FParams& p, int cta) {
    if (++kb < kb1) return;
    u += p.G;
    settle(p, cta);
  }
  __device__ __forceinline__ int tile(const FParams& p) const { return u / p.gm[g].splits; }
};

// ---------------------------------------------------------------- LayerNorm row
// x_row <- bf16(x + add + bias) (when add != null); y_row = LN(x_row) * gamma + beta,
// reproducing add_ln_kernel<NT, *>'s arithmetic and reduction tree with 128 threads:
// real warp w holds virtual warps w*VPT .. w*VPT+VPT-1 of the NT-thread block.
// One memory round trip: thread 0 bulk-copies the row, its addend, the bias, gamma
// and beta (h bf16 each) into shared memory (stg); no register arrays (with 227 KB of
// shared memory carved out, a register spill would cost an L2 round trip).
__device__ __forceinline__ void ln_row(__nv_bfloat16* px, __nv_bfloat16* py, int h, int nt, float eps, int row,
                                       const __nv_bfloat16* add, const __nv_bfloat16* add_bias,
                                       const __nv_bfloat16* gamma, const __nv_bfloat16* beta, float* red,
                                       uint4* stg, uint64_t* lnbar, uint32_t parity, int tid) {
  const int nv = h >> 3, vpt = nt / 128;
  const int warp = tid >> 5, lane = tid & 31;
  uint4* sX = stg;          // the row; becomes bf16(x + add + bias)
  uint4* sA = sX + nv;
  uint4* sB = sA + nv;
  uint4* sG = sB + nv;
  uint4* sBe = sG + nv;
  if (tid == 0) {
    fence_proxy_async_global();   // x / add were written by other CTAs' generic stores (acquired)
    fence_proxy_async_smem();     // stg was read / written by generic accesses before
    const uint32_t rb = (uint32_t)h * 2;
    mbar_arrive_expect_tx(lnbar, rb * (add ? 5 : 3));
    bulk_load(sX, px + (int64_t)row * h, rb, lnbar);
    if (add) {
      bulk_load(sA, add + (int64_t)row * h, rb, lnbar);
      bulk_load(sB, add_bias, rb, lnbar);
    }
    bulk_load(sG, gamma, rb, lnbar);
    bulk_load(sBe, beta, rb, lnbar);
  }
  mbar_wait(lnbar, parity);
  uint4* xr = reinterpret_cast<uint4*>(px + (int64_t)row * h);
  for (int i = 0; i < vpt; ++i) {
    const int t = (warp * vpt + i) * 32 + lane;   // virtual thread
    float s = 0.f;
    for (int v = t; v < nv; v += nt) {
      float r[8];
      bf16x8_to_f32(sX[v], r);
      if (add) {
        float a[8];
        bf16x8_to_f32(sA[v], a);
#pragma unroll
        for (int e = 0; e < 8; ++e) r[e] += a[e];
        bf16x8_to_f32(sB[v], a);
#pragma unroll
        for (int e = 0; e < 8; ++e) r[e] += a[e];
        uint4 pk;
        __nv_bfloat162* ph = reinterpret_cast<__nv_bfloat162*>(&pk);
#pragma unroll
        for (int e = 0; e < 4; ++e) ph[e] = __floats2bfloat162_rn(r[2 * e], r[2 * e + 1]);
        bf16x8_to_f32(pk, r);   // the residual stream is stored in bf16
        xr[v] = pk;
        sX[v] = pk;
      }
#pragma unroll
      for (int e = 0; e < 8; ++e) s += r[e];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) red[warp * vpt + i] = s;
  }
  worker_sync();
  float tot = 0.f;
  for (int i = 0; i < nt / 32; ++i) tot += red[i];
  const float mean = tot / (float)h;
  worker_sync();   // every thread has read the sums out of red
  for (int i = 0; i < vpt; ++i) {
    const int t = (warp * vpt + i) * 32 + lane;
    float q = 0.f;
    for (int v = t; v < nv; v += nt) {
      float r[8];
      bf16x8_to_f32(sX[v], r);
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const float dlt = r[e] - mean;
        q += dlt * dlt;
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    if (lane == 0) red[warp * vpt + i] = q;
  }
  worker_sync();
  float qt = 0.f;
  for (int i = 0; i < nt / 32; ++i) qt += red[i];
  const float var = qt / (float)h;
  const float rstd = 1.0f / sqrtf(var + eps);
  uint4* yr = reinterpret_cast<uint4*>(py + (int64_t)row * h);
  for (int v = tid; v < nv; v += 128) {
    float r[8], g[8], b[8], o[8];
    bf16x8_to_f32(sX[v], r);
    bf16x8_to_f32(sG[v], g);
    bf16x8_to_f32(sBe[v], b);
#pragma unroll
    for (int e = 0; e < 8; ++e) o[e] = (r[e] - mean) * rstd * g[e] + b[e];
    uint4 pk;
    __nv_bfloat162* ph = reinterpret_cast<__nv_bfloat162*>(&pk);
#pragma unroll
    for (int e = 0; e < 4; ++e) ph[e] = __floats2bfloat162_rn(o[2 * e], o[2 * e + 1]);
    yr[v] = pk;
  }
  worker_sync();   // red / stg are reused
}

template <int D, int CH>
__global__ void __launch_bounds__(FD_THREADS, 1)
    fused_decode_kernel(const __grid_constant__ CUtensorMap map_y, const __grid_constant__ CUtensorMap map_attn,
                        const __grid_constant__ CUtensorMap map_h, const __grid_constant__ FParams p) {
  const uint64_t tr0 = trace_now();
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int S = p.S;
  const int B_BYTES = p.bn * FD_BK * 2;
  uint8_t* smW = smem;
  uint8_t* smX = smW + (size_t)S * FD_A_BYTES;
  __nv_bfloat16* kvbuf = reinterpret_cast<__nv_bfloat16*>(smX + (size_t)S * B_BYTES);   // [2][K|V][CH][D]
  constexpr int SLOTS = DecAttnSmem<D, CH>::SLOTS;
  float* f_sc = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(kvbuf) + p.stage_bytes);
  float* f_red = f_sc + 64;            // >= NT/32 (16) and DC_THREADS/32
  float* f_part = f_red + 32;          // SLOTS * D
  float* f_mw = f_part + SLOTS * D;    // DC_MAX_SPLITS
  float* f_lw = f_mw + DC_MAX_SPLITS;
  int* f_flag = reinterpret_cast<int*>(f_lw + DC_MAX_SPLITS);   // [4]
  __nv_bfloat16* f_q = reinterpret_cast<__nv_bfloat16*>(f_flag + 4);   // [4][D] staged queries (16-B aligned)
  uint64_t* bars = reinterpret_cast<uint64_t*>(f_q + 4 * D);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* tmem_full = bars + 2 * S;
  uint64_t* tmem_empty = tmem_full + FD_TS;
  uint64_t* kvbar = tmem_empty + FD_TS;   // [4]
  uint64_t* lnbar = kvbar + 4;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(lnbar + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int G = p.G, cta = blockIdx.x;
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 2);   // weight producer + activation producer
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < FD_TS; ++i) {
      mbar_init(&tmem_full[i], 1);
      mbar_init(&tmem_empty[i], 4);
    }
    for (int i = 0; i < 4; ++i) mbar_init(&kvbar[i], 1);
    mbar_init(lnbar, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_slot, FD_TS * FD_ACC_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------ weight producer
    // Streams W blocks into the smem ring, never waiting on data.  (An L2 prefetch
    // cursor running ahead of the ring was measured: 26 % slower passes.)
    if (lane == 0) {
      const uint64_t pol_w = policy_evict_first();
      WCursor c;
      c.init(p, cta);
      int it = 0;
      int last_lg = -1;
      for (; !c.done; c.next(p, cta), ++it) {
        const int lg = c.l * 4 + c.g;
        if (lg != last_lg) {
          tma_prefetch_desc(&c_wmap[lg]);
          last_lg = lg;
        }
        const int s = it % S;
        mbar_wait(&empty[s], ((it / S) & 1) ^ 1);
        mbar_arrive_expect_tx(&full[s], FD_A_BYTES);
        tma_load_2d_hint(smW + (size_t)s * FD_A_BYTES, &c_wmap[lg], &full[s], 0,
                         (c.tile(p) * p.gm[c.g].nkb + c.kb) * FD_BM, pol_w);
      }
    }
  } else if (warp == 2) {
    // ------------------------------------------------ activation producer
    if (lane == 0) {
      tma_prefetch_desc(&map_y);
      tma_prefetch_desc(&map_attn);
      tma_prefetch_desc(&map_h);
      int it = 0;
      for (int l = 0; l < p.L; ++l) {
        for (int g = 0; g < 4; ++g) {
          const FGemm& gm = p.gm[g];
          const CUtensorMap* xm = g == 1 ? &map_attn : (g == 3 ? &map_h : &map_y);
          const int k = FD_PHASES * l + gemm_phase(g);
          bool waited = false;
          for (int u = first_unit(p, l, g, cta); u < gm.units; u += G) {
            if (!waited) {   // X = the output of phase k-1, complete on every CTA
              wait_counter(p.sync, p.sync_base + (unsigned long long)G * k);
              fence_proxy_async_global();
              waited = true;
            }
            const int z = u % gm.splits;
            const int kb0 = z * gm.kcb, kb1 = min(gm.nkb, kb0 + gm.kcb);
            for (int kb = kb0; kb < kb1; ++kb, ++it) {
              const int s = it % S;
              mbar_wait(&empty[s], ((it / S) & 1) ^ 1);
              mbar_arrive_expect_tx(&full[s], B_BYTES);
              tma_load_2d(smX + (size_t)s * B_BYTES, xm, &full[s], kb * FD_BK, 0);
            }
          }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer
    if (lane == 0) {
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(p.bn >> 3) << 17) |
                             ((uint32_t)(FD_BM >> 4) << 24);
      int it = 0, lu = 0;
      for (int l = 0; l < p.L; ++l) {
        for (int g = 0; g < 4; ++g) {
          const FGemm& gm = p.gm[g];
          for (int u = first_unit(p, l, g, cta); u < gm.units; u += G, ++lu) {
            const int z = u % gm.splits;
            const int kb0 = z * gm.kcb, kb1 = min(gm.nkb, kb0 + gm.kcb);
            const int acc = lu % FD_TS;
            mbar_wait(&tmem_empty[acc], ((lu / FD_TS) & 1) ^ 1);
            tc_fence_after();
            const uint32_t tacc = tmem_base + (uint32_t)acc * FD_ACC_COLS;
            for (int kb = kb0; kb < kb1; ++kb, ++it) {
              const int s = it % S;
              mbar_wait(&full[s], (it / S) & 1);
              tc_fence_after();
              const uint64_t adesc = umma_desc_sw128(smem_u32(smW + (size_t)s * FD_A_BYTES));
              const uint64_t bdesc = umma_desc_sw128(smem_u32(smX + (size_t)s * B_BYTES));
#pragma unroll
              for (int k = 0; k < FD_BK / 16; ++k)
                umma_bf16(tacc, adesc + 2 * k, bdesc + 2 * k, idesc, (kb > kb0 || k) ? 1u : 0u);
              umma_commit(&empty[s]);
            }
            umma_commit(&tmem_full[acc]);
          }
        }
      }
    }
  } else if (warp >= 4) {
    // ------------------------------------------------ workers (128 threads)
    const int tid = threadIdx.x - 128;
    const int q = warp & 3;   // TMEM lane quarter
    DecAttnSmem<D, CH> asm_;
    asm_.sc = f_sc;
    asm_.red = f_red;
    asm_.part = f_part;
    asm_.mw = f_mw;
    asm_.lw = f_lw;
    asm_.last = f_flag;
    int lu = 0;          // accumulator units consumed
    unsigned ln_rows = 0;  // LayerNorm rows processed (lnbar parity)
    unsigned items = 0;  // attention items processed (KV buffer / parity sequence)
    const int b = p.M;
    const int n_items = p.heads * b * p.nsp;
    auto phase_done = [&](int k) {
      // every phase before k complete everywhere, and this CTA's share of k done
      // (bar.sync + one release by thread 0 publishes the group's writes)
      if (tid == 0) wait_counter(p.sync, p.sync_base + (unsigned long long)G * k);
      worker_sync();
      if (tid == 0) red_release_add_u64(p.sync, 1ull);
    };
    auto wait_phase = [&](int k) {
      if (tid == 0) wait_counter(p.sync, p.sync_base + (unsigned long long)G * k);
      worker_sync();
    };
    // publish this group's plain stores, then bump counters without waiting for a reply
    auto publish = [&]() {
      worker_sync();
      if (tid == 0) asm volatile("fence.acq_rel.gpu;" ::: "memory");
    };
    auto red_add = [&](int* c) { asm volatile("red.relaxed.gpu.global.add.s32 [%0], 1;" ::"l"(c) : "memory"); };
    auto wait_count = [&](const int* c, int target) {   // tid 0 only
      const uint64_t t0 = trace_now();
      while (true) {
        int v;
        asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(c) : "memory");
        if (v >= target) break;
        __nanosleep(64);
        if (trace_now() - t0 > 2000000000ull) __trap();
      }
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
    };
    for (int l = 0; l < p.L; ++l) {
      const FLayer& W = p.layers[l];
      for (int ph = 0; ph < FD_PHASES; ++ph) {
        const int k = FD_PHASES * l + ph;
        const uint64_t tq0 = trace_now();
        if (ph == 0 || ph == 4) {
          // -------------------------------- add + LayerNorm rows (p0: LN1, p4: LN2)
          wait_phase(k);
          const __nv_bfloat16* add = nullptr;
          const __nv_bfloat16* ab = nullptr;
          if (ph == 4) {
            add = p.part;
            ab = W.b_o;
          } else if (!(l == 0 && p.first_no_add)) {
            add = p.part;
            ab = p.layers[l - 1 >= 0 ? l - 1 : 0].b_2;
          }
          const __nv_bfloat16* gam = ph == 0 ? W.g1 : W.g2;
          const __nv_bfloat16* bet = ph == 0 ? W.be1 : W.be2;
          const uint64_t tw = trace_now();
          bool had = false;
          for (int r = ((cta - k * 7) % G + G) % G; r < b; r += G) {
            had = true;
            // the KV staging region is idle during LN phases
            ln_row(p.x, p.y, p.h, p.ln_nt, p.eps, r, add, ab, gam, bet, f_red, reinterpret_cast<uint4*>(kvbuf),
                   lnbar, ln_rows & 1, tid);
            ++ln_rows;
          }
          const uint64_t tl = trace_now();
          phase_done(k);
          if (had && tid == 0) trace_write(0x400u, tw, tl);   // LN row CTA: wait released, rows done, signalled
        } else if (ph == 2) {
          // -------------------------------- attention: chunk items (double-buffered staging
          // of q, K, V), then the (sequence, head) merges owned by this CTA
          wait_phase(k);
          DecAttnArgs aa = p.attn;
          aa.kv_pool = p.kv + (size_t)l * p.kv_layer_elems;
          const int i0 = ((cta - (int)(((long long)k * 13) % G)) % G + G) % G;
          const int NB = p.nbuf;
          auto issue = [&](int i, unsigned cnt) {
            const int hd = i % p.heads, bi = (i / p.heads) % b, sp = i / (p.heads * b);
            const unsigned buf = cnt % NB;
            __nv_bfloat16* sK = kvbuf + (size_t)buf * 2 * CH * D;
            fence_proxy_async_smem();   // the buffer held generic writes of an earlier item
            __syncwarp();
            dec_attn_issue<D, CH>(aa, hd, bi, sp, sK, sK + CH * D, &kvbar[buf], tid, f_q + buf * D);
          };
          // items are staged NB - 1 ahead of the one being computed
          int i_iss = i0;
          unsigned c_iss = items;
          for (int j = 0; j < NB - 1 && i_iss < n_items; ++j, i_iss += G, ++c_iss)
            if (tid < 32) issue(i_iss, c_iss);
          for (int i = i0; i < n_items; i += G, ++items) {
            if (i_iss < n_items) {
              if (tid < 32) issue(i_iss, c_iss);
              i_iss += G;
              ++c_iss;
            }
            const int hd = i % p.heads, bi = (i / p.heads) % b, sp = i / (p.heads * b);
            const unsigned buf = items % NB;
            asm_.sK = kvbuf + (size_t)buf * 2 * CH * D;
            asm_.sV = asm_.sK + CH * D;
            asm_.bar = &kvbar[buf];
            dec_attn_partial<D, CH>(aa, hd, bi, sp, p.nsp, asm_, (items / NB) & 1, tid, WorkerSync{},
                                    f_q + buf * D);
          }
          const uint64_t ta1 = trace_now();
          if (p.nsp > 1) {
            publish();
            if (tid == 0)
              for (int i = i0; i < n_items; i += G) red_add(&aa.counters[(i / p.heads) % b * p.heads + i % p.heads]);
            const int n_units = b * p.heads;
            for (int u = ((cta - (int)(((long long)k * 29) % G)) % G + G) % G; u < n_units; u += G) {
              if (tid == 0) wait_count(&aa.counters[u], p.nsp);
              worker_sync();
              dec_attn_merge<D, CH>(aa, u % p.heads, u / p.heads, p.nsp, asm_, tid, WorkerSync{});
              if (tid == 0) aa.counters[u] = 0;
            }
          }
          const uint64_t ta2 = trace_now();
          phase_done(k);
          if (tid == 0) trace_write(0x430u, ta1, ta2);   // items done, merges done, signalled
        } else {
          // -------------------------------- GEMM: epilogues / split partials, then the
          // split reductions of the tiles this CTA owns
          const int g = ph == 1 ? 0 : (ph == 3 ? 1 : (ph == 5 ? 2 : 3));
          const FGemm& gm = p.gm[g];
          const __nv_bfloat16* bias = g == 0 ? W.b_qkv : (g == 2 ? W.b_1 : nullptr);
          __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(gm.out);
          const int mcount = b;
          const int u_first = first_unit(p, l, g, cta);
          for (int u = u_first; u < gm.units; u += G, ++lu) {
            const int z = u % gm.splits, tile = u / gm.splits;
            const int row = q * 32 + lane;
            const int n = tile * FD_BM + row;
            const int acc = lu % FD_TS;
            const uint64_t tu0 = trace_now();
            mbar_wait(&tmem_full[acc], (lu / FD_TS) & 1);
            tc_fence_after();
            if (tid == 0) trace_write(0x300u + (uint32_t)g, tu0, trace_now());   // per-unit (diagnostics)
            const uint32_t tacc = tmem_base + (uint32_t)acc * FD_ACC_COLS + ((uint32_t)(q * 32) << 16);
            float* my_ws = p.ws + ((int64_t)z * gm.tiles + tile) * (FD_BM * p.bn) + row;
            const float bias_v = (gm.splits == 1 && bias) ? __bfloat162float(bias[n]) : 0.0f;
            for (int c0 = 0; c0 < p.bn; c0 += 16) {
              if (c0 >= mcount) break;
              uint32_t r[16];
              tmem_ld_32x32b_x16(tacc + (uint32_t)c0, r);
              tmem_ld_wait();
              if (gm.splits == 1) {
#pragma unroll
                for (int j = 0; j < 16; ++j)
                  if (c0 + j < mcount)
                    out[(int64_t)(c0 + j) * gm.ldo + n] =
                        __float2bfloat16_rn(fd_epi(gm, __uint_as_float(r[j]), n, bias_v));
              } else {
#pragma unroll
                for (int j = 0; j < 16; ++j)
                  if (c0 + j < mcount) __stcg(my_ws + (int64_t)(c0 + j) * FD_BM, __uint_as_float(r[j]));
              }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tmem_empty[acc]);
          }
          const uint64_t tg1 = trace_now();
          uint64_t tg2 = tg1;
          if (gm.splits > 1) {
            publish();
            if (tid == 0)
              for (int u = u_first; u < gm.units; u += G) red_add(&p.tile_cnt[u / gm.splits]);
            tg2 = trace_now();
            const int64_t zstride = (int64_t)gm.tiles * (FD_BM * p.bn);
            for (int tile = ((cta - (int)(((long long)k * 31) % G)) % G + G) % G; tile < gm.tiles; tile += G) {
              if (tid == 0) wait_count(&p.tile_cnt[tile], gm.splits);
              worker_sync();
              // reduce in z order; thread <-> (token m, 4 consecutive rows), 8 chunks in flight
              for (int w = tid; w < mcount * (FD_BM / 4); w += 128) {
                const int m = w / (FD_BM / 4), rq = w % (FD_BM / 4);
                const float* src = p.ws + (int64_t)tile * (FD_BM * p.bn) + (int64_t)m * FD_BM + rq * 4;
                float4 a = __ldcg(reinterpret_cast<const float4*>(src));
                for (int z0 = 1; z0 < gm.splits; z0 += 8) {
                  float4 v[8];
#pragma unroll
                  for (int i = 0; i < 8; ++i)
                    v[i] = (z0 + i < gm.splits) ? __ldcg(reinterpret_cast<const float4*>(src + (z0 + i) * zstride))
                                                : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
                  for (int i = 0; i < 8; ++i)
                    if (z0 + i < gm.splits) {
                      a.x += v[i].x;
                      a.y += v[i].y;
                      a.z += v[i].z;
                      a.w += v[i].w;
                    }
                }
                const int n0 = tile * FD_BM + rq * 4;
                const float av[4] = {a.x, a.y, a.z, a.w};
                __align__(8) __nv_bfloat16 o4[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                  const float bv = bias ? __bfloat162float(bias[n0 + i]) : 0.0f;
                  o4[i] = __float2bfloat16_rn(fd_epi(gm, av[i], n0 + i, bv));
                }
                *reinterpret_cast<uint2*>(out + (int64_t)m * gm.ldo + n0) = *reinterpret_cast<const uint2*>(o4);
              }
              if (tid == 0) p.tile_cnt[tile] = 0;
            }
          }
          const uint64_t tg3 = trace_now();
          phase_done(k);
          if (tid == 0) {
            trace_write(0x410u + g, tg1, tg2);   // units done, partials published, (now)
            trace_write(0x420u + g, tg2, tg3);   // published, owned reductions done, signalled
          }
        }
        if (tid == 0) trace_write(0x200u + (uint32_t)ph, tq0, tq0);   // per-phase timeline (diagnostics)
      }
    }
    if (tid == 0) trace_write(TK_FUSED, tr0, tr0);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem_base, FD_TS * FD_ACC_COLS);
  }
}

int num_sms_fd() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

int ln_threads(int h) {   // add_layernorm_launch's choice
  const int nv = h / 8;
  if (nv <= 512) return 128;
  if (nv <= 1024) return 256;
  return 512;
}

}  // namespace

struct FusedDecodeState {
  FLayer* d_layers = nullptr;      // [L]
  int L = 0;
  std::vector<const void*> key;    // weight pointers the tables were built from
  std::vector<CUtensorMap> maps;   // host copy of the weight descriptors
  unsigned long long* d_sync = nullptr;
  unsigned long long sync_total = 0;   // counter increments of all earlier launches
  int G = 0;
};

void fused_decode_free(FusedDecodeState* st) {
  if (!st) return;
  if (st->d_layers) cudaFree(st->d_layers);
  if (st->d_sync) cudaFree(st->d_sync);
  delete st;
}

bool fused_decode_supported(int M, int h, int heads, int d, int ffn) {
  if (M < 1 || M > 32) return false;
  if (d != 64 && d != 128) return false;
  if (h % 128 || ffn % 128 || (3 * heads * d) % 128 || (heads * d) % 64) return false;
  if (h / 8 > 512 * 4) return false;   // LayerNorm rows of at most 4 vectors per virtual thread
  return true;
}

int fused_decode_launch(FusedDecodeState** pst, const FusedDecodeArgs& a, cudaStream_t stream) {
  if (!fused_decode_supported(a.M, a.h, a.heads, a.d, a.ffn) || a.L > FD_MAX_LAYERS) return LIGER_EINVAL;
  const int L = a.L, M = a.M, h = a.h, hl = a.heads * a.d;
  const int G = num_sms_fd();
  FusedDecodeState* st = *pst;
  if (!st) {
    st = new FusedDecodeState();
    *pst = st;
    if (cudaMalloc(&st->d_sync, sizeof(unsigned long long)) != cudaSuccess) return LIGER_ENOMEM;
    cudaMemset(st->d_sync, 0, sizeof(unsigned long long));
    st->G = G;
  }
  // per-layer weight descriptors and vector pointers (rebuilt when the weights change)
  std::vector<const void*> key;
  key.reserve((size_t)L * 12);
  for (int l = 0; l < L; ++l) {
    const FusedLayerPtrs& w = a.layers[l];
    const void* v[12] = {w.w_qkv, w.w_o, w.w_1, w.w_2, w.b_qkv, w.b_o, w.b_1, w.b_2, w.g1, w.be1, w.g2, w.be2};
    key.insert(key.end(), v, v + 12);
  }
  // the constant-memory descriptor table is shared by every state of the process
  static std::vector<const void*> c_key;
  if (key != st->key) {
    if (st->d_layers) cudaFree(st->d_layers);
    st->d_layers = nullptr;
    std::vector<CUtensorMap> maps((size_t)L * 4);
    std::vector<FLayer> lay(L);
    const int NN[4] = {3 * hl, h, a.ffn, h}, KK[4] = {h, hl, h, a.ffn};
    for (int l = 0; l < L; ++l) {
      const FusedLayerPtrs& w = a.layers[l];
      const void* ws[4] = {w.w_qkv, w.w_o, w.w_1, w.w_2};
      for (int g = 0; g < 4; ++g)
        if (gemm_weight_map(&maps[(size_t)l * 4 + g], ws[g], NN[g], KK[g])) return LIGER_ECUDA;
      lay[l] = FLayer{(const __nv_bfloat16*)w.b_qkv, (const __nv_bfloat16*)w.b_o, (const __nv_bfloat16*)w.b_1,
                      (const __nv_bfloat16*)w.b_2,   (const __nv_bfloat16*)w.g1,  (const __nv_bfloat16*)w.be1,
                      (const __nv_bfloat16*)w.g2,    (const __nv_bfloat16*)w.be2};
    }
    if (cudaMalloc(&st->d_layers, lay.size() * sizeof(FLayer)) != cudaSuccess) return LIGER_ENOMEM;
    cudaMemcpy(st->d_layers, lay.data(), lay.size() * sizeof(FLayer), cudaMemcpyHostToDevice);
    st->key = key;
    st->L = L;
    st->maps.swap(maps);
  }
  if (key != c_key) {   // stream-ordered: earlier launches keep their table until they finish
    if (cudaMemcpyToSymbolAsync(c_wmap, st->maps.data(), st->maps.size() * sizeof(CUtensorMap), 0,
                                cudaMemcpyHostToDevice, stream) != cudaSuccess)
      return LIGER_ECUDA;
    c_key = key;
  }

  FParams p{};
  p.L = L;
  p.M = M;
  p.h = h;
  p.heads = a.heads;
  p.d = a.d;
  p.G = G;
  p.pos = a.pos;
  p.first_no_add = a.first_no_add;
  p.eps = a.eps;
  p.ln_nt = ln_threads(h);

  const int NN[4] = {3 * hl, h, a.ffn, h}, KK[4] = {h, hl, h, a.ffn};
  void* outs[4] = {a.qkv, a.part, a.hbuf, a.part};
  const int64_t ldos[4] = {3 * hl, h, a.ffn, h};
  size_t ws_need = GEMM_COUNTER_BYTES;
  p.units_layer = 0;
  for (int g = 0; g < 4; ++g) {
    const GemmPlan pl = gemm_plan(M, NN[g], KK[g]);   // the per-kernel path's plan: same bits
    FGemm& f = p.gm[g];
    f.N = NN[g];
    f.K = KK[g];
    f.nkb = KK[g] / FD_BK;
    f.kcb = pl.kc / FD_BK;
    f.splits = pl.splits;
    f.tiles = NN[g] / FD_BM;
    f.units = f.tiles * f.splits;
    f.scale_cols = g == 0 ? hl : 0;
    f.scale = g == 0 ? a.qscale : 1.0f;
    f.act = g == 2 ? a.act : LIGER_ACT_NONE;
    f.out = outs[g];
    f.ldo = ldos[g];
    p.bn = pl.bn;
    p.units_layer += f.units;
    if (f.tiles > FD_MAX_TILES) return LIGER_EINVAL;
    if (f.splits > 1)
      ws_need = std::max(ws_need, GEMM_COUNTER_BYTES + (size_t)f.splits * f.tiles * FD_BM * pl.bn * sizeof(float));
  }
  if (p.bn > FD_ACC_COLS || ws_need > a.gemm_ws_bytes || (size_t)FD_MAX_TILES * 4 > GEMM_COUNTER_BYTES)
    return LIGER_EINVAL;
  p.tile_cnt = reinterpret_cast<int*>(a.gemm_ws);
  p.ws = reinterpret_cast<float*>(reinterpret_cast<char*>(a.gemm_ws) + GEMM_COUNTER_BYTES);
  p.sync = st->d_sync;
  p.sync_base = st->sync_total;
  p.layers = st->d_layers;
  p.x = (__nv_bfloat16*)a.x;
  p.y = (__nv_bfloat16*)a.y;
  p.part = (__nv_bfloat16*)a.part;
  p.kv = (__nv_bfloat16*)a.kv;
  p.kv_layer_elems = a.kv_layer_elems;
  // attention: the standalone kernel's chunking (same bits)
  const int ctx = a.pos + 1;
  const int CH = dec_attn_chunk(M, a.heads, ctx);
  p.nsp = (ctx + CH - 1) / CH;
  if (p.nsp > DC_MAX_SPLITS) return LIGER_EINVAL;
  if (p.nsp > 1 && (!a.attn_ws || a.attn_ws_bytes < attn_decode_workspace_bytes(M, a.heads, a.d, ctx)))
    return LIGER_EINVAL;
  p.attn.qkv = (const __nv_bfloat16*)a.qkv;
  p.attn.o = (__nv_bfloat16*)a.attn;
  p.attn.kv_pool = nullptr;
  p.attn.page_table = a.page_table;
  p.attn.max_pages = a.max_pages;
  p.attn.pos = a.pos;
  p.attn.heads = a.heads;
  p.attn.counters = (int*)a.attn_ws;
  p.attn.ws = a.attn_ws ? (float*)((char*)a.attn_ws + ATTN_COUNTER_BYTES) : nullptr;

  CUtensorMap my, ma, mh;
  if (gemm_act_map(&my, a.y, M, h, h, p.bn) || gemm_act_map(&ma, a.attn, M, hl, hl, p.bn) ||
      gemm_act_map(&mh, a.hbuf, M, a.ffn, a.ffn, p.bn))
    return LIGER_ECUDA;

  // shared memory: weight ring + activation ring + 2 KV staging buffers + attention scratch
  const int D = a.d;
  // KV staging (2 items) -- reused by the LayerNorm phases for the row, gamma and beta
  const size_t item_bytes = (size_t)2 * CH * D * 2;
  p.nbuf = 3 * item_bytes <= 64 * 1024 ? 3 : 2;
  const size_t kv_bytes = std::max(p.nbuf * item_bytes, ((size_t)5 * h * 2 + 1023) / 1024 * 1024);
  p.stage_bytes = (int)kv_bytes;
  const size_t misc = (64 + 32 + (size_t)(DC_THREADS / (D / 8)) * D + 2 * DC_MAX_SPLITS) * 4 + 16 + 4 * D * 2 +
                      8 * 64 + 16;
  const size_t stage = FD_A_BYTES + (size_t)p.bn * FD_BK * 2;
  long long avail = (long long)FD_MAX_SMEM - 1024 - (long long)kv_bytes - (long long)misc;
  int S = (int)(avail / (long long)stage);
  if (S > 12) S = 12;
  if (const char* e = getenv("LIGER_FD_STAGES")) {   // experiments only
    const int f = atoi(e);
    if (f >= 2 && f < S) S = f;
  }
  if (S < 3) return LIGER_EINVAL;
  p.S = S;
  const size_t smem = 1024 + (size_t)S * stage + kv_bytes + misc;

  cudaError_t e;
#define FD_LAUNCH(DD, CC)                                                                                    \
  {                                                                                                          \
    static bool attr = false;                                                                                \
    if (!attr) {                                                                                             \
      cudaFuncSetAttribute(fused_decode_kernel<DD, CC>, cudaFuncAttributeMaxDynamicSharedMemorySize, FD_MAX_SMEM); \
      attr = true;                                                                                           \
    }                                                                                                        \
    fused_decode_kernel<DD, CC><<<G, FD_THREADS, smem, stream>>>(my, ma, mh, p);                             \
  }
  if (D == 128 && CH == 32) FD_LAUNCH(128, 32)
  else if (D == 128) FD_LAUNCH(128, 64)
  else if (CH == 32) FD_LAUNCH(64, 32)
  else FD_LAUNCH(64, 64)
#undef FD_LAUNCH
  e = cudaGetLastError();
  if (e != cudaSuccess) return LIGER_ECUDA;
  st->sync_total += (unsigned long long)G * FD_PHASES * L;
  return 0;
}

LIGER_TRACE_SETTER(fused)

}  // namespace liger
