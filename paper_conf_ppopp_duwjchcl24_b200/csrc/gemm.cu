// tcgen05 / TMEM / TMA GEMM for the TP decoder-layer projections (sm_100a).
//
// Computes, for the output-column slice [n0, n1) (runtime kernel decomposition,
// PAPER.md §3.6, "vertical" split of Fig. 9):
//     out[m, n] = epi( sum_k X[m, k] * W[n, k] )          m < M, n0 <= n < n1
// X: activations bf16 row-major [M, K] (row stride ldx); W: weights bf16
// row-major [N, K] (nn.Linear layout, i.e. K-major); fp32 accumulation in TMEM.
// epi: + bias[n], * scale for n < scale_cols (q scaling), ReLU / tanh-GELU,
// then bf16 (or fp32) store.
//
// Orientation ("swap-AB"): the MMA M dimension (128 TMEM lanes) runs over the
// weight rows n, the MMA N dimension over tokens m (bn = 16..256).  Decode
// (M = batch <= 32) therefore costs one 128 x 16 MMA per K step and the kernel
// streams W from HBM; prefill uses 128 x 256 tiles.
//
// Bit-exactness of decomposition (SURVEY AMB-9): every per-element quantity --
// the token tiling bn, the split-K chunk kc and the K order, the fixed z-order
// of the split-K reduction -- is a function of (M, K) only, never of N or of
// the slice, so a slice computes exactly the bits of the full GEMM.
//
// Warp roles (192 threads): warp 0 = TMA producer, warp 1 = TMEM allocator +
// single-thread MMA issuer, warps 2..5 = epilogue (TMEM -> registers -> HBM).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <algorithm>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "common.cuh"
#include "kernels.h"

namespace liger {

constexpr int BM = 128;           // weight rows per tile (MMA M)
constexpr int BK = 64;            // K per stage (one 128-byte swizzle atom)
constexpr int A_BYTES = BM * BK * 2;
constexpr int GEMM_THREADS = 192;
constexpr int MAX_SMEM = 227 * 1024;

static int num_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

struct GemmParams {
  int M, N, K;
  int n0, n1;
  int kc, splits;
  int bn;
  int stages;
  int n_tiles, m_tiles;
  int units;            // n_tiles * m_tiles * splits
  int w_tiled;          // W stored as [N/128][K/64][128][64] (each TMA box contiguous)
  int nkb_total;        // K / 64

  const __nv_bfloat16* bias;
  int act;
  int scale_cols;
  float scale;
  void* out;
  int64_t ldo;
  int out_f32;
  float* ws;
  // fused all-reduce producer (fixup kernel): publish pub_epoch on pub_flag (system
  // scope) once every CTA's output stores are visible
  unsigned long long* pub_flag;
  unsigned int* pub_counter;
  unsigned long long pub_epoch;
  // LayerNorm folded into the GEMM (decode, t = 1): W holds W*gamma; the epilogue
  // computes v = rstd_m * (acc - mean_m * ln_u[n]) + ln_c[n] (ln_c = W.beta + bias)
  // with mean_m / rstd_m of the raw input rows X[m, :] (which the kernel computes
  // itself, and CTA 0 publishes in ln_stats for the split-K fixup)
  int ln_fold;
  const float* ln_u;
  const float* ln_c;
  float* ln_stats;                  // [M][2] (mean, rstd) written by CTA 0, read by the fixup
  const __nv_bfloat16* ln_x;        // X (the rows to normalise), row stride ln_ldx
  int64_t ln_ldx;
  float ln_eps;
  // residual add in the final store: out[m, n] = resid[m, n] + v (may alias out)
  const __nv_bfloat16* resid;
};

// mean / rstd (population variance, eps inside the sqrt) of rows m < M of X[M, K]
// into st[2m], st[2m + 1]: one fp32 pass over the row, shifted by its first element
// (s1 = sum(x - x0), s2 = sum((x - x0)^2); mean = x0 + s1/K, var = s2/K - (s1/K)^2),
// which keeps the cancellation of the one-pass form small.  The calling threads are
// whole warps (tid 0..nthreads-1); warp w takes rows w, w + nwarps, ...
__device__ __forceinline__ void ln_row_stats(const __nv_bfloat16* X, int64_t ldx, int M, int K, float eps, float* st,
                                             int tid, int nthreads) {
  const int lane = tid & 31, w = tid >> 5, nw = nthreads >> 5;
  const int nv = K >> 3;
  for (int m = w; m < M; m += nw) {
    const __nv_bfloat16* rowp = X + (int64_t)m * ldx;
    const uint4* row = reinterpret_cast<const uint4*>(rowp);
    const float x0 = __bfloat162float(rowp[0]);
    float s1 = 0.f, s2 = 0.f;
    for (int v0 = lane; v0 < nv; v0 += 32 * 8) {
      uint4 q[8];
#pragma unroll
      for (int i = 0; i < 8; ++i)
        if (v0 + i * 32 < nv) q[i] = __ldcg(row + v0 + i * 32);
#pragma unroll
      for (int i = 0; i < 8; ++i)
        if (v0 + i * 32 < nv) {
          const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&q[i]);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float2 f = __bfloat1622float2(h2[e]);
            const float a = f.x - x0, b = f.y - x0;
            s1 += a + b;
            s2 += a * a + b * b;
          }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      s1 += __shfl_xor_sync(0xffffffffu, s1, o);
      s2 += __shfl_xor_sync(0xffffffffu, s2, o);
    }
    if (lane == 0) {
      const float d = s1 / (float)K;
      st[2 * m] = x0 + d;
      st[2 * m + 1] = 1.0f / sqrtf(fmaxf(s2 / (float)K - d * d, 0.0f) + eps);
    }
  }
}

// EXT: the folded-LayerNorm / residual-add epilogue (a separate instantiation, so
// the plain epilogue of the prefill GEMMs keeps its code)
template <bool EXT>
__device__ __forceinline__ float epi_apply(const GemmParams& p, float v, int m, int n, float bias_v,
                                           const float* st) {
  if (EXT && p.ln_fold) v = st[2 * m + 1] * (v - st[2 * m] * p.ln_u[n]) + p.ln_c[n];
  v += bias_v;
  if (n < p.scale_cols) v *= p.scale;
  if (p.act == LIGER_ACT_RELU) v = fmaxf(v, 0.0f);
  else if (p.act == LIGER_ACT_GELU_TANH) v = gelu_tanh_f(v);
  return v;
}

template <bool EXT>
__device__ __forceinline__ void epi_store(const GemmParams& p, int m, int n, float v) {
  if (EXT && p.resid) v += __bfloat162float(p.resid[(int64_t)m * p.ldo + n]);
  if (p.out_f32)
    reinterpret_cast<float*>(p.out)[(int64_t)m * p.ldo + n] = v;
  else
    reinterpret_cast<__nv_bfloat16*>(p.out)[(int64_t)m * p.ldo + n] = __float2bfloat16_rn(v);
}

// Work unit u -> (n tile, m tile, K chunk).  m is the inner tile index so that the
// CTAs running concurrently (units i, i+G, ...) share weight tiles through L2;
// chunks of one tile are adjacent.
struct Unit {
  int nt, mt, z;
};
__device__ __forceinline__ Unit unit_of(const GemmParams& p, int u) {
  Unit r;
  r.z = u % p.splits;
  const int t = u / p.splits;
  r.mt = t % p.m_tiles;
  r.nt = t / p.m_tiles;
  return r;
}

// Persistent: one CTA per SM, CTA i processes units i, i + G, i + 2G, ...
template <bool EXT>
__global__ void __launch_bounds__(GEMM_THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const GemmParams p) {
  const TraceStart tr0 = trace_begin();
  uint64_t tr1 = tr0.t0;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int S = p.stages;
  const int B_BYTES = p.bn * BK * 2;
  uint8_t* smA = smem;
  uint8_t* smB = smem + (size_t)S * A_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smB + (size_t)S * B_BYTES);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* tmem_full = bars + 2 * S;       // [TS]
  uint64_t* tmem_empty = bars + 2 * S + 4;  // [TS]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * S + 8);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int G = gridDim.x;
  const uint32_t acc_cols = p.bn <= 32 ? 32 : (p.bn <= 64 ? 64 : (p.bn <= 128 ? 128 : 256));
  const int TS = acc_cols >= 256 ? 2 : 4;          // TMEM accumulator stages (epilogue slack)
  const uint32_t tmem_cols = (uint32_t)TS * acc_cols;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < TS; ++i) {
      mbar_init(&tmem_full[i], 1);
      mbar_init(&tmem_empty[i], 4);   // one arrive per epilogue warp
    }
    fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
  }
  if (warp == 1) tmem_alloc(tmem_slot, tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      const uint64_t pol_w = policy_evict_first();   // weights: streamed once per tile
      // Programmatic dependent launch: the weight tiles of the first S stages do
      // not depend on the previous kernel, so they are requested before
      // griddepcontrol.wait; activation tiles only after it.
      int pre = 0;
      {
        int it = 0;
        for (int u = blockIdx.x; u < p.units && it < S; u += G) {
          const Unit w = unit_of(p, u);
          const int k0 = w.z * p.kc;
          const int nkb = (min(p.K, k0 + p.kc) - k0 + BK - 1) / BK;
          for (int kb = 0; kb < nkb && it < S; ++kb, ++it) {
            mbar_arrive_expect_tx(&full[it], A_BYTES + B_BYTES);
            const int kk = k0 + kb * BK, nb = p.n0 + w.nt * BM;
            tma_load_2d_hint(smA + (size_t)it * A_BYTES, &tmA, &full[it], p.w_tiled ? 0 : kk,
                             p.w_tiled ? ((nb / BM) * p.nkb_total + kk / BK) * BM : nb, pol_w);
          }
        }
        pre = it;
      }
      grid_dependency_wait();
      grid_dependency_trigger();   // after the wait: dependents overlap only this kernel
      tr1 = trace_now();
      int it = 0, s = 0;   // ring slot / parity advanced incrementally (no divisions in the loop)
      uint32_t ph = 0;
      for (int u = blockIdx.x; u < p.units; u += G) {
        const Unit w = unit_of(p, u);
        const int k0 = w.z * p.kc;
        const int nkb = (min(p.K, k0 + p.kc) - k0 + BK - 1) / BK;
        const int n_base = p.n0 + w.nt * BM, m_base = w.mt * p.bn;
        for (int kb = 0; kb < nkb; ++kb, ++it, (++s == S) ? (s = 0, ph ^= 1u) : 0u) {
          const int kk = k0 + kb * BK;
          if (it >= pre) {
            mbar_wait(&empty[s], ph ^ 1);
            mbar_arrive_expect_tx(&full[s], A_BYTES + B_BYTES);
            tma_load_2d_hint(smA + (size_t)s * A_BYTES, &tmA, &full[s], p.w_tiled ? 0 : kk,
                             p.w_tiled ? ((n_base / BM) * p.nkb_total + kk / BK) * BM : n_base, pol_w);
          }
          tma_load_2d(smB + (size_t)s * B_BYTES, &tmB, &full[s], kk, m_base);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // kind::f16 instruction descriptor: D=f32, A=B=bf16, both K-major, N=bn, M=128.
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(p.bn >> 3) << 17) |
                             ((uint32_t)(BM >> 4) << 24);
      int s = 0, acc = 0;
      uint32_t ph = 0, acc_ph = 0;
      for (int u = blockIdx.x; u < p.units; u += G, (++acc == TS) ? (acc = 0, acc_ph ^= 1u) : 0u) {
        const Unit w = unit_of(p, u);
        const int k0 = w.z * p.kc;
        const int nkb = (min(p.K, k0 + p.kc) - k0 + BK - 1) / BK;
        mbar_wait(&tmem_empty[acc], acc_ph ^ 1);
        tc_fence_after();
        const uint32_t tacc = tmem_base + (uint32_t)acc * acc_cols;
        for (int kb = 0; kb < nkb; ++kb, (++s == S) ? (s = 0, ph ^= 1u) : 0u) {
          mbar_wait(&full[s], ph);
          tc_fence_after();
          const uint64_t adesc = umma_desc_sw128(smem_u32(smA + (size_t)s * A_BYTES));
          const uint64_t bdesc = umma_desc_sw128(smem_u32(smB + (size_t)s * B_BYTES));
#pragma unroll
          for (int k = 0; k < BK / 16; ++k)
            umma_bf16(tacc, adesc + 2 * k, bdesc + 2 * k, idesc, (kb | k) != 0);
          umma_commit(&empty[s]);
        }
        umma_commit(&tmem_full[acc]);
      }
    }
  } else {
    // ---------------- epilogue: warps 2..5 own TMEM lane quarters (warp % 4)
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const int etid = threadIdx.x - 64;
    const int tiles = p.n_tiles * p.m_tiles;
    float* lnst = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(bars) + 512);
    if (EXT && p.ln_fold) {
      // row statistics of the raw input while the producer / MMA warps run the
      // mainloop (X comes from the preceding kernel: wait for it first)
      grid_dependency_wait();
      if (p.splits == 1) {   // this CTA's epilogue applies the fold: every row here
        ln_row_stats(p.ln_x, p.ln_ldx, p.M, p.K, p.ln_eps, lnst, etid, 128);
        named_bar_sync(1, 128);
      } else {
        // the fixup applies it: CTA b publishes rows b, b + G, ... (one warp per row)
        for (int m = blockIdx.x + (etid >> 5) * G; m < p.M; m += 4 * G) {
          ln_row_stats(p.ln_x + (int64_t)m * p.ln_ldx, p.ln_ldx, 1, p.K, p.ln_eps, p.ln_stats + 2 * m, lane, 32);
          __syncwarp();
        }
      }
    }
    int lu = 0;
    for (int u = blockIdx.x; u < p.units; u += G, ++lu) {
      const Unit w = unit_of(p, u);
      const int n_base = p.n0 + w.nt * BM, m_base = w.mt * p.bn;
      const int n = n_base + row;
      const bool nval = (n < p.n1) && (n < p.N);
      const float bias_v = (p.bias != nullptr && nval) ? __bfloat162float(p.bias[n]) : 0.0f;
      const int acc = lu % TS;
      const uint32_t acc_ph = (lu / TS) & 1;
      const int mcount = min(p.bn, p.M - m_base);
      const int tile_id = w.nt * p.m_tiles + w.mt;
      // fp32 partial of (chunk z, tile): [bn cols][128 rows] (a warp writes 128 B per column)
      float* my_ws = p.splits > 1 ? p.ws + ((int64_t)w.z * tiles + tile_id) * (BM * p.bn) + row : nullptr;
      mbar_wait(&tmem_full[acc], acc_ph);
      tc_fence_after();
      const uint32_t tacc = tmem_base + (uint32_t)acc * acc_cols + ((uint32_t)(q * 32) << 16);
      for (int c0 = 0; c0 < p.bn; c0 += 16) {
        if (c0 >= mcount) break;   // warp-uniform
        uint32_t r[16];
        tmem_ld_32x32b_x16(tacc + (uint32_t)c0, r);
        tmem_ld_wait();
        if (p.splits == 1) {
          if (nval) {
#pragma unroll
            for (int j = 0; j < 16; ++j)
              if (c0 + j < mcount)
                epi_store<EXT>(p, m_base + c0 + j, n, epi_apply<EXT>(p, __uint_as_float(r[j]), m_base + c0 + j, n, bias_v, lnst));
          }
        } else {
#pragma unroll
          for (int j = 0; j < 16; ++j)
            if (c0 + j < mcount) __stcg(my_ws + (int64_t)(c0 + j) * BM, __uint_as_float(r[j]));
        }
      }
      // accumulator drained: hand the TMEM buffer back to the MMA warp
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tmem_empty[acc]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem_base, tmem_cols);
  }
  if (threadIdx.x == 0) trace_write(TK_GEMM, tr0, tr1);
}

// Split-K fixup: out[m, n] = epi( sum_{z=0..S-1} partial[z] ) in chunk order (the
// same bits whatever slice or CTA produced each chunk).  One thread per (m, 4 rows n),
// reading the column-major per-tile partials coalesced.
template <bool EXT>
__global__ void __launch_bounds__(256) splitk_reduce_kernel(const GemmParams p) {
  const TraceStart tr0 = trace_begin();
  const int tiles = p.n_tiles * p.m_tiles;
  const int64_t zstride = (int64_t)tiles * (BM * p.bn);
  const int slice_w = p.n1 - p.n0;
  const int64_t total = (int64_t)p.M * (BM / 4) * p.n_tiles;   // (m, tile row group of 4)
  const int64_t t_first = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  // The epilogue operands of this thread's first item (usually its only one) do not
  // depend on the GEMM -- bias, the folded-LN vectors, and the residual rows, written
  // by a fixup at least three kernels back -- so they are loaded before the PDL wait.
  float pb[4] = {0.f, 0.f, 0.f, 0.f}, pu[4] = {0.f, 0.f, 0.f, 0.f}, pc[4] = {0.f, 0.f, 0.f, 0.f},
        pr[4] = {0.f, 0.f, 0.f, 0.f};
  if (t_first < total) {
    const int rq = (int)(t_first % (BM / 4));
    const int64_t t2 = t_first / (BM / 4);
    const int nt = (int)(t2 % p.n_tiles);
    const int m = (int)(t2 / p.n_tiles);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int row = rq * 4 + i;
      const int n = p.n0 + nt * BM + row;
      if (nt * BM + row < slice_w && n < p.N) {
        if (p.bias) pb[i] = __bfloat162float(p.bias[n]);
        if (EXT && p.ln_fold) {
          pu[i] = p.ln_u[n];
          pc[i] = p.ln_c[n];
        }
        if (EXT && p.resid) pr[i] = __bfloat162float(p.resid[(int64_t)m * p.ldo + n]);
      }
    }
  }
  pdl_enter();
  const uint64_t tr1 = trace_now();
  const float* lnst = p.ln_stats;
  for (int64_t t = t_first; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int rq = (int)(t % (BM / 4));
    const int64_t t2 = t / (BM / 4);
    const int nt = (int)(t2 % p.n_tiles);
    const int m = (int)(t2 / p.n_tiles);
    const int mt = m / p.bn, col = m % p.bn;
    const int tile_id = nt * p.m_tiles + mt;
    const float4* src = reinterpret_cast<const float4*>(p.ws + (int64_t)tile_id * (BM * p.bn) + (int64_t)col * BM) + rq;
    // chunk order z = 0..S-1; a group of 8 chunks' loads are all in flight before the adds
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int z0 = 0; z0 < p.splits; z0 += 8) {
      float4 v[8];
#pragma unroll
      for (int i = 0; i < 8; ++i)
        v[i] = (z0 + i < p.splits)
                   ? __ldcg(reinterpret_cast<const float4*>(reinterpret_cast<const float*>(src) + (z0 + i) * zstride))
                   : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int i = 0; i < 8; ++i)
        if (z0 + i < p.splits) {
          if (z0 + i == 0) {
            acc = v[0];
          } else {
            acc.x += v[i].x;
            acc.y += v[i].y;
            acc.z += v[i].z;
            acc.w += v[i].w;
          }
        }
    }
    const float a[4] = {acc.x, acc.y, acc.z, acc.w};
    const bool pre = t == t_first;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int row = rq * 4 + i;
      const int n = p.n0 + nt * BM + row;
      if (nt * BM + row < slice_w && n < p.N) {
        if (pre) {   // epi_apply / epi_store with the prefetched operands (same arithmetic)
          float v = a[i];
          if (EXT && p.ln_fold) v = lnst[2 * m + 1] * (v - lnst[2 * m] * pu[i]) + pc[i];
          v += pb[i];
          if (n < p.scale_cols) v *= p.scale;
          if (p.act == LIGER_ACT_RELU) v = fmaxf(v, 0.0f);
          else if (p.act == LIGER_ACT_GELU_TANH) v = gelu_tanh_f(v);
          if (EXT && p.resid) v += pr[i];
          if (p.out_f32)
            reinterpret_cast<float*>(p.out)[(int64_t)m * p.ldo + n] = v;
          else
            reinterpret_cast<__nv_bfloat16*>(p.out)[(int64_t)m * p.ldo + n] = __float2bfloat16_rn(v);
        } else {
          const float bias_v = p.bias ? __bfloat162float(p.bias[n]) : 0.0f;
          epi_store<EXT>(p, m, n, epi_apply<EXT>(p, a[i], m, n, bias_v, lnst));
        }
      }
    }
  }
  if (p.pub_flag) {   // fused all-reduce: the staged partial is complete once every CTA got here
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) {
      const unsigned int prev = atomicAdd(p.pub_counter, 1u);
      if (prev == gridDim.x - 1) {
        *p.pub_counter = 0;
        __threadfence_system();
        asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p.pub_flag), "l"(p.pub_epoch) : "memory");
      }
    }
  }
  if (threadIdx.x == 0) trace_write(TK_FIXUP, tr0, tr1);
}

// ------------------------------------------------------------------ host side
typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static PFN_encodeTiled get_encode() {
  static PFN_encodeTiled fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeTiled>(f);
  });
  return fn;
}

struct MapKey {
  const void* ptr;
  int64_t rows, cols, ld;
  int box_rows;
  bool operator==(const MapKey& o) const {
    return ptr == o.ptr && rows == o.rows && cols == o.cols && ld == o.ld && box_rows == o.box_rows;
  }
};
struct MapKeyHash {
  size_t operator()(const MapKey& k) const {
    size_t h = std::hash<const void*>()(k.ptr);
    h ^= std::hash<int64_t>()(k.rows * 1315423911ll + k.cols * 2654435761ll + k.ld) + 0x9e3779b9 + (h << 6);
    return h ^ (size_t)k.box_rows;
  }
};

static std::mutex g_map_mu;
static std::unordered_map<MapKey, CUtensorMap, MapKeyHash> g_maps;

// 2-D bf16 tensor [rows, cols] with row stride ld (elements); box = [64, box_rows], SWIZZLE_128B.
static int make_map(CUtensorMap* out, const void* ptr, int64_t rows, int64_t cols, int64_t ld, int box_rows) {
  MapKey key{ptr, rows, cols, ld, box_rows};
  {
    std::lock_guard<std::mutex> g(g_map_mu);
    auto it = g_maps.find(key);
    if (it != g_maps.end()) {
      *out = it->second;
      return 0;
    }
  }
  PFN_encodeTiled enc = get_encode();
  if (!enc) return LIGER_ECUDA;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * 2)};
  cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(out, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return LIGER_ECUDA;
  std::lock_guard<std::mutex> g(g_map_mu);
  if (g_maps.size() > 65536) g_maps.clear();
  g_maps.emplace(key, *out);
  return 0;
}

int gemm_weight_map(void* out_, const void* w_tiled, int N, int K) {
  CUtensorMap* out = static_cast<CUtensorMap*>(out_);
  if (K % BK) return LIGER_EINVAL;
  const int64_t rows = (int64_t)((N + BM - 1) / BM) * (K / BK) * BM;
  return make_map(out, w_tiled, rows, BK, BK, BM);
}
int gemm_act_map(void* out_, const void* x, int M, int K, int64_t ldx, int bn) {
  CUtensorMap* out = static_cast<CUtensorMap*>(out_);
  return make_map(out, x, M, K, ldx, bn);
}

void gemm_forget_pointer_range(const void* base, size_t bytes) {
  std::lock_guard<std::mutex> g(g_map_mu);
  for (auto it = g_maps.begin(); it != g_maps.end();) {
    const char* p = static_cast<const char*>(it->first.ptr);
    if (p >= static_cast<const char*>(base) && p < static_cast<const char*>(base) + bytes)
      it = g_maps.erase(it);
    else
      ++it;
  }
}


// Pipeline stages for a token tile bn within a per-CTA shared-memory budget.
static int stages_for(int bn, int extra_smem, int budget) {
  const int stage_bytes = A_BYTES + bn * BK * 2;
  int st = (budget - 1024 - 512 - extra_smem) / stage_bytes;
  if (st > 12) st = 12;
  static const int dec_cap = getenv("LIGER_GEMM_DECODE_STAGES") ? atoi(getenv("LIGER_GEMM_DECODE_STAGES")) : 6;
  if (bn <= 32 && st > dec_cap) st = dec_cap;   // decode: 96 KiB of weights in flight suffices (measured)
  if (const char* e = getenv("LIGER_GEMM_STAGES")) {   // experiments only
    const int f = atoi(e);
    if (f >= 2 && f < st) st = f;
  }
  return st;
}

constexpr int LN_STATS_SMEM = 2 * 64 * 4;   // folded-LayerNorm row statistics (M <= 64)

// Tiling policy.  A decomposition piece of a GEMM (a column slice [n0, n1)) keeps
// the full GEMM's (M, N, K), so every per-element quantity -- the token tiling
// bn, the split-K chunk kc, the K order inside a chunk and the z-order of the
// split reduction -- is a function of (M, N, K) and identical for the full GEMM
// and all of its slices: slices are bit-exact.  The split count is chosen by a
// small cost model that balances the weight stream over the SMs.  Split chunks
// are summed by the PDL-chained fixup kernel.  (An in-cluster DSMEM reduction, a
// last-CTA reduction and an early fixup were built, measured slower and removed:
// profiles/r01/cluster_splitk.txt.)
static GemmPlan gemm_plan_compute(int M, int N, int K);

// The plan of a shape is computed once per host thread (the cost model loops over split
// counts: ~1-2 us, paid on every launch otherwise -- host time Algorithm 1's rounds
// cannot afford when kernels run for a few microseconds)
GemmPlan gemm_plan(int M, int N, int K) {
  static thread_local std::unordered_map<uint64_t, GemmPlan> cache;
  const uint64_t key = ((uint64_t)(uint32_t)M << 42) ^ ((uint64_t)(uint32_t)N << 21) ^ (uint64_t)(uint32_t)K;
  if (M >= 0 && N >= 0 && K >= 0 && M < (1 << 21) && N < (1 << 21) && K < (1 << 21)) {
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    const GemmPlan pl = gemm_plan_compute(M, N, K);
    if (cache.size() < 4096) cache.emplace(key, pl);
    return pl;
  }
  return gemm_plan_compute(M, N, K);
}

static GemmPlan gemm_plan_compute(int M, int N, int K) {
  GemmPlan pl{};
  const int G = num_sms();
  const int n_tiles = (N + BM - 1) / BM;
  const int nkb = (K + BK - 1) / BK;
  int mt = (M + 255) / 256;
  int bn = (M + mt - 1) / mt;
  bn = (bn + 15) / 16 * 16;
  if (bn < 16) bn = 16;
  const int tiles = n_tiles * mt;
  // Cost model in SM cycles (prefill): a k-block costs max(MMA = 8 bn, weight
  // stream at ~23 B/clk/SM + activation tile from L2 at ~64 B/clk); a unit adds
  // 300; units spread over G persistent CTAs; a split adds the fixup kernel
  // (launch + S*M*N*4 B of partial traffic x 2).
  const double kb_time = fmax(8.0 * bn, A_BYTES / 23.0 + 128.0 * bn / 64.0);
  int best_s = 1;
  double best = 1e300;
  // Prefill GEMMs that already fill the SMs are not split (their fp32 partials
  // would exceed L2); decode GEMMs always consider it.
  const int smax = (M > 64 && tiles >= G) ? 1 : (nkb >= 8 ? nkb / 4 : 1);
  for (int sp = 1; sp <= smax; ++sp) {
    const int kcb = (nkb + sp - 1) / sp;
    const int S = (nkb + kcb - 1) / kcb;
    if (S != sp) continue;
    double cost;
    if (M <= 64) {
      // Decode (weight stream), in us, fitted to tools/split_sweep2.py on B200
      // (profiles/r01/split_sweep_decode.txt): the persistent grid runs rounds of
      // up to G units; a round takes max(its weight bytes at the achievable HBM
      // rate 5.75 TB/s, one unit's k-blocks at a single SM's ~48 GB/s); a split
      // adds the fixup hand-off (0.8 us) and its fp32 partial traffic through L2.
      cost = 0.0;
      const double blk_us = A_BYTES / 48.0e3 + (double)bn * BK * 2 / 200.0e3;   // weights from HBM, activations from L2
      for (double left = (double)tiles * S; left > 0; left -= G) {
        const double units = fmin(left, (double)G);
        const double kb = fmin((double)kcb, (double)nkb);
        cost += fmax(units * kb * A_BYTES / 5.75e6, kb * blk_us) + 0.05;
      }
      if (S > 1) cost += 0.8 + (double)S * M * N * 8.0 / 10.0e6;
    } else {
      const double units = (double)tiles * S;
      cost = ceil(units / G) * (kcb * kb_time + 300.0);
      if (S > 1) cost += 6000.0 + (double)S * M * N * 8.0 / 2600.0;   // fixup launch + partial traffic
    }
    if (cost < best - 1e-9) {
      best = cost;
      best_s = S;
    }
  }
  // Prefill token tiling: an unsplit prefill GEMM also tries smaller token tiles, down
  // to bn = 144, so that its units fill the waves of G persistent CTAs better (e.g.
  // M = 1024, N = 5120: 4 x 256 gives 160 units = 2 rounds of which the second is 8%
  // full; 7 x 160 gives 280 units in 2 rounds of shorter units: 75 -> 56 us on B200,
  // profiles/r02/gemm_prefill_tiling.txt).  Per-k-block cost 430 + 1.8 bn cycles,
  // fitted to the large-M bn = 256 / 192 / 128 times there; a smaller tile must win
  // by 5% (model error).  Below 144 the fixed 16 KiB weight tile per k-block
  // dominates (bn = 128 measured up to 1.45x slower per flop than 256).
  static const bool bn_fixed = getenv("LIGER_GEMM_BN_FIXED") != nullptr;   // experiments only
  constexpr int BN_MIN_PREFILL = 144;
  if (M > 64 && best_s == 1 && !bn_fixed) {
    auto cost1 = [&](int mt_, int bn_) {
      return ceil((double)n_tiles * mt_ / G) * (nkb * (430.0 + 1.8 * bn_) + 300.0);
    };
    const double base = cost1(mt, bn);
    double cbest = base;
    int mt_b = mt, bn_b = bn;
    for (int m2 = mt + 1; m2 <= (M + BN_MIN_PREFILL - 1) / BN_MIN_PREFILL; ++m2) {
      const int b2 = ((M + m2 - 1) / m2 + 15) / 16 * 16;
      if ((M + b2 - 1) / b2 != m2 || b2 < BN_MIN_PREFILL) continue;
      const double c2 = cost1(m2, b2);
      if (c2 < cbest) {
        cbest = c2;
        mt_b = m2;
        bn_b = b2;
      }
    }
    if (cbest < 0.95 * base) {
      mt = mt_b;
      bn = bn_b;
    }
  }
  if (const char* e = getenv("LIGER_GEMM_FORCE_SPLITS")) {   // experiments only
    const int f = atoi(e);
    if (f >= 1 && f <= nkb) best_s = f;
  }
  const int kcb = (nkb + best_s - 1) / best_s;
  pl.bn = bn;
  pl.m_tiles = mt;
  pl.kc = kcb * BK;
  pl.splits = (nkb + kcb - 1) / kcb;
  pl.stages = stages_for(bn, LN_STATS_SMEM, MAX_SMEM);
  pl.smem = 1024 + pl.stages * (A_BYTES + pl.bn * BK * 2) + 512 + LN_STATS_SMEM;
  return pl;
}

size_t gemm_workspace_bytes(int M, int N, int K) {
  GemmPlan pl = gemm_plan(M, N, K);
  if (pl.splits <= 1) return GEMM_COUNTER_BYTES;
  const size_t tiles = (size_t)((N + BM - 1) / BM + 1) * pl.m_tiles;   // +1: unaligned slices
  return GEMM_COUNTER_BYTES + (size_t)pl.splits * tiles * BM * pl.bn * sizeof(float);
}

int gemm_launch(const GemmArgs& a, cudaStream_t stream) {
  if (a.M <= 0 || a.n1 <= a.n0) return 0;
  if (a.K <= 0 || a.K % 8 || a.ldx % 8 || (!a.w_tiled && a.ldw % 8) || a.n0 < 0 || a.n1 > a.N) return LIGER_EINVAL;
  GemmPlan pl = gemm_plan(a.M, a.N, a.K);
  const int ntiles = (a.n1 - a.n0 + BM - 1) / BM;
  if (pl.splits > 1) {
    if (!a.workspace) return LIGER_EINVAL;
    const size_t need = GEMM_COUNTER_BYTES + (size_t)pl.splits * ntiles * pl.m_tiles * BM * pl.bn * sizeof(float);
    if (a.ws_bytes < need) return LIGER_EINVAL;
  }
  CUtensorMap tA, tB;
  int rc;
  if (a.w_tiled) {
    if (a.K % BK || a.n0 % BM) return LIGER_EINVAL;
    const int64_t rows = (int64_t)((a.N + BM - 1) / BM) * (a.K / BK) * BM;
    rc = make_map(&tA, a.w, rows, BK, BK, BM);
  } else {
    rc = make_map(&tA, a.w, a.N, a.K, a.ldw, BM);
  }
  if (rc) return rc;
  rc = make_map(&tB, a.x, a.M, a.K, a.ldx, pl.bn);
  if (rc) return rc;
  static bool attr_set = false;
  if (!attr_set) {
    for (auto k : {gemm_tc_kernel<false>, gemm_tc_kernel<true>}) {
      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, MAX_SMEM);
      cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    }
    attr_set = true;
  }
  GemmParams p;
  p.M = a.M; p.N = a.N; p.K = a.K; p.n0 = a.n0; p.n1 = a.n1;
  p.kc = pl.kc; p.splits = pl.splits; p.bn = pl.bn; p.stages = pl.stages;
  p.bias = reinterpret_cast<const __nv_bfloat16*>(a.bias);
  p.act = a.act; p.scale_cols = a.scale_cols; p.scale = a.scale;
  p.out = a.out; p.ldo = a.ldo; p.out_f32 = a.out_f32;
  p.pub_flag = nullptr; p.pub_counter = nullptr; p.pub_epoch = 0;
  p.ln_fold = a.ln_fold; p.ln_u = a.ln_u; p.ln_c = a.ln_c; p.ln_stats = a.ln_stats;
  p.ln_x = reinterpret_cast<const __nv_bfloat16*>(a.x); p.ln_ldx = a.ldx; p.ln_eps = a.ln_eps;
  p.resid = reinterpret_cast<const __nv_bfloat16*>(a.resid);
  if (a.ln_fold && (a.M > 64 || !a.ln_u || !a.ln_c || (pl.splits > 1 && !a.ln_stats) || a.K % 8)) return LIGER_EINVAL;
  const bool ext = a.ln_fold || a.resid;
  if (a.far) {   // fused all-reduce producer: needs the fixup kernel and the whole GEMM
    if (pl.splits <= 1 || a.out_f32 || a.n0 != 0 || a.n1 != a.N) return LIGER_EINVAL;
    p.out = a.far->stage;
    p.ldo = a.N;
    p.pub_flag = a.far->flag;
    p.pub_counter = a.far->counter;
    p.pub_epoch = a.far->epoch;
  }
  p.ws = a.workspace ? reinterpret_cast<float*>(reinterpret_cast<char*>(a.workspace) + GEMM_COUNTER_BYTES) : nullptr;
  p.w_tiled = a.w_tiled;
  p.nkb_total = (a.K + BK - 1) / BK;
  p.n_tiles = ntiles;
  p.m_tiles = pl.m_tiles;
  p.units = ntiles * pl.m_tiles * pl.splits;
  // unit u runs on CTA u % grid: the grid size never changes what a unit computes
  const int sms = (a.sm_budget > 0 && a.sm_budget < num_sms()) ? a.sm_budget : num_sms();
  const int grid = p.units < sms ? p.units : sms;
  const int rc2 = launch_pdl(ext ? gemm_tc_kernel<true> : gemm_tc_kernel<false>, dim3(grid), dim3(GEMM_THREADS),
                             pl.smem, stream, tA, tB, p);
  const bool fixup = p.splits > 1;
  if (a.had_fixup) *a.had_fixup = fixup;
  if (a.ev_mid) cudaEventRecord(a.ev_mid, stream);
  if (rc2 || !fixup) return rc2 ? LIGER_ECUDA : 0;
  const int64_t work = (int64_t)p.M * (BM / 4) * p.n_tiles;
  int rblocks = (int)((work + 255) / 256);
  if (rblocks > num_sms() * 8) rblocks = num_sms() * 8;
  return (ext ? launch_pdl(splitk_reduce_kernel<true>, dim3(rblocks), dim3(256), 0, stream, p)
              : launch_pdl(splitk_reduce_kernel<false>, dim3(rblocks), dim3(256), 0, stream, p))
             ? LIGER_ECUDA
             : 0;
}

void preload_gemm_kernels() {
  for (auto k : {gemm_tc_kernel<false>, gemm_tc_kernel<true>}) {
    preload_kernel(k);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, MAX_SMEM);
  }
  preload_kernel(splitk_reduce_kernel<false>);
  preload_kernel(splitk_reduce_kernel<true>);
}

LIGER_TRACE_SETTER(gemm)

}  // namespace liger
