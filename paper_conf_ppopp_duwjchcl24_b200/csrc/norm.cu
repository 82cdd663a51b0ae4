// Memory-bound kernels of the hot path: fused residual add + LayerNorm (a2/a7/a11),
// embedding (a1), row argmax for greedy decoding (a12), the device-side C0
// weight generator, and small helpers.  All vectorised 16-byte accesses.
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include "common.cuh"
#include "kernels.h"

namespace liger {

struct __align__(16) bf16x8 {
  __nv_bfloat162 h[4];
};

__device__ __forceinline__ void unpack8(const bf16x8& v, float* f) {
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    float2 t = __bfloat1622float2(v.h[i]);
    f[2 * i] = t.x;
    f[2 * i + 1] = t.y;
  }
}
__device__ __forceinline__ bf16x8 pack8(const float* f) {
  bf16x8 v;
#pragma unroll
  for (int i = 0; i < 4; ++i) v.h[i] = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
  return v;
}

template <int NT>
__device__ __forceinline__ float block_sum(float v, float* red) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  __syncthreads();
  if (l == 0) red[w] = v;
  __syncthreads();
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < NT / 32; ++i) s += red[i];   // same order in every thread
  return s;
}

// One CTA per output row; each thread owns up to MAXV 8-element vectors.  All
// global loads of a row (x, add, bias, gamma, beta) are issued before any use so
// the kernel pays one memory round trip (decode rows are latency-bound).
// PEER: the added operand is the fused all-reduce of the row-parallel partials the
// peers staged for epoch far.epoch (peer_ar.cu protocol): wait for every peer's
// flag, then sum the staged rows over ranks 0..t-1 in fp32 in that order and round
// to bf16 -- the one-shot all-reduce's bits, without its kernel.
// LATE: gamma / beta are loaded where they are used (after the statistics) instead of
// being held in registers from the start -- fewer live registers, more resident rows per
// SM: the variant for many-row (prefill) launches, where occupancy, not one row's
// latency, bounds the kernel.
template <int NT, int MAXV, bool PEER, bool LATE = false>
__global__ void __launch_bounds__(NT) add_ln_kernel(const bf16x8* __restrict__ x, const bf16x8* __restrict__ add,
                                                    const bf16x8* __restrict__ add_bias, bf16x8* x_out,
                                                    bf16x8* __restrict__ y, const bf16x8* __restrict__ gamma,
                                                    const bf16x8* __restrict__ beta, int h, int in_row_step,
                                                    int in_row_off, float eps, const FusedARDesc far) {
  __shared__ float red[NT / 32];
  const TraceStart tr0 = trace_begin();
  const int nv = h >> 3;
  const int64_t in_row = (int64_t)blockIdx.x * in_row_step + in_row_off;
  const bf16x8* xr = x + in_row * nv;
  bf16x8 vx[MAXV], va[MAXV], vb[MAXV], vg[MAXV], vbe[MAXV];
  // PDL prologue: every kernel of the path triggers its dependents only after its own
  // griddepcontrol.wait, so while this CTA runs, all kernels but the immediately
  // preceding one have completed.  The LN parameters and the bias are constants, and
  // in the residual-add case (add != NULL) x was written at least two kernels ago
  // (by the previous add + LN; the partial `add` comes from the preceding kernel):
  // their loads are issued before the wait.  Without `add`, x may come from the
  // preceding kernel (the embedding) and is loaded after it.
  const bool x_early = PEER || add != nullptr;
#pragma unroll
  for (int j = 0; j < MAXV; ++j) {
    const int v = threadIdx.x + j * NT;
    if (v < nv) {
      if (x_early) vx[j] = xr[v];
      if (add_bias) vb[j] = add_bias[v];
      if (!LATE) {
        vg[j] = gamma[v];
        vbe[j] = beta[v];
      }
    }
  }
  if (PEER) {
    // dependents are released only after every peer has arrived (a kernel parked at
    // its griddepcontrol.wait must not hold SMs peers sharing this GPU may need)
    grid_dependency_wait();
    if (threadIdx.x == 0) {
      const uint64_t t0 = trace_now();
      for (int q = 0; q < far.world; ++q) {
        unsigned long long f;
        for (;;) {
          asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(f) : "l"(far.peer_flag[q]) : "memory");
          if (f >= far.epoch) break;
          __nanosleep(64);
          if (trace_now() - t0 > 10000000000ull) __trap();   // a peer never arrived: fail, do not hang
        }
      }
    }
    __syncthreads();
    grid_dependency_trigger();
  } else {
    pdl_enter();
  }
  const uint64_t tr1 = trace_now();
#pragma unroll
  for (int j = 0; j < MAXV; ++j) {
    const int v = threadIdx.x + j * NT;
    if (v < nv) {
      if (!x_early) vx[j] = xr[v];
      if (!PEER && add) va[j] = add[in_row * nv + v];
    }
  }
  if (PEER) {
    uint4 pv[MAXV][8];
#pragma unroll
    for (int q = 0; q < 8; ++q)
#pragma unroll
      for (int j = 0; j < MAXV; ++j) {
        const int v = threadIdx.x + j * NT;
        if (q < far.world && v < nv)
          pv[j][q] = __ldcv(reinterpret_cast<const uint4*>(far.peer_stage[q]) + in_row * nv + v);
      }
#pragma unroll
    for (int j = 0; j < MAXV; ++j) {
      const int v = threadIdx.x + j * NT;
      if (v < nv) {
        float acc[8];
        unpack8(*reinterpret_cast<const bf16x8*>(&pv[j][0]), acc);
#pragma unroll
        for (int q = 1; q < 8; ++q)
          if (q < far.world) {
            float f[8];
            unpack8(*reinterpret_cast<const bf16x8*>(&pv[j][q]), f);
#pragma unroll
            for (int e = 0; e < 8; ++e) acc[e] += f[e];
          }
        va[j] = pack8(acc);
      }
    }
  }
  float r[MAXV][8];
  float s = 0.f;
#pragma unroll
  for (int j = 0; j < MAXV; ++j) {
    const int v = threadIdx.x + j * NT;
    if (v < nv) {
      unpack8(vx[j], r[j]);
      if (PEER || add) {
        float a[8];
        unpack8(va[j], a);
#pragma unroll
        for (int e = 0; e < 8; ++e) r[j][e] += a[e];
      }
      if (add_bias) {
        float a[8];
        unpack8(vb[j], a);
#pragma unroll
        for (int e = 0; e < 8; ++e) r[j][e] += a[e];
      }
      bf16x8 pk = pack8(r[j]);          // the residual stream is stored in bf16
      unpack8(pk, r[j]);
      if (x_out) x_out[(int64_t)blockIdx.x * nv + v] = pk;
#pragma unroll
      for (int e = 0; e < 8; ++e) s += r[j][e];
    }
  }
  const float mean = block_sum<NT>(s, red) / (float)h;
  float q = 0.f;
#pragma unroll
  for (int j = 0; j < MAXV; ++j) {
    const int v = threadIdx.x + j * NT;
    if (v < nv) {
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const float dlt = r[j][e] - mean;
        q += dlt * dlt;
      }
    }
  }
  const float var = block_sum<NT>(q, red) / (float)h;
  const float rstd = 1.0f / sqrtf(var + eps);
#pragma unroll
  for (int j = 0; j < MAXV; ++j) {
    const int v = threadIdx.x + j * NT;
    if (v < nv) {
      float g[8], b[8], o[8];
      unpack8(LATE ? gamma[v] : vg[j], g);
      unpack8(LATE ? beta[v] : vbe[j], b);
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = (r[j][e] - mean) * rstd * g[e] + b[e];
      y[(int64_t)blockIdx.x * nv + v] = pack8(o);
    }
  }
  if (threadIdx.x == 0) trace_write(TK_ADDLN, tr0, tr1);
}

int add_layernorm_launch(const void* x, const void* add, const void* add_bias, void* x_out, void* y,
                         const void* gamma, const void* beta, int rows, int h, int in_row_step, int in_row_off,
                         float eps, cudaStream_t stream) {
  if (rows <= 0) return 0;
  if (h % 8 || h > 16384 || !x || !y || !gamma || !beta) return LIGER_EINVAL;
  const bf16x8* X = (const bf16x8*)x;
  const bf16x8* A = (const bf16x8*)add;
  const bf16x8* AB = (const bf16x8*)add_bias;
  const int nv = h / 8;
  const FusedARDesc nofar{};
#define LIGER_LN(NT, MV)                                                                                  \
  launch_pdl(add_ln_kernel<NT, MV, false>, dim3(rows), dim3(NT), 0, stream, X, A, AB, (bf16x8*)x_out,     \
             (bf16x8*)y, (const bf16x8*)gamma, (const bf16x8*)beta, h, in_row_step, in_row_off, eps, nofar)
  int rc;
  // many rows (prefill): the LATE variant with NT = nv / 4 rounded up to a warp (fewer
  // live registers: 4 rows per SM instead of 2 at h = 5120; tools/kbench_ln.py, 4096
  // rows: 68.5 -> 47.9 us); few rows (decode): everything loaded before the PDL wait
  if (rows > 2 * 148 && nv > 512 && nv <= 1536) {
#define LIGER_LN_L(NT)                                                                                          \
  launch_pdl(add_ln_kernel<NT, 4, false, true>, dim3(rows), dim3(NT), 0, stream, X, A, AB, (bf16x8*)x_out,  \
             (bf16x8*)y, (const bf16x8*)gamma, (const bf16x8*)beta, h, in_row_step, in_row_off, eps, nofar)
    rc = nv <= 640 ? LIGER_LN_L(160) : nv <= 896 ? LIGER_LN_L(224) : nv <= 1152 ? LIGER_LN_L(288) : LIGER_LN_L(384);
#undef LIGER_LN_L
  } else if (nv <= 128) rc = LIGER_LN(128, 1);
  else if (nv <= 512) rc = LIGER_LN(128, 4);
  else if (nv <= 1024) rc = LIGER_LN(256, 4);
  else rc = LIGER_LN(512, 4);
#undef LIGER_LN
  return rc ? LIGER_ECUDA : 0;
}

int peer_add_layernorm_launch(const FusedARDesc& far, const void* x, const void* add_bias, void* x_out, void* y,
                              const void* gamma, const void* beta, int rows, int h, float eps, cudaStream_t stream) {
  if (rows <= 0) return 0;
  if (h % 8 || h > 16384 || far.world < 1 || far.world > 8 || !x || !y || !gamma || !beta) return LIGER_EINVAL;
  const bf16x8* X = (const bf16x8*)x;
  const bf16x8* AB = (const bf16x8*)add_bias;
  const int nv = h / 8;
#define LIGER_LN(NT, MV)                                                                                      \
  launch_pdl(add_ln_kernel<NT, MV, true>, dim3(rows), dim3(NT), 0, stream, X, (const bf16x8*)nullptr, AB,     \
             (bf16x8*)x_out, (bf16x8*)y, (const bf16x8*)gamma, (const bf16x8*)beta, h, 1, 0, eps, far)
  int rc;
  if (nv <= 128) rc = LIGER_LN(128, 1);
  else if (nv <= 512) rc = LIGER_LN(128, 4);
  else if (nv <= 1024) rc = LIGER_LN(256, 4);
  else rc = LIGER_LN(512, 4);
#undef LIGER_LN
  return rc ? LIGER_ECUDA : 0;
}

// ------------------------------------------------------------------ embedding
__global__ void embed_kernel(const int32_t* __restrict__ ids, const bf16x8* __restrict__ e_tok,
                             const bf16x8* __restrict__ e_pos, bf16x8* __restrict__ out, int h, int seq_len,
                             int start_pos) {
  pdl_enter();
  const int i = blockIdx.x;
  const int nv = h >> 3;
  const int64_t id = ids[i];
  const int pos = start_pos + (seq_len > 0 ? i % seq_len : 0) + 2;   // OPT learned positions, offset 2
  for (int v = threadIdx.x; v < nv; v += blockDim.x) {
    float a[8], b[8];
    unpack8(e_tok[id * nv + v], a);
    unpack8(e_pos[(int64_t)pos * nv + v], b);
#pragma unroll
    for (int e = 0; e < 8; ++e) a[e] += b[e];
    out[(int64_t)i * nv + v] = pack8(a);
  }
}

int embed_launch(const int32_t* ids, const void* e_tok, const void* e_pos, void* out, int rows, int h, int seq_len,
                 int start_pos, cudaStream_t stream) {
  if (rows <= 0) return 0;
  if (h % 8) return LIGER_EINVAL;
  int nt = h / 8 < 256 ? ((h / 8 + 31) / 32 * 32) : 256;
  return launch_pdl(embed_kernel, dim3(rows), dim3(nt), 0, stream, ids, (const bf16x8*)e_tok, (const bf16x8*)e_pos,
                    (bf16x8*)out, h, seq_len, start_pos)
             ? LIGER_ECUDA
             : 0;
}

// ------------------------------------------------------------------ argmax (lowest index on ties)
__device__ __forceinline__ void better(float& bv, int& bi, float v, int i) {
  if (v > bv || (v == bv && i < bi)) {
    bv = v;
    bi = i;
  }
}

__global__ void argmax_kernel(const float* __restrict__ logits, int64_t ld, int n, int idx_offset,
                              float* max_out, int32_t* idx_out) {
  __shared__ float sv[32];
  __shared__ int si[32];
  pdl_enter();
  const float* row = logits + (int64_t)blockIdx.x * ld;
  float bv = -INFINITY;
  int bi = 0x7fffffff;
  // 16-byte loads, four independent (max, index) states per thread so that several loads
  // are in flight (a scalar loop was one dependent L2 / HBM round trip per element);
  // `better` is a total order (larger value, then lower index), so the result does not
  // depend on the visiting order
  int done = 0;
  if ((reinterpret_cast<uintptr_t>(row) & 15) == 0) {
    const int n4 = n >> 2;
    const float4* r4 = reinterpret_cast<const float4*>(row);
    float v4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
    int i4[4] = {0x7fffffff, 0x7fffffff, 0x7fffffff, 0x7fffffff};
    int k = threadIdx.x;
    for (; k + 3 * (int)blockDim.x < n4; k += 4 * blockDim.x) {
      float4 q[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) q[u] = __ldcg(r4 + k + u * blockDim.x);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int e = 4 * (k + u * (int)blockDim.x);
        better(v4[u], i4[u], q[u].x, e);
        better(v4[u], i4[u], q[u].y, e + 1);
        better(v4[u], i4[u], q[u].z, e + 2);
        better(v4[u], i4[u], q[u].w, e + 3);
      }
    }
    for (; k < n4; k += blockDim.x) {
      const float4 q = __ldcg(r4 + k);
      better(v4[0], i4[0], q.x, 4 * k);
      better(v4[0], i4[0], q.y, 4 * k + 1);
      better(v4[0], i4[0], q.z, 4 * k + 2);
      better(v4[0], i4[0], q.w, 4 * k + 3);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) better(bv, bi, v4[u], i4[u]);
    done = n4 << 2;
  }
  for (int i = done + threadIdx.x; i < n; i += blockDim.x) better(bv, bi, row[i], i);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    float ov = __shfl_xor_sync(0xffffffffu, bv, o);
    int oi = __shfl_xor_sync(0xffffffffu, bi, o);
    better(bv, bi, ov, oi);
  }
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  if (l == 0) {
    sv[w] = bv;
    si[w] = bi;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < (int)(blockDim.x >> 5); ++k) better(bv, bi, sv[k], si[k]);
    max_out[blockIdx.x] = bv;
    idx_out[blockIdx.x] = bi + idx_offset;
  }
}

int argmax_launch(const float* logits, int64_t ld, int rows, int n, int idx_offset, float* max_out,
                  int32_t* idx_out, cudaStream_t stream) {
  if (rows <= 0) return 0;
  return launch_pdl(argmax_kernel, dim3(rows), dim3(1024), 0, stream, logits, ld, n, idx_offset, max_out, idx_out)
             ? LIGER_ECUDA
             : 0;
}

// vals/idx: [world][rows] gathered from every rank's vocab shard.  Writes the
// greedy token to tok_cur[r] (fed to the next decode pass) and to
// tok_out[r * out_stride + out_col] (the batch's generated sequence).
__global__ void argmax_pick_kernel(const float* vals, const int32_t* idx, int world, int rows, int32_t* tok_cur,
                                   int32_t* tok_out, int out_stride, int out_col) {
  pdl_enter();
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= rows) return;
  float bv = vals[r];
  int bi = idx[r];
  for (int w = 1; w < world; ++w) better(bv, bi, vals[w * rows + r], idx[w * rows + r]);
  tok_cur[r] = bi;
  if (tok_out) tok_out[(int64_t)r * out_stride + out_col] = bi;
}

int argmax_pick_launch(const float* vals, const int32_t* idx, int world, int rows, int32_t* tok_cur,
                       int32_t* tok_out, int out_stride, int out_col, cudaStream_t stream) {
  if (rows <= 0) return 0;
  return launch_pdl(argmax_pick_kernel, dim3((rows + 127) / 128), dim3(128), 0, stream, vals, idx, world, rows,
                    tok_cur, tok_out, out_stride, out_col)
             ? LIGER_ECUDA
             : 0;
}

// ------------------------------------------------------------------ C0 generator (device side)
// Same definition as liger_inputs/c0.py, implemented independently.
__device__ __forceinline__ uint64_t mix64_dev(uint64_t x) {
  x ^= x >> 30;
  x *= 0xBF58476D1CE4E5B9ull;
  x ^= x >> 27;
  x *= 0x94D049BB133111EBull;
  x ^= x >> 31;
  return x;
}

__global__ void c0_fill_kernel(__nv_bfloat16* dst, int rows, int cols, int64_t ld, uint64_t base, int64_t row_off,
                               int64_t col_off, int64_t irs, int64_t ics, float scale, int kind, int tiled) {
  const int64_t total = (int64_t)rows * cols;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = t / cols, c = t % cols;
    const uint64_t idx = (uint64_t)((r + row_off) * irs + (c + col_off) * ics);
    const int64_t dpos = tiled ? tiled_offset((int)(r + ld), (int)c, cols) : r * ld + c;   // tiled: ld = first row
    const uint64_t u = mix64_dev(base + idx);
    const int32_t iv = (int32_t)(u >> 40) - (1 << 23);
    const float v = (float)iv * (1.0f / 8388608.0f);
    float w;
    if (kind == 1) w = __fadd_rn(1.0f, __fmul_rn(v, 0.0625f));
    else if (kind == 2) w = __fmul_rn(v, 0.0625f);
    else w = __fmul_rn(v, scale);
    dst[dpos] = __float2bfloat16_rn(w);
  }
}

int c0_fill_launch(void* dst, int rows, int cols, int64_t ld, uint64_t seed, uint64_t tensor_id, int64_t row_off,
                   int64_t col_off, int64_t idx_row_stride, int64_t idx_col_stride, int exp, int kind,
                   cudaStream_t stream) {
  if (rows <= 0 || cols <= 0) return 0;
  const uint64_t G = 0x9E3779B97F4A7C15ull, T = 0xD1B54A32D192ED03ull;
  const uint64_t base = seed * G + tensor_id * T + G;
  const float scale = ldexpf(1.0f, exp);
  const int64_t total = (int64_t)rows * cols;
  int blocks = (int)((total + 255) / 256);
  if (blocks > 148 * 32) blocks = 148 * 32;
  const int tiled = (kind & LIGER_C0_TILED) ? 1 : 0;   // dst in the tiled GEMM weight layout
  if (tiled && cols % 64) return LIGER_EINVAL;
  c0_fill_kernel<<<blocks, 256, 0, stream>>>((__nv_bfloat16*)dst, rows, cols, ld, base, row_off, col_off,
                                             idx_row_stride, idx_col_stride, scale, kind & 3, tiled);
  return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
}

// row-major [N, K] (row stride ld) -> tiled [ceil(N/128)][K/64][128][64] (padding rows zero)
__global__ void tile_weight_kernel(const __nv_bfloat16* src, int64_t ld, __nv_bfloat16* dst, int N, int K) {
  const int64_t npad = (int64_t)(N + 127) / 128 * 128;
  const int64_t total = npad * K;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int n = (int)(t / K), k = (int)(t % K);
    dst[tiled_offset(n, k, K)] = n < N ? src[(int64_t)n * ld + k] : __float2bfloat16_rn(0.f);
  }
}
int tile_weight_launch(const void* src, int64_t ld, void* dst, int N, int K, cudaStream_t stream) {
  if (K % 64 || N <= 0) return LIGER_EINVAL;
  tile_weight_kernel<<<148 * 8, 256, 0, stream>>>((const __nv_bfloat16*)src, ld, (__nv_bfloat16*)dst, N, K);
  return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
}

// tiled element e: k = ((e / 8192) % (K / 64)) * 64 + e % 64 (kernels.h tiled_offset)
__global__ void fold_gamma_tiled_kernel(const __nv_bfloat16* src, __nv_bfloat16* dst, const __nv_bfloat16* gamma,
                                        int64_t total, int kb) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int k = (int)((e >> 13) % kb) * 64 + (int)(e & 63);
    dst[e] = __float2bfloat16_rn(__bfloat162float(src[e]) * __bfloat162float(gamma[k]));
  }
}
int fold_gamma_tiled_launch(const void* src, void* dst, const void* gamma, int N, int K, cudaStream_t stream) {
  if (K % 64 || N <= 0) return LIGER_EINVAL;
  const int64_t total = (int64_t)(N + 127) / 128 * 128 * K;
  fold_gamma_tiled_kernel<<<148 * 8, 256, 0, stream>>>((const __nv_bfloat16*)src, (__nv_bfloat16*)dst,
                                                       (const __nv_bfloat16*)gamma, total, K / 64);
  return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
}

__global__ void copy_i32_kernel(const int32_t* s, int32_t* d, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) d[i] = s[i];
}
int copy_tokens_launch(const int32_t* src, int32_t* dst, int n, cudaStream_t stream) {
  if (n <= 0) return 0;
  copy_i32_kernel<<<(n + 255) / 256, 256, 0, stream>>>(src, dst, n);
  return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
}

void preload_norm_kernels() {
  preload_kernel(add_ln_kernel<128, 1, false>);
  preload_kernel(add_ln_kernel<128, 4, false>);
  preload_kernel(add_ln_kernel<256, 4, false>);
  preload_kernel(add_ln_kernel<512, 4, false>);
  preload_kernel(add_ln_kernel<160, 4, false, true>);
  preload_kernel(add_ln_kernel<224, 4, false, true>);
  preload_kernel(add_ln_kernel<288, 4, false, true>);
  preload_kernel(add_ln_kernel<384, 4, false, true>);
  preload_kernel(add_ln_kernel<128, 1, true>);
  preload_kernel(add_ln_kernel<128, 4, true>);
  preload_kernel(add_ln_kernel<256, 4, true>);
  preload_kernel(add_ln_kernel<512, 4, true>);
  preload_kernel(embed_kernel);
  preload_kernel(argmax_kernel);
  preload_kernel(argmax_pick_kernel);
  preload_kernel(c0_fill_kernel);
  preload_kernel(tile_weight_kernel);
  preload_kernel(fold_gamma_tiled_kernel);
  preload_kernel(copy_i32_kernel);
}

LIGER_TRACE_SETTER(norm)

}  // namespace liger
