// Internal declarations shared by the kernel files and the runtime.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include "../../include/liger.h"

namespace liger {

constexpr size_t GEMM_COUNTER_BYTES = 16384;   // split-K tile counters at the head of a GEMM workspace
constexpr size_t ATTN_COUNTER_BYTES = 16384;

struct GemmPlan {
  int bn, m_tiles, kc, splits, stages, smem;
};

// Descriptor of one fused all-reduce (epoch) for kernels that do the one-shot
// all-reduce's two phases themselves: the producer (row-parallel GEMM fixup) writes
// its bf16 partial into `stage` and publishes `epoch` on `flag` when its grid is
// done; the consumer (add + LN) waits for every peer's flag and sums the peers'
// staged rows in rank order -- the one-shot kernel's arithmetic.
struct FusedARDesc {
  void* stage;                        // this rank's staging buffer (epoch parity)
  unsigned long long* flag;           // this rank's epoch flag
  unsigned int* counter;              // producer-grid completion counter (zero between uses)
  const void* peer_stage[8];          // every rank's staging buffer of this epoch
  const unsigned long long* peer_flag[8];
  int world;
  unsigned long long epoch;
};

struct GemmArgs {
  const void* x;
  int64_t ldx;
  const void* w;
  int64_t ldw;
  void* out;
  int64_t ldo;
  int M, N, K, n0, n1;
  const void* bias;
  int act;
  int scale_cols;
  float scale;
  int out_f32;
  void* workspace;
  size_t ws_bytes;
  int w_tiled;   // 0: W row-major [N, K] (row stride ldw); 1: tiled [ceil(N/128)][K/64][128][64]
  // optional: recorded on the stream between the GEMM kernel and its split-K fixup
  // (per-kernel timing; breaks the PDL overlap of the two)
  cudaEvent_t ev_mid = nullptr;
  bool* had_fixup = nullptr;
  // t > 1 fused all-reduce: the fixup kernel writes the bf16 result into far->stage
  // (row-major [M, N], replacing `out`) and publishes far->epoch when the grid is done
  const FusedARDesc* far = nullptr;
  // SM budget of the persistent GEMM grid (0 = every SM): leaves SMs to a
  // communication kernel running concurrently (contention control)
  int sm_budget = 0;
  // LayerNorm folded into the GEMM (M <= 64): W holds W*gamma (per K column), the
  // epilogue applies v = rstd_m (acc - mean_m u[n]) + c[n] with the statistics of
  // the raw input rows x; u = W'.1, c = W.beta (+ bias folded by the caller, bias = 0).
  // ln_stats: [M][2] fp32 scratch the split-K fixup reads the statistics from.
  int ln_fold = 0;
  const float* ln_u = nullptr;
  const float* ln_c = nullptr;
  float* ln_stats = nullptr;
  float ln_eps = 1e-5f;
  // residual add in the final store: out[m, n] = resid[m, n] + epilogue(v) (may alias out)
  const void* resid = nullptr;
};

// Load every kernel of the library up front (called once from check_device): with CUDA's
// lazy module loading a kernel is loaded at its first launch, and loading may wait for
// kernels already running -- on the loopback backend (or any process whose running
// kernels spin on peers) a peer spinning on this rank's flag then never sees it: a
// deadlock seen in the fused all-reduce test.
void preload_kernels();
void preload_gemm_kernels();
void preload_norm_kernels();
void preload_attention_kernels();
void preload_comm_kernels();

GemmPlan gemm_plan(int M, int N, int K);
size_t gemm_workspace_bytes(int M, int N, int K);
int gemm_launch(const GemmArgs& a, cudaStream_t stream);
void gemm_forget_pointer_range(const void* base, size_t bytes);
// TMA descriptors as gemm_launch builds them (CUtensorMap, 128 B): a tiled weight
// matrix (box 64 x 128, SWIZZLE_128B) and a row-major activation [M, K] (box 64 x bn).
int gemm_weight_map(void* out_map, const void* w_tiled, int N, int K);
int gemm_act_map(void* out_map, const void* x, int M, int K, int64_t ldx, int bn);

int add_layernorm_launch(const void* x, const void* add, const void* add_bias, void* x_out, void* y,
                         const void* gamma, const void* beta, int rows, int h, int in_row_step, int in_row_off,
                         float eps, cudaStream_t stream);
// add + LN whose added operand is the all-reduce (rank-ordered fp32 sum, RNE to bf16)
// of the peers' staged partials of epoch far.epoch; waits for every peer's flag.
int peer_add_layernorm_launch(const FusedARDesc& far, const void* x, const void* add_bias, void* x_out, void* y,
                              const void* gamma, const void* beta, int rows, int h, float eps, cudaStream_t stream);
int embed_launch(const int32_t* ids, const void* e_tok, const void* e_pos, void* out, int rows, int h, int seq_len,
                 int start_pos, cudaStream_t stream);
int argmax_launch(const float* logits, int64_t ld, int rows, int n, int idx_offset, float* max_out,
                  int32_t* idx_out, cudaStream_t stream);
int argmax_pick_launch(const float* vals, const int32_t* idx, int world, int rows, int32_t* tok_cur,
                       int32_t* tok_out, int out_stride, int out_col, cudaStream_t stream);
int attn_prefill_launch(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                        int s, int heads, int d, cudaStream_t stream);
size_t attn_decode_workspace_bytes(int b, int heads, int d, int ctx);
int attn_decode_launch(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                       int pos, int heads, int d, void* workspace, size_t ws_bytes, cudaStream_t stream);
int c0_fill_launch(void* dst, int rows, int cols, int64_t ld, uint64_t seed, uint64_t tensor_id, int64_t row_off,
                   int64_t col_off, int64_t idx_row_stride, int64_t idx_col_stride, int exp, int kind,
                   cudaStream_t stream);
int copy_tokens_launch(const int32_t* src, int32_t* dst, int n, cudaStream_t stream);
int tile_weight_launch(const void* src, int64_t ld, void* dst, int N, int K, cudaStream_t stream);
// dst = bf16(src * gamma[k]) for a tiled [ceil(N/128)][K/64][128][64] weight (may alias)
int fold_gamma_tiled_launch(const void* src, void* dst, const void* gamma, int N, int K, cudaStream_t stream);
// storage offset (elements) of logical W[n, k] in the tiled layout
inline __host__ __device__ int64_t tiled_offset(int n, int k, int K) {
  return (((int64_t)(n >> 7) * (K >> 6) + (k >> 6)) << 13) + ((n & 127) << 6) + (k & 63);
}

// timeline trace (common.cuh TraceRec): per translation unit buffer installers
struct TraceRec;
void trace_set_gemm(TraceRec* rec, unsigned int* n, unsigned int cap);
void trace_set_norm(TraceRec* rec, unsigned int* n, unsigned int cap);
void trace_set_attention(TraceRec* rec, unsigned int* n, unsigned int cap);

}  // namespace liger
