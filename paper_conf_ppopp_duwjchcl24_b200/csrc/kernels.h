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
  // Optional fused residual add + LayerNorm on the split-K fixup (full rows only,
  // n0 == 0 && n1 == N, splits > 1): x_out = bf16(x + bf16(out) + add_bias),
  // y = LN(x_out) * g + b; `out` itself is then not written.
  // optional: recorded on the stream between the GEMM kernel and its split-K fixup
  // (per-kernel timing; breaks the PDL overlap of the two)
  cudaEvent_t ev_mid = nullptr;
  bool* had_fixup = nullptr;
};

GemmPlan gemm_plan(int M, int N, int K);
// true when gemm_launch can fuse add + LN for this full GEMM
bool gemm_can_fuse_ln(int M, int N, int K);
size_t gemm_workspace_bytes(int M, int N, int K);
int gemm_launch(const GemmArgs& a, cudaStream_t stream);
void gemm_forget_pointer_range(const void* base, size_t bytes);

int add_layernorm_launch(const void* x, const void* add, const void* add_bias, void* x_out, void* y,
                         const void* gamma, const void* beta, int rows, int h, int in_row_step, int in_row_off,
                         float eps, cudaStream_t stream);
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
// storage offset (elements) of logical W[n, k] in the tiled layout
inline __host__ __device__ int64_t tiled_offset(int n, int k, int K) {
  return (((int64_t)(n >> 7) * (K >> 6) + (k >> 6)) << 13) + ((n & 127) << 6) + (k & 63);
}

}  // namespace liger
