// C-ABI wrappers of the single hot-path kernels (include/liger.h "kernel entry points").
#include <cuda_runtime.h>
#include <stdio.h>
#include <string.h>
#include <mutex>
#include <string>

#include "comm.h"
#include "kernels.h"

namespace liger {

static std::mutex g_err_mu;
static std::string g_last_error;

void set_global_error(const std::string& s) {
  std::lock_guard<std::mutex> g(g_err_mu);
  g_last_error = s;
}
const char* global_error() { return g_last_error.c_str(); }

// Returns 0 if the current device is an sm_100 part, LIGER_ENODEV otherwise.
void preload_kernels() {
  preload_gemm_kernels();
  preload_norm_kernels();
  preload_attention_kernels();
  preload_comm_kernels();
  cudaGetLastError();
}

int check_device() {
  static int state = 1;   // 1 = unknown
  static std::once_flag once;
  std::call_once(once, [] {
    int dev = 0, n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
      state = LIGER_ENODEV;
      cudaGetLastError();
      return;
    }
    cudaGetDevice(&dev);
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, dev);
    state = (p.major == 10) ? 0 : LIGER_ENODEV;
    if (!state) preload_kernels();
  });
  if (state) set_global_error("liger: no sm_100 (B200) CUDA device available; there is no CPU fallback");
  return state;
}

static int ret(int rc, const char* what) {
  if (rc) {
    char buf[256];
    snprintf(buf, sizeof buf, "%s failed: status %d (%s)", what, rc, cudaGetErrorString(cudaGetLastError()));
    set_global_error(buf);
  }
  return rc;
}

}  // namespace liger

using namespace liger;

extern "C" {

int liger_op_gemm(const void* x, int64_t ldx, const void* w, int64_t ldw, void* out, int64_t ldo, int M, int N,
                  int K, int n0, int n1, const void* bias, int act, int scale_cols, float scale, int out_f32,
                  void* workspace, size_t ws_bytes, void* stream) {
  if (int rc = check_device()) return rc;
  GemmArgs a{x, ldx, w, ldw, out, ldo, M, N, K, n0, n1, bias, act, scale_cols, scale, out_f32, workspace, ws_bytes, 0};
  return ret(gemm_launch(a, (cudaStream_t)stream), "liger_op_gemm");
}

int liger_op_gemm_tiled(const void* x, int64_t ldx, const void* w, void* out, int64_t ldo, int M, int N, int K,
                        int n0, int n1, const void* bias, int act, int scale_cols, float scale, int out_f32,
                        void* workspace, size_t ws_bytes, void* stream) {
  if (int rc = check_device()) return rc;
  GemmArgs a{x, ldx, w, 64, out, ldo, M, N, K, n0, n1, bias, act, scale_cols, scale, out_f32, workspace, ws_bytes, 1};
  return ret(gemm_launch(a, (cudaStream_t)stream), "liger_op_gemm_tiled");
}

int liger_op_tile_weight(const void* w, int64_t ld, void* w_tiled, int N, int K, void* stream) {
  if (int rc = check_device()) return rc;
  return ret(tile_weight_launch(w, ld, w_tiled, N, K, (cudaStream_t)stream), "liger_op_tile_weight");
}

size_t liger_gemm_workspace_bytes(int M, int N, int K) { return gemm_workspace_bytes(M, N, K); }

int liger_gemm_plan(int M, int N, int K, int32_t* out) {
  if (!out || M <= 0 || N <= 0 || K <= 0) return LIGER_EINVAL;
  GemmPlan pl = gemm_plan(M, N, K);
  out[0] = pl.bn; out[1] = pl.m_tiles; out[2] = pl.kc; out[3] = pl.splits; out[4] = pl.stages;
  return LIGER_OK;
}

int liger_op_add_layernorm(const void* x, const void* add, const void* add_bias, void* x_out, void* y,
                           const void* gamma, const void* beta, int rows, int h, int in_row_step, int in_row_off,
                           float eps, void* stream) {
  if (int rc = check_device()) return rc;
  return ret(add_layernorm_launch(x, add, add_bias, x_out, y, gamma, beta, rows, h, in_row_step, in_row_off, eps,
                                  (cudaStream_t)stream),
             "liger_op_add_layernorm");
}

int liger_op_embed(const int32_t* ids, const void* e_tok, const void* e_pos, void* out, int rows, int h,
                   int seq_len, int start_pos, void* stream) {
  if (int rc = check_device()) return rc;
  return ret(embed_launch(ids, e_tok, e_pos, out, rows, h, seq_len, start_pos, (cudaStream_t)stream),
             "liger_op_embed");
}

int liger_op_attn_prefill(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                          int s, int heads, int d, void* stream) {
  if (int rc = check_device()) return rc;
  return ret(attn_prefill_launch(qkv, o, kv_pool, page_table, max_pages, b, s, heads, d, (cudaStream_t)stream),
             "liger_op_attn_prefill");
}

int liger_op_attn_decode(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                         int pos, int heads, int d, void* workspace, size_t ws_bytes, void* stream) {
  if (int rc = check_device()) return rc;
  return ret(attn_decode_launch(qkv, o, kv_pool, page_table, max_pages, b, pos, heads, d, workspace, ws_bytes,
                                (cudaStream_t)stream),
             "liger_op_attn_decode");
}

size_t liger_attn_decode_workspace_bytes(int b, int heads, int d, int ctx) {
  return attn_decode_workspace_bytes(b, heads, d, ctx);
}

int liger_op_argmax(const float* logits, int64_t ld, int rows, int n, int idx_offset, float* max_out,
                    int32_t* idx_out, void* stream) {
  if (int rc = check_device()) return rc;
  return ret(argmax_launch(logits, ld, rows, n, idx_offset, max_out, idx_out, (cudaStream_t)stream),
             "liger_op_argmax");
}

int liger_op_c0_fill(void* dst, int rows, int cols, int64_t ld, uint64_t seed, uint64_t tensor_id, int64_t row_off,
                     int64_t col_off, int64_t idx_row_stride, int64_t idx_col_stride, int exp, int kind,
                     void* stream) {
  if (int rc = check_device()) return rc;
  return ret(c0_fill_launch(dst, rows, cols, ld, seed, tensor_id, row_off, col_off, idx_row_stride, idx_col_stride,
                            exp, kind, (cudaStream_t)stream),
             "liger_op_c0_fill");
}

// ------------------------------------------------------------------ CUDA-IPC peer regions (transport tests)
int liger_ipc_region_create(size_t cap, void** region, uint8_t* handle) {
  if (int rc = check_device()) return rc;
  if (!region || !handle || cap == 0 || cap % 256) return LIGER_EINVAL;
  const size_t rb = peer_ar_region_bytes(cap);
  void* r = nullptr;
  if (cudaMalloc(&r, rb) != cudaSuccess) return ret(LIGER_ENOMEM, "liger_ipc_region_create");
  cudaIpcMemHandle_t h;
  if (cudaMemset(r, 0, rb) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess ||
      cudaIpcGetMemHandle(&h, r) != cudaSuccess) {
    cudaFree(r);
    return ret(LIGER_ECUDA, "liger_ipc_region_create");
  }
  memcpy(handle, &h, sizeof(h));
  *region = r;
  return LIGER_OK;
}

int liger_ipc_region_open(const uint8_t* handle, void** peer) {
  if (int rc = check_device()) return rc;
  if (!handle || !peer) return LIGER_EINVAL;
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  if (cudaIpcOpenMemHandle(peer, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
    return ret(LIGER_ECUDA, "liger_ipc_region_open");
  return LIGER_OK;
}

int liger_ipc_region_close(void* peer) { return cudaIpcCloseMemHandle(peer) == cudaSuccess ? LIGER_OK : LIGER_ECUDA; }

int liger_ipc_region_free(void* region) { return cudaFree(region) == cudaSuccess ? LIGER_OK : LIGER_ECUDA; }

int liger_op_oneshot_allreduce(void* buf, size_t count, void* const* regions, int world, int rank, size_t cap,
                               uint64_t epoch, int phases, void* stream) {
  if (int rc = check_device()) return rc;
  if (!buf || !regions || world < 1 || world > 8 || rank < 0 || rank >= world || epoch == 0 || phases < 1 ||
      phases > 3)
    return LIGER_EINVAL;
  PeerAR par;
  if (int rc = par.init(world, rank, cap, regions[rank], regions)) return ret(rc, "liger_op_oneshot_allreduce");
  par.epoch = epoch - 1;   // this call is epoch `epoch` (allreduce_bf16 pre-increments)
  return ret(par.allreduce_bf16(buf, count, (cudaStream_t)stream, phases), "liger_op_oneshot_allreduce");
}

int liger_op_oneshot_allreduce_emulated(void* const* bufs, size_t count, void* const* regions, int world, size_t cap,
                                        uint64_t epoch, void* stream) {
  if (int rc = check_device()) return rc;
  if (!bufs || !regions) return LIGER_EINVAL;
  return ret(oneshot_allreduce_emulated(bufs, count, regions, world, cap, epoch, (cudaStream_t)stream),
             "liger_op_oneshot_allreduce_emulated");
}

// the fused producer / consumer descriptor of call `epoch` on explicit regions
static int fused_desc(void* const* regions, int world, int rank, size_t cap, uint64_t epoch, size_t bytes,
                      FusedARDesc* far) {
  if (!regions || world < 1 || world > 8 || rank < 0 || rank >= world || epoch == 0) return LIGER_EINVAL;
  PeerAR par;
  if (int rc = par.init(world, rank, cap, regions[rank], regions)) return rc;
  par.epoch = epoch - 1;   // fused_begin pre-increments
  return par.fused_begin(bytes, far);
}

int liger_op_gemm_fused_ar_stage(const void* x, int64_t ldx, const void* w_tiled, int M, int N, int K,
                                 void* const* regions, int world, int rank, size_t cap, uint64_t epoch,
                                 void* workspace, size_t ws_bytes, void* stream) {
  if (int rc = check_device()) return rc;
  FusedARDesc far{};
  if (int rc = fused_desc(regions, world, rank, cap, epoch, (size_t)M * N * 2, &far))
    return ret(rc, "liger_op_gemm_fused_ar_stage");
  GemmArgs a{x, ldx, w_tiled, 64, nullptr, N, M, N, K, 0, N, nullptr, LIGER_ACT_NONE, 0, 1.0f, 0, workspace,
             ws_bytes, 1};
  a.far = &far;
  return ret(gemm_launch(a, (cudaStream_t)stream), "liger_op_gemm_fused_ar_stage");
}

int liger_op_add_layernorm_fused_ar(void* const* regions, int world, int rank, size_t cap, uint64_t epoch,
                                    const void* x, const void* add_bias, void* x_out, void* y, const void* gamma,
                                    const void* beta, int rows, int h, float eps, void* stream) {
  if (int rc = check_device()) return rc;
  FusedARDesc far{};
  if (int rc = fused_desc(regions, world, rank, cap, epoch, (size_t)rows * h * 2, &far))
    return ret(rc, "liger_op_add_layernorm_fused_ar");
  return ret(peer_add_layernorm_launch(far, x, add_bias, x_out, y, gamma, beta, rows, h, eps, (cudaStream_t)stream),
             "liger_op_add_layernorm_fused_ar");
}

}  // extern "C"

// ------------------------------------------------------------------ timeline trace (diagnostics)
static void* g_trace_rec = nullptr;
static unsigned int* g_trace_n = nullptr;
static unsigned int g_trace_cap = 0;

extern "C" int liger_trace_start(unsigned int capacity) {
  if (capacity == 0) return LIGER_EINVAL;
  if (g_trace_rec) cudaFree(g_trace_rec);
  if (g_trace_n) cudaFree(g_trace_n);
  g_trace_rec = nullptr;
  g_trace_n = nullptr;
  if (cudaMalloc(&g_trace_rec, (size_t)capacity * LIGER_TRACE_REC_BYTES) != cudaSuccess ||
      cudaMalloc((void**)&g_trace_n, sizeof(unsigned int)) != cudaSuccess ||
      cudaMemset(g_trace_n, 0, sizeof(unsigned int)) != cudaSuccess)
    return LIGER_ECUDA;
  g_trace_cap = capacity;
  TraceRec* r = (TraceRec*)g_trace_rec;
  trace_set_gemm(r, g_trace_n, capacity);
  trace_set_norm(r, g_trace_n, capacity);
  trace_set_attention(r, g_trace_n, capacity);
  return cudaDeviceSynchronize() == cudaSuccess ? LIGER_OK : LIGER_ECUDA;
}

extern "C" int liger_trace_stop(void* host_records, unsigned int capacity, unsigned int* n_out) {
  if (!g_trace_rec) return LIGER_ESTATE;
  if (cudaDeviceSynchronize() != cudaSuccess) return LIGER_ECUDA;
  trace_set_gemm(nullptr, nullptr, 0);
  trace_set_norm(nullptr, nullptr, 0);
  trace_set_attention(nullptr, nullptr, 0);
  unsigned int n = 0;
  cudaMemcpy(&n, g_trace_n, sizeof(n), cudaMemcpyDeviceToHost);
  if (n > g_trace_cap) n = g_trace_cap;
  if (n_out) *n_out = n;
  if (host_records && capacity)
    cudaMemcpy(host_records, g_trace_rec, (size_t)(n < capacity ? n : capacity) * LIGER_TRACE_REC_BYTES,
               cudaMemcpyDeviceToHost);
  cudaFree(g_trace_rec);
  cudaFree(g_trace_n);
  g_trace_rec = nullptr;
  g_trace_n = nullptr;
  return cudaGetLastError() == cudaSuccess ? LIGER_OK : LIGER_ECUDA;
}
