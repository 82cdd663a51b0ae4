// Liger runtime: sharded weights, paged KV pool, batch state machines ("function
// assembly", §3.2), waiting queue + processing list (§3.3
// P:168), Algorithm 1 rounds with hybrid synchronization (§3.4),
// contention factor (§3.5) and runtime decomposition (§3.6).
//
// One process per GPU; tensor-parallel ranks talk through NCCL (loaded with
// dlopen, bootstrapped with a caller-broadcast ncclUniqueId).  Computation
// kernels run on the compute stream, all-reduce / all-gather pieces on the
// communication stream.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>
#include <time.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <deque>
#include <memory>
#include <string>
#include <vector>

#include "comm.h"
#include "kernels.h"
#include "planner.h"

namespace liger {
void set_global_error(const std::string& s);
const char* global_error();
int check_device();
}  // namespace liger

using namespace liger;

namespace {

double now_s() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return ts.tv_sec + ts.tv_nsec * 1e-9;
}

// weight scale exponent of a GEMM with logical fan-in K (C0): round-half-even;
// output projections (W_o, W_2) get one more halving.
int weight_exp(int K, bool out_proj = false) {
  return (int)std::nearbyint(0.5 * std::log2(3.0 / K)) - (out_proj ? 2 : 1);
}
constexpr int BIAS_EXP = -6;
// embeddings: 2^(round(-log2(h)/2) - 1) (C0, reading R16)
int emb_exp(int h) { return (int)std::nearbyint(-0.5 * std::log2((double)h)) - 1; }
constexpr uint64_t GID_ETOK = 0xFFFF00, GID_EPOS = 0xFFFF01, GID_LNFG = 0xFFFF02, GID_LNFB = 0xFFFF03;

// ------------------------------------------------------------------ ops of one pass
enum Op { OP_EMBED, OP_LN1, OP_QKV, OP_ATTN, OP_OUT, OP_AR1, OP_LN2, OP_FC1, OP_FC2, OP_AR2, OP_HEAD, OP_TOKG,
          OP_PICK, OP_RECV_X, OP_SEND_X, OP_RECV_TOK, OP_SEND_TOK, OP_COUNT };
const char* kOpName[OP_COUNT] = {"embed", "ln1",  "qkv",    "attn",   "out",      "ar1",     "ln2", "fc1", "fc2",
                                 "ar2",   "head", "tokg",   "pick",   "recv_x",   "send_x",  "recv_tok", "send_tok"};
inline bool op_is_comm(int op) {
  return op == OP_AR1 || op == OP_AR2 || op == OP_TOKG || op == OP_RECV_X || op == OP_SEND_X || op == OP_RECV_TOK ||
         op == OP_SEND_TOK;
}
inline bool op_is_gemm(int op) { return op == OP_QKV || op == OP_OUT || op == OP_FC1 || op == OP_FC2; }
inline bool op_is_ar(int op) { return op == OP_AR1 || op == OP_AR2; }

struct PassOp {
  int op, layer;
};

struct bf16p {
  void* p = nullptr;
};

struct LayerW {
  void *w_qkv, *b_qkv, *w_o, *b_o, *w_1, *b_1, *w_2, *b_2, *g1, *be1, *g2, *be2;
  // LayerNorm folded into QKV / FC1 for decode passes (t = 1): W*gamma (tiled) and
  // the fp32 epilogue vectors u = (W*gamma).1, c = W.beta + bias
  void *w_qkv_f = nullptr, *w_1_f = nullptr;
  float *u_qkv = nullptr, *c_qkv = nullptr, *u_1 = nullptr, *c_1 = nullptr;
};

struct Batch;

// Per in-flight batch slot device buffers.
struct Slot {
  void *x, *y, *qkv, *attn, *part, *hbuf, *yhead;
  void* xhead = nullptr;   // [B, h] bf16: the last token's residual after the last layer (LM-head input)
  float *logits, *vals_all;
  int32_t *idx_all, *cur_tok, *tok_out, *prompt, *page_table;
  void *gemm_ws, *attn_ws;
  size_t gemm_ws_bytes, attn_ws_bytes;
  float* ln_stats = nullptr;   // [64][2] folded-LN row statistics for the split-K fixup
  int32_t* h_page_table;   // pinned
  int32_t* h_prompt;       // pinned
  int32_t* h_tok_out;      // pinned
  cudaEvent_t free_ev;     // completes when the last batch using the slot finished
  Batch* owner = nullptr;  // batch currently (or last) assigned to the slot
  // fused all-reduce (t > 1, serial mode): the last row-parallel GEMM's fixup staged
  // its partial for epoch far.epoch; the next add + LN reduces it over the peers
  bool far_pending = false;
  FusedARDesc far{};
};

struct DurTable {
  // per op: M grid x (F+1) pieces; linear interpolation in M
  std::vector<int> mgrid;
  std::vector<std::vector<double>> t[OP_COUNT];   // t[op][mi][k] (k = 0..F)
  bool have = false;
};

struct Batch;

struct Engine;

struct Piece {
  Batch* bt;
  int pass, idx, u0, u1;
};

struct Batch {
  int64_t id;
  int b, s, n_new;
  double arrival_s, submit_s, start_s = 0;
  std::atomic<double> finish_s{0.0};
  const int32_t* dev_tokens = nullptr;   // user device tokens (tokens_on_device)
  std::vector<int32_t> host_tokens;
  bool results_to_host = true;
  int slot = -1;
  std::vector<int> pages;
  // cursor
  int pass = 0, idx = 0, done = 0;   // done = units of the current op already launched
  bool all_launched = false, finished = false, results_copied = false;
  bool captured = false;   // the LM head ran with debug capture on (liger_debug_read)
  // debug capture (liger_set_debug_capture), allocated at admission: per pass, this
  // rank's fp32 logits shard [n_new][b][V/t] and the LM-head input rows [n_new][b][h] bf16
  float* dbg_logits = nullptr;
  void* dbg_resid = nullptr;
  cudaEvent_t last_ev = nullptr;
  int last_stream = -1;
  bool has_last_ev = false;
  cudaEvent_t final_ev = nullptr;
  std::vector<int32_t> tokens;   // host copy of results
  Engine* eng = nullptr;
};

}  // namespace

struct liger_ctx {
  int world = 1, rank = 0;
  int tp = 1, tp_rank = 0;   // tensor-parallel degree / index (1 / 0 in pipeline mode)
  bool pipe = false;         // inter-operator pipeline baseline
  int l0 = 0, l1 = 0;        // this rank's layers [l0, l1) (all of them in TP modes)
  int64_t admitted = 0;      // batches admitted so far (round-robin slot assignment)
  liger_cfg cfg;
  int h, a, d, f, V, hl, al, fl, Vl, L, F;
  double cf;
  std::string err;
  Comm* comm = nullptr;   // NCCL or loopback (comm.cu); nullptr at world == 1
  cudaStream_t s_comp = nullptr, s_comm = nullptr;
  bool own_streams = true;   // false after liger_set_streams (borrowed: never destroyed)
  std::vector<LayerW> layers;
  void *e_tok = nullptr, *e_pos = nullptr, *lnf_g = nullptr, *lnf_b = nullptr;
  std::vector<void*> allocs;
  // KV pool
  void* kv = nullptr;
  int n_pages = 0, max_pages = 0;
  size_t kv_layer_elems = 0;
  std::vector<Slot> slots;
  std::vector<PassOp> pass_ops;
  // scheduler state
  std::deque<std::unique_ptr<Batch>> waiting;
  std::vector<Batch*> processing;
  std::vector<std::unique_ptr<Batch>> all_batches;   // id -> batch
  int64_t next_id = 0;
  cudaEvent_t e1 = nullptr, e2 = nullptr;
  cudaEvent_t e_end[2] = {nullptr, nullptr};   // CPU_GPU sync: end of the round on each stream
  bool have_round = false;
  // E1 placement (liger_step): host time of one round after its E1 wait (EMA, us), and a
  // fixed lead from LIGER_E1_LEAD_US (< 0: use the EMA)
  double host_round_us = 0.0;
  double e1_lead_us = -1.0;
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_next = 0;
  DurTable dur;
  double attn_scale[2] = {1.0, 1.0};   // calibration of the attention duration model (prefill, decode)
  uint32_t dbg_skip = 0;               // LIGER_DBG_SKIP=op,op,...: timing experiments only (wrong results)
  bool ar_atomic_chunks = false;
  size_t ar_decomp_min_bytes = 1 << 20;   // all-reduces below this are not decomposed
  // t > 1, serial mode (LIGER_FUSED_AR=1, needs the one-shot peer backend): the
  // all-reduce of out-proj / FC2 is fused into the GEMM's fixup (stage + publish)
  // and the following add + LN (wait + rank-ordered sum): no all-reduce kernel
  bool fused_ar = false;
  // SMs a t > 1 GEMM leaves free for a concurrent all-reduce (LIGER_GEMM_SM_RESERVE,
  // liger_set_gemm_sm_reserve); the grid size never changes a GEMM's bits
  int gemm_sm_reserve = 0;
  int th_parts = 1;
  // decode passes at t = 1 (LIGER_LN_FOLD, default on): LN1 / LN2 folded into the
  // QKV / FC1 GEMMs, residual adds into the out-proj / FC2 epilogues -- two
  // kernels and two hand-offs per layer fewer
  bool ln_fold = false;
  // t = 1, interleaved mode (default; LIGER_T1_STREAMS=0 disables): with no
  // communication to interleave, the in-flight batches' kernel lists run concurrently on
  // the two streams (batch slot parity), so one batch's latency-bound kernels
  // (attention, fixups, hand-offs) overlap another's weight-streaming GEMMs: +2 % on the
  // OPT-13B bench (24.96 vs 24.44 req/s, same box); bits per batch unchanged
  bool t1_streams = false;   // Inter-Th: projection GEMMs issued as this many partitioned kernels
  bool calibrating = false;   // liger_calibrate_cf at t = 1 (proxy communicator)
  // debug capture arena (liger_set_debug_capture): batches admitted while it is on take
  // their capture buffers from it in admission order (bump allocation, never reused)
  char* dbg_arena = nullptr;
  size_t dbg_arena_bytes = 0, dbg_arena_used = 0;
  bool dbg_capture = false;
  int n_sms = 148;
  // stats / timing
  liger_stats_t st{};
  bool timing = false;
  struct TimedLaunch {
    int cls;
    cudaEvent_t a, b;
    double bytes, flops;
  };
  std::vector<TimedLaunch> timed;
  std::vector<cudaEvent_t> timing_pool;
  size_t timing_next = 0;
  int64_t tcount[LIGER_KT_CLASSES] = {};
  double tms[LIGER_KT_CLASSES] = {}, tbytes[LIGER_KT_CLASSES] = {}, tflops[LIGER_KT_CLASSES] = {};
};

namespace {

int fail(liger_ctx* c, int rc, const std::string& msg) {
  std::string m = msg;
  if (rc == LIGER_ECUDA || rc == -1000) {   // say which CUDA error (sticky errors surface at a later launch)
    const cudaError_t e = cudaPeekAtLastError();
    if (e != cudaSuccess) m += std::string(" [") + cudaGetErrorString(e) + "]";
  }
  if (c) c->err = m;
  set_global_error(m);
  return rc;
}

#define CK(call)                                                                                   \
  do {                                                                                             \
    cudaError_t e_ = (call);                                                                       \
    if (e_ != cudaSuccess)                                                                         \
      return fail(c, LIGER_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_));             \
  } while (0)
#define CKR(call)                                                                                  \
  do {                                                                                             \
    int r_ = (call);                                                                               \
    if (r_ < 0) return fail(c, r_, std::string(#call) + " failed");                                \
  } while (0)

void* dalloc(liger_ctx* c, size_t bytes) {
  void* p = nullptr;
  if (cudaMalloc(&p, bytes ? bytes : 16) != cudaSuccess) return nullptr;
  c->allocs.push_back(p);
  return p;
}

// cudaDeviceSynchronize inside a [collective] call, followed by a barrier of the ranks:
// on the loopback backend the ranks share the GPU, and a rank that left the call and
// launched a kernel spinning on its peers (one-shot all-reduce) would keep a peer's
// device-wide synchronize from ever returning.
int device_sync_collective(liger_ctx* c) {
  const cudaError_t e = cudaDeviceSynchronize();
  if (c->comm) c->comm->barrier();
  return e == cudaSuccess ? 0 : LIGER_ECUDA;
}

// Ring of reusable events for per-batch cross-stream dependencies.  Re-recording
// an event that an older wait still references is safe: cudaStreamWaitEvent
// captures the event's state at the time of the call.
cudaEvent_t pool_event(liger_ctx* c) {
  if (c->ev_pool.empty()) {
    c->ev_pool.resize(4096);
    for (auto& e : c->ev_pool) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  }
  return c->ev_pool[c->ev_next++ % c->ev_pool.size()];
}

// ------------------------------------------------------------------ geometry helpers
// Units (1/F pieces) an op of a pass with M tokens splits into.  Decomposition
// exists to fill a communication window; at t = 1 there is none.  An
// all-reduce is a "giant kernel" worth splitting only when its message is
// large: decode-size messages (< ar_decomp_min_bytes) are latency-bound and stay
// whole -- a function of M only, identical on every rank and in every mode.
int op_units(liger_ctx* c, int op, int M) {
  if (c->F <= 1 || c->tp == 1) return 1;
  if (op_is_gemm(op)) return c->F;
  if (op_is_ar(op)) return (M >= 0 && (size_t)M * c->h * 2 < c->ar_decomp_min_bytes) ? 1 : c->F;
  return 1;
}

// All-reduce of units [u0, u1) of F of the bf16 buffer buf[E].  With atomic chunks
// (t > 2 over NCCL, whose reduction order depends on the message), every unit is
// its own collective, so a piece of k units and the whole all-reduce produce the
// same bits (R9).
int issue_ar(liger_ctx* c, void* buf, size_t E, int u0, int u1, int F, cudaStream_t st) {
  if (c->ar_atomic_chunks && F > 1) {
    for (int u = u0; u < u1; ++u) {
      const size_t e0 = E * u / F, e1 = E * (u + 1) / F;
      if (e1 > e0)
        if (c->comm->allreduce((char*)buf + e0 * 2, e1 - e0, CD_BF16, CO_SUM, st)) return LIGER_ENCCL;
    }
    return 0;
  }
  const size_t e0 = E * u0 / F, e1 = E * u1 / F;
  if (e1 > e0 && c->comm->allreduce((char*)buf + e0 * 2, e1 - e0, CD_BF16, CO_SUM, st)) return LIGER_ENCCL;
  return 0;
}

int gemm_N(liger_ctx* c, int op) {
  switch (op) {
    case OP_QKV: return 3 * c->hl;
    case OP_OUT: return c->h;
    case OP_FC1: return c->fl;
    case OP_FC2: return c->h;
  }
  return 0;
}
int gemm_K(liger_ctx* c, int op) {
  switch (op) {
    case OP_QKV: return c->h;
    case OP_OUT: return c->hl;
    case OP_FC1: return c->h;
    case OP_FC2: return c->fl;
  }
  return 0;
}
// column boundary of unit u (of F) for an N-wide GEMM: multiples of 128 (the
// tiled weight layout's row tile), last = N.  Small GEMMs may get empty pieces.
int unit_col(int N, int u, int F) {
  if (u >= F) return N;
  int c = (int)((int64_t)N * u / F);
  return c / 128 * 128;
}
int pad128(int n) { return (n + 127) / 128 * 128; }

int batch_M(const Batch* bt, int pass) { return pass == 0 ? bt->b * bt->s : bt->b; }

// ------------------------------------------------------------------ durations
double model_dur(liger_ctx* c, int op, int M, int k, int ctx_len, int s_len) {
  const double F = c->F > 1 ? c->F : 1;
  const double frac = (op_units(c, op, M) > 1) ? k / F : 1.0;
  const double bw = 5.0e12, tc = 1.0e15;
  if (op_is_gemm(op)) {
    const double N = gemm_N(c, op) * frac, K = gemm_K(c, op);
    return 4e-6 + std::max(2.0 * M * N * K / tc, (N * K + M * K + M * N) * 2 / bw);
  }
  if (op_is_ar(op)) {
    const double bytes = (double)M * c->h * 2 * frac;
    return 8e-6 + bytes * 2 * (c->tp - 1) / c->tp / 600e9;
  }
  switch (op) {
    case OP_EMBED:
    case OP_LN1:
    case OP_LN2: return 3e-6 + (double)M * c->h * 2 * 3 / bw;
    case OP_ATTN:
      if (s_len > 0) return 5e-6 + 4.0 * M * s_len * c->al * c->d / 2 / 3e14;
      return 5e-6 + 4.0 * M * ctx_len * c->al * c->d / bw;
    case OP_HEAD: return 10e-6 + (double)c->Vl * c->h * 2 / bw;
    case OP_TOKG: return 10e-6;
    case OP_PICK: return 2e-6;
  }
  return 5e-6;
}

double table_dur(liger_ctx* c, int op, int M, int k) {
  const DurTable& T = c->dur;
  if (!T.have || T.t[op].empty()) return -1;
  const auto& g = T.mgrid;
  auto at = [&](size_t mi) { return T.t[op][mi][k]; };
  double v;
  if (M <= g.front()) {
    v = at(0);
  } else if (M >= g.back()) {
    v = at(g.size() - 1) * (double)M / g.back();
  } else {
    size_t i = 1;
    while (g[i] < M) ++i;
    const double w = (double)(M - g[i - 1]) / (g[i] - g[i - 1]);
    if (at(i - 1) <= 0 || at(i) <= 0) return -1;
    v = at(i - 1) * (1 - w) + at(i) * w;
  }
  return v > 0 ? v : -1;
}

double op_dur(liger_ctx* c, const Batch* bt, int pass, int op, int k) {
  const int M = batch_M(bt, pass);
  const int ctx_len = bt->s + pass;
  const int s_len = pass == 0 ? bt->s : 0;
  if (op == OP_ATTN) {
    const double m = model_dur(c, op, M, k, ctx_len, s_len);
    return m * (s_len > 0 ? c->attn_scale[0] : c->attn_scale[1]);
  }
  const int kk = op_units(c, op, M) > 1 ? k : std::max(1, c->F);
  const double t = table_dur(c, op, M, kk);
  return t > 0 ? t : model_dur(c, op, M, k, ctx_len, s_len);
}

// ------------------------------------------------------------------ timing instrumentation
void timed_begin(liger_ctx* c, cudaStream_t s, cudaEvent_t* a) {
  if (!c->timing) return;
  if (c->timing_next + 3 > c->timing_pool.size()) {
    for (int i = 0; i < 256; ++i) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      c->timing_pool.push_back(e);
    }
  }
  *a = c->timing_pool[c->timing_next++];
  cudaEventRecord(*a, s);
}
// a spare timing event (recorded by gemm_launch between the GEMM kernel and its fixup)
cudaEvent_t timed_mid(liger_ctx* c) {
  if (!c->timing) return nullptr;
  return c->timing_pool[c->timing_next++];
}
void timed_end(liger_ctx* c, cudaStream_t s, cudaEvent_t a, int cls, double bytes, double flops) {
  if (!c->timing) return;
  cudaEvent_t b = c->timing_pool[c->timing_next++];
  cudaEventRecord(b, s);
  c->timed.push_back({cls, a, b, bytes, flops});
}
void timing_flush(liger_ctx* c) {
  if (c->timed.empty()) return;
  cudaStreamSynchronize(c->s_comp);   // this rank's streams only (peers may be running spinning kernels)
  cudaStreamSynchronize(c->s_comm);
  for (auto& t : c->timed) {
    float ms = 0;
    cudaEventElapsedTime(&ms, t.a, t.b);
    c->tcount[t.cls]++;
    c->tms[t.cls] += ms;
    c->tbytes[t.cls] += t.bytes;
    c->tflops[t.cls] += t.flops;
  }
  c->timed.clear();
  c->timing_next = 0;
}

// ------------------------------------------------------------------ launching one piece
// add + LN over the peers' staged partials of a fused all-reduce epoch
static int peer_add_ln(liger_ctx* c, Slot& S, const void* bias, const void* gamma, const void* beta, int M,
                       cudaStream_t st) {
  S.far_pending = false;
  return peer_add_layernorm_launch(S.far, S.x, bias, S.x, S.y, gamma, beta, M, c->h, c->cfg.ln_eps, st);
}

int launch_piece(liger_ctx* c, Batch* bt, int pass, int pidx, int u0, int u1, cudaStream_t st) {
  const PassOp po = c->pass_ops[pidx];
  Slot& S = c->slots[bt->slot];
  const int M = batch_M(bt, pass);
  const int h = c->h;
  const float eps = c->cfg.ln_eps;
  // decode pass with LayerNorm folded into the GEMMs: up to 16 tokens, whose row
  // statistics every single-chunk GEMM CTA computes within its mainloop (measured:
  // decode pass -2.5 % at b = 2..8; at b = 32 (generative) the statistics outlast
  // the QKV mainloop: 1492 vs 1506 seq/s folded vs not)
  static const int fold_max = getenv("LIGER_LN_FOLD_MAX") ? atoi(getenv("LIGER_LN_FOLD_MAX")) : 16;
  const bool fold = c->ln_fold && M <= std::min(fold_max, 64);
  const int li = po.layer;
  const LayerW* W = li >= 0 ? &c->layers[li] : nullptr;
  int rc = 0;
  cudaEvent_t ta = nullptr;
  if (c->dbg_skip & (1u << po.op)) return 0;
  switch (po.op) {
    case OP_EMBED: {
      const int32_t* ids = pass == 0 ? (bt->dev_tokens ? bt->dev_tokens : S.prompt) : S.cur_tok;
      rc = embed_launch(ids, c->e_tok, c->e_pos, S.x, M, h, pass == 0 ? bt->s : 0, pass == 0 ? 0 : bt->s + pass - 1,
                        st);
      c->st.gpu_launches++;
      break;
    }
    case OP_LN1: {
      if (fold) break;   // folded into the QKV GEMM (the residual add happened in FC2's epilogue)
      timed_begin(c, st, &ta);
      if (li == c->l0)   // first layer of the model / of this pipeline stage: x is complete
        rc = add_layernorm_launch(S.x, nullptr, nullptr, nullptr, S.y, W->g1, W->be1, M, h, 1, 0, eps, st);
      else if (S.far_pending)
        rc = peer_add_ln(c, S, c->layers[li - 1].b_2, W->g1, W->be1, M, st);
      else
        rc = add_layernorm_launch(S.x, S.part, c->layers[li - 1].b_2, S.x, S.y, W->g1, W->be1, M, h, 1, 0, eps, st);
      timed_end(c, st, ta, LIGER_KT_LN, (double)M * h * 2 * (li == c->l0 ? 2 : 4), 0);
      c->st.gpu_launches++;
      break;
    }
    case OP_LN2: {
      if (fold) break;   // folded into the FC1 GEMM (the residual add happened in out-proj's epilogue)
      timed_begin(c, st, &ta);
      if (S.far_pending)
        rc = peer_add_ln(c, S, W->b_o, W->g2, W->be2, M, st);
      else
        rc = add_layernorm_launch(S.x, S.part, W->b_o, S.x, S.y, W->g2, W->be2, M, h, 1, 0, eps, st);
      timed_end(c, st, ta, LIGER_KT_LN, (double)M * h * 2 * 4, 0);
      c->st.gpu_launches++;
      break;
    }
    case OP_QKV:
    case OP_OUT:
    case OP_FC1:
    case OP_FC2: {
      const int N = gemm_N(c, po.op), K = gemm_K(c, po.op);
      const int F = op_units(c, po.op, M);
      GemmArgs g{};
      g.M = M; g.N = N; g.K = K;
      g.n0 = unit_col(N, u0, F);
      g.n1 = unit_col(N, u1, F);
      g.workspace = S.gemm_ws; g.ws_bytes = S.gemm_ws_bytes;
      g.scale = 1.0f;
      g.w_tiled = 1;
      if (c->gemm_sm_reserve > 0 && (c->comm || c->calibrating || c->t1_streams))
        g.sm_budget = std::max(1, c->n_sms - c->gemm_sm_reserve);
      if (po.op == OP_QKV) {
        g.x = S.y; g.ldx = h; g.w = W->w_qkv; g.ldw = K; g.out = S.qkv; g.ldo = N; g.bias = W->b_qkv;
        g.scale_cols = c->hl; g.scale = 1.0f / sqrtf((float)c->d);
      } else if (po.op == OP_OUT) {
        g.x = S.attn; g.ldx = c->hl; g.w = W->w_o; g.ldw = K; g.out = S.part; g.ldo = h;
      } else if (po.op == OP_FC1) {
        g.x = S.y; g.ldx = h; g.w = W->w_1; g.ldw = K; g.out = S.hbuf; g.ldo = N; g.bias = W->b_1;
        g.act = c->cfg.act;
      } else {
        g.x = S.hbuf; g.ldx = c->fl; g.w = W->w_2; g.ldw = K; g.out = S.part; g.ldo = h;
      }
      if (fold) {
        if (po.op == OP_QKV || po.op == OP_FC1) {   // LN folded: raw residual rows in, statistics in-kernel
          const bool q = po.op == OP_QKV;
          g.x = S.x;
          g.w = q ? W->w_qkv_f : W->w_1_f;
          g.ln_fold = 1;
          g.ln_u = q ? W->u_qkv : W->u_1;
          g.ln_c = q ? W->c_qkv : W->c_1;
          g.bias = nullptr;   // in ln_c
          g.ln_stats = S.ln_stats;
          g.ln_eps = eps;
        } else {   // residual stream updated in the epilogue: x += P + bias
          g.out = S.x;
          g.resid = S.x;
          g.bias = po.op == OP_OUT ? W->b_o : W->b_2;
        }
      }
      if (c->tp > 1 && c->fused_ar && c->cfg.mode == LIGER_MODE_SERIAL && u0 == 0 && u1 == F &&
          (po.op == OP_OUT || (po.op == OP_FC2 && li + 1 < c->l1))) {
        const GemmPlan pl = gemm_plan(M, N, K);
        PeerAR* par = c->comm ? c->comm->peer_ar(st) : nullptr;
        if (pl.splits > 1 && par && (size_t)M * N * 2 <= par->cap) {
          if (par->fused_begin((size_t)M * N * 2, &S.far)) return fail(c, LIGER_ECUDA, "fused all-reduce setup");
          g.far = &S.far;
          S.far_pending = true;
        }
      }
      timed_begin(c, st, &ta);
      cudaEvent_t tmid = timed_mid(c);
      bool fix = false;
      g.ev_mid = tmid;
      g.had_fixup = &fix;
      if (c->th_parts > 1) {
        // Inter-Th: the GEMM as th_parts partitioned kernels over its output columns
        // (each a full-plan slice: the bits of the whole GEMM)
        const int P = c->th_parts, a0 = g.n0, a1 = g.n1;
        for (int r = 0; r < P && !rc; ++r) {
          g.n0 = std::max(a0, unit_col(N, r, P));
          g.n1 = std::min(a1, r + 1 == P ? N : unit_col(N, r + 1, P));
          if (g.n1 > g.n0) rc = gemm_launch(g, st);
        }
        c->st.gpu_launches += P - 1;
      } else {
        rc = gemm_launch(g, st);
      }
      const double n = g.n1 - g.n0;
      if (c->timing) {
        // GEMM kernel: algorithmic bytes / flops; fixup: fp32 partials read + output written
        c->timed.push_back({M <= 64 ? LIGER_KT_GEMM_DECODE : LIGER_KT_GEMM_PREFILL, ta, tmid,
                            (n * K + (double)M * K + (double)M * n) * 2, 2.0 * M * n * K});
        if (fix) {
          const GemmPlan pl = gemm_plan(M, N, K);
          timed_end(c, st, tmid, LIGER_KT_FIXUP,
                    (double)pl.splits * M * n * 4 + (double)M * n * 2, 0);
        }
      }
      c->st.gpu_launches += fix ? 2 : 1;   // the GEMM (+ its split-K fixup kernel)
      break;
    }
    case OP_ATTN: {
      void* pool = (char*)c->kv + (size_t)(li - c->l0) * c->kv_layer_elems * 2;
      timed_begin(c, st, &ta);
      if (pass == 0) {
        rc = attn_prefill_launch(S.qkv, S.attn, pool, S.page_table, c->max_pages, bt->b, bt->s, c->al, c->d, st);
        timed_end(c, st, ta, LIGER_KT_ATTN, (double)M * c->hl * 2 * 6, 2.0 * bt->b * c->al * c->d * (double)bt->s * bt->s);
      } else {
        const int pos = bt->s + pass - 1;
        rc = attn_decode_launch(S.qkv, S.attn, pool, S.page_table, c->max_pages, bt->b, pos, c->al, c->d,
                                S.attn_ws, S.attn_ws_bytes, st);
        timed_end(c, st, ta, LIGER_KT_ATTN, (double)bt->b * c->hl * 2 * 2 * (pos + 1),
                  4.0 * bt->b * c->al * c->d * (double)(pos + 1));
      }
      c->st.gpu_launches++;
      break;
    }
    case OP_AR1:
    case OP_AR2: {
      if (S.far_pending) break;   // fused into the preceding GEMM and the next add + LN
      const int F = op_units(c, po.op, M);
      const size_t E = (size_t)M * h;
      timed_begin(c, st, &ta);
      const double h0 = now_s();
      if (issue_ar(c, S.part, E, u0, u1, F, st)) return fail(c, LIGER_ENCCL, c->comm->err);
      c->st.comm_host_us += (now_s() - h0) * 1e6;
      timed_end(c, st, ta, LIGER_KT_ALLREDUCE, (double)(E * u1 / F - E * u0 / F) * 2, 0);
      c->st.comm_kernels++;
      c->st.gpu_launches++;
      break;
    }
    case OP_HEAD: {
      const int b = bt->b;
      const LayerW& Wl = c->layers[c->L - 1];
      // residual add of the last layer + final LN on the last token of each sequence
      const int step = pass == 0 ? bt->s : 1, off = pass == 0 ? bt->s - 1 : 0;
      // (folded decode pass: the last FC2 already added its output and bias to x)
      rc = add_layernorm_launch(S.x, fold ? nullptr : S.part, fold ? nullptr : Wl.b_2, S.xhead, S.yhead, c->lnf_g,
                                c->lnf_b, b, h, step, off, eps, st);
      if (rc) break;
      GemmArgs g{};
      g.x = S.yhead; g.ldx = h;
      g.w = (char*)c->e_tok + (size_t)c->tp_rank * c->Vl * h * 2; g.ldw = h;
      g.out = S.logits; g.ldo = c->Vl; g.out_f32 = 1;
      g.M = b; g.N = c->Vl; g.K = h; g.n0 = 0; g.n1 = c->Vl; g.scale = 1.0f;
      g.workspace = S.gemm_ws; g.ws_bytes = S.gemm_ws_bytes;
      timed_begin(c, st, &ta);
      rc = gemm_launch(g, st);
      timed_end(c, st, ta, LIGER_KT_LMHEAD, ((double)c->Vl * h + (double)b * h) * 2 + (double)b * c->Vl * 4,
                2.0 * b * c->Vl * h);
      if (rc) break;
      rc = argmax_launch(S.logits, c->Vl, b, c->Vl, c->tp_rank * c->Vl, S.vals_all + (size_t)c->tp_rank * b,
                         S.idx_all + (size_t)c->tp_rank * b, st);
      if (rc) break;
      c->st.gpu_launches += 3;
      if (bt->dbg_logits) {   // test readback (liger_debug_read): copies only
        cudaMemcpyAsync(bt->dbg_logits + (size_t)pass * b * c->Vl, S.logits, (size_t)b * c->Vl * 4,
                        cudaMemcpyDeviceToDevice, st);
        cudaMemcpyAsync((char*)bt->dbg_resid + (size_t)pass * b * h * 2, S.xhead, (size_t)b * h * 2,
                        cudaMemcpyDeviceToDevice, st);
        bt->captured = true;
      }
      if (c->tp == 1) {
        rc = argmax_pick_launch(S.vals_all, S.idx_all, 1, b, S.cur_tok, S.tok_out, bt->n_new, pass, st);
        c->st.gpu_launches++;
      }
      break;
    }
    case OP_TOKG: {
      const int b = bt->b;
      const double h0 = now_s();
      if (c->comm->allgather2(S.vals_all + (size_t)c->rank * b, S.vals_all, b, CD_F32,
                              S.idx_all + (size_t)c->rank * b, S.idx_all, b, CD_I32, st))
        return fail(c, LIGER_ENCCL, c->comm->err);
      c->st.comm_host_us += (now_s() - h0) * 1e6;
      c->st.comm_kernels++;
      c->st.gpu_launches++;
      break;
    }
    case OP_PICK: {
      rc = argmax_pick_launch(S.vals_all, S.idx_all, c->tp, bt->b, S.cur_tok, S.tok_out, bt->n_new, pass, st);
      c->st.gpu_launches++;
      break;
    }
    // ---- inter-operator pipeline baseline: stage-to-stage activations and the token
    case OP_RECV_X: {
      if (c->comm->recv(S.x, (size_t)M * h * 2, c->rank - 1, st)) return fail(c, LIGER_ENCCL, c->comm->err);
      c->st.comm_kernels++;
      break;
    }
    case OP_SEND_X: {
      // complete the residual stream of the stage's last layer (x += FC2 + b_2), then send it on
      // (a folded decode pass did that in FC2's epilogue)
      if (!fold) {
        rc = add_layernorm_launch(S.x, S.part, c->layers[c->l1 - 1].b_2, S.x, S.y, c->lnf_g, c->lnf_b, M, h, 1, 0,
                                  eps, st);
        if (rc) break;
        c->st.gpu_launches++;
      }
      if (c->comm->send(S.x, (size_t)M * h * 2, c->rank + 1, st)) return fail(c, LIGER_ENCCL, c->comm->err);
      c->st.comm_kernels++;
      break;
    }
    case OP_RECV_TOK: {   // stage 0, pass > 0: the token of the previous pass from the last stage
      if (pass == 0) break;
      if (c->comm->recv(S.cur_tok, (size_t)bt->b * 4, c->world - 1, st)) return fail(c, LIGER_ENCCL, c->comm->err);
      c->st.comm_kernels++;
      rc = argmax_pick_launch(S.vals_all, S.cur_tok, 1, bt->b, S.cur_tok, S.tok_out, bt->n_new, pass - 1, st);
      c->st.gpu_launches++;
      break;
    }
    case OP_SEND_TOK: {   // last stage: the new token back to stage 0 (not after the final pass)
      if (pass == bt->n_new - 1) break;
      if (c->comm->send(S.cur_tok, (size_t)bt->b * 4, 0, st)) return fail(c, LIGER_ENCCL, c->comm->err);
      c->st.comm_kernels++;
      break;
    }
  }
  if (rc < 0) return fail(c, rc, std::string("launch of ") + kOpName[po.op] + " failed");
  return 0;
}

// ------------------------------------------------------------------ batch cursor for the planner
struct BatchCursor : Cursor {
  liger_ctx* c;
  Batch* bt;
  std::vector<Piece>* out;
  BatchCursor(liger_ctx* c_, Batch* b_, std::vector<Piece>* o) : c(c_), bt(b_), out(o) {}
  bool empty() const override { return bt->all_launched; }
  int cur_op() const { return c->pass_ops[bt->idx].op; }
  int head_type() const override { return op_is_comm(cur_op()) ? KT_COMM : KT_COMPUTE; }
  int units() const { return op_units(c, cur_op(), batch_M(bt, bt->pass)); }
  int head_left() const override { return units() - bt->done; }
  bool head_decomposable() const override { return units() > 1; }
  double head_dur(int k) const override {
    // duration of units [done, done + k): profiled piece of k units
    return op_dur(c, bt, bt->pass, cur_op(), k);
  }
  int next_type() const override {
    int pass = bt->pass, idx = bt->idx + 1;
    if (idx >= (int)c->pass_ops.size()) {
      idx = 0;
      ++pass;
    }
    if (pass >= bt->n_new) return -1;
    return op_is_comm(c->pass_ops[idx].op) ? KT_COMM : KT_COMPUTE;
  }
  int64_t take(int k) override {
    Piece p{bt, bt->pass, bt->idx, bt->done, bt->done + k};
    out->push_back(p);
    bt->done += k;
    if (bt->done >= units()) {
      bt->done = 0;
      if (++bt->idx >= (int)c->pass_ops.size()) {
        bt->idx = 0;
        if (++bt->pass >= bt->n_new) bt->all_launched = true;
      }
    }
    return (int64_t)out->size() - 1;
  }
};

// ------------------------------------------------------------------ admission / completion
void reap(liger_ctx* c);

// Admission is a pure function of the submit order and of the launch state (slots
// with a fixed page range each, taken round-robin from the next one, skipping slots
// whose owner has kernels left to launch -- the same on every rank, since all ranks
// make identical plans), so every rank admits the same batch into the same slot at
// the same liger_step and all ranks issue identical plans / collectives.  A slot is
// reusable once its previous owner has launched everything (its final event is
// recorded); the host waits for that event before overwriting the slot's pinned
// staging buffers.  Returns false (batch stays waiting) when no slot is reusable.
bool admit(liger_ctx* c, Batch* bt) {
  const int ns = (int)c->slots.size();
  int slot = -1;
  for (int i = 0; i < ns && slot < 0; ++i) {
    const int s = (int)((c->admitted + i) % ns);
    const Batch* o = c->slots[s].owner;
    if (!o || o->all_launched) slot = s;
  }
  if (slot < 0) return false;
  c->admitted = slot + 1;
  Slot& S = c->slots[slot];
  if (S.owner && !S.owner->finished) {
    cudaEventSynchronize(S.owner->final_ev);
    reap(c);
  }
  S.owner = bt;
  bt->slot = slot;
  const int ppseq = (bt->s + bt->n_new + LIGER_KV_BLOCK - 1) / LIGER_KV_BLOCK;
  const int base = slot * c->cfg.max_batch * c->max_pages;
  for (int i = 0; i < bt->b; ++i)
    for (int p = 0; p < ppseq; ++p) S.h_page_table[i * c->max_pages + p] = base + i * c->max_pages + p;
  // inputs for the first kernels: wait until the previous user of the slot is done
  const int si = (c->t1_streams && !c->timing) ? (slot & 1) : 0;
  cudaStream_t st = si ? c->s_comm : c->s_comp;
  cudaStreamWaitEvent(st, S.free_ev, 0);
  cudaMemcpyAsync(S.page_table, S.h_page_table, sizeof(int32_t) * bt->b * c->max_pages, cudaMemcpyHostToDevice, st);
  if (!bt->dev_tokens) {
    memcpy(S.h_prompt, bt->host_tokens.data(), sizeof(int32_t) * bt->b * bt->s);
    cudaMemcpyAsync(S.prompt, S.h_prompt, sizeof(int32_t) * bt->b * bt->s, cudaMemcpyHostToDevice, st);
  }
  bt->last_stream = si;
  bt->last_ev = pool_event(c);
  cudaEventRecord(bt->last_ev, st);
  bt->has_last_ev = true;
  if (c->dbg_capture && c->l1 == c->L) {   // test readback buffers of this batch (liger_debug_read)
    // (from the preallocated arena: no cudaMalloc while peers may spin in one-shot kernels)
    const size_t nl = ((size_t)bt->n_new * bt->b * c->Vl * 4 + 255) / 256 * 256;
    const size_t nr = ((size_t)bt->n_new * bt->b * c->h * 2 + 255) / 256 * 256;
    if (c->dbg_arena_used + nl + nr <= c->dbg_arena_bytes) {
      bt->dbg_logits = reinterpret_cast<float*>(c->dbg_arena + c->dbg_arena_used);
      bt->dbg_resid = c->dbg_arena + c->dbg_arena_used + nl;
      c->dbg_arena_used += nl + nr;
    }
  }
  bt->host_tokens.clear();   // staged in the slot's pinned buffer (copied in stream order)
  bt->host_tokens.shrink_to_fit();
  return true;
}

void CUDART_CB host_finish(void* p) {
  Batch* bt = static_cast<Batch*>(p);
  bt->finish_s.store(now_s());
}

void finalize_batch_launch(liger_ctx* c, Batch* bt, cudaStream_t st) {
  Slot& S = c->slots[bt->slot];
  if (bt->results_to_host)
    cudaMemcpyAsync(S.h_tok_out, S.tok_out, sizeof(int32_t) * bt->b * bt->n_new, cudaMemcpyDeviceToHost, st);
  cudaEventRecord(bt->final_ev, st);
  cudaEventRecord(S.free_ev, st);
  cudaLaunchHostFunc(st, host_finish, bt);
}

// a finished batch releases its pages and slot (host side)
void reap(liger_ctx* c) {
  for (auto& up : c->all_batches) {
    Batch* bt = up.get();
    if (!bt || !bt->all_launched || bt->finished) continue;
    if (cudaEventQuery(bt->final_ev) != cudaSuccess) continue;
    bt->finished = true;
    Slot& S = c->slots[bt->slot];
    if (bt->results_to_host) {
      bt->tokens.assign(S.h_tok_out, S.h_tok_out + bt->b * bt->n_new);
      bt->results_copied = true;
    }
    if (bt->finish_s.load() == 0) bt->finish_s.store(now_s());
    cudaEventDestroy(bt->final_ev);   // complete; nothing waits on it any more
    bt->final_ev = nullptr;
  }
}

void update_list(liger_ctx* c) {
  // completed batches leave the processing list; waiting batches are admitted FIFO.
  std::vector<Batch*> keep;
  for (Batch* b : c->processing)
    if (!b->all_launched) keep.push_back(b);
  c->processing.swap(keep);
  const int cap = c->cfg.mode == LIGER_MODE_SERIAL ? 1 : std::max(1, c->cfg.max_inflight);
  reap(c);
  while ((int)c->processing.size() < cap && !c->waiting.empty()) {
    Batch* bt = c->waiting.front().get();
    if (!admit(c, bt)) break;
    c->processing.push_back(bt);
    c->all_batches[bt->id] = std::move(c->waiting.front());
    c->waiting.pop_front();
  }
}

// stream index: 0 = compute, 1 = communication
cudaStream_t stream_of(liger_ctx* c, int idx) { return idx ? c->s_comm : c->s_comp; }

// Launch a run of pieces on stream `si`, honouring each batch's cross-stream data dependency.
int launch_run(liger_ctx* c, const std::vector<Piece>& pieces, const std::vector<int>& which, int si) {
  cudaStream_t st = stream_of(c, si);
  for (size_t j = 0; j < which.size(); ++j) {
    const Piece& p = pieces[which[j]];
    Batch* bt = p.bt;
    if (bt->has_last_ev && bt->last_stream != si) cudaStreamWaitEvent(st, bt->last_ev, 0);
    if (bt->start_s == 0) bt->start_s = now_s();
    int rc = launch_piece(c, bt, p.pass, p.idx, p.u0, p.u1, st);
    if (rc < 0) return rc;
    c->st.kernels++;
    const int units = op_units(c, c->pass_ops[p.idx].op, batch_M(bt, p.pass));
    if (p.u1 - p.u0 < units) c->st.split_pieces++;
    const bool batch_changes = (j + 1 == which.size()) || pieces[which[j + 1]].bt != bt;
    if (batch_changes) {
      bt->last_ev = pool_event(c);
      cudaEventRecord(bt->last_ev, st);
      bt->last_stream = si;
      bt->has_last_ev = true;
    }
    if (bt->all_launched && p.pass == bt->n_new - 1 && p.idx == (int)c->pass_ops.size() - 1 && p.u1 == units)
      finalize_batch_launch(c, bt, st);
  }
  return 0;
}

}  // namespace

// ================================================================== C ABI
extern "C" {

int liger_loopback_unique_id(uint8_t* uid) {
  if (!uid) return LIGER_EINVAL;
  make_loopback_uid(uid);
  return LIGER_OK;
}

int liger_nccl_unique_id(uint8_t* uid) {
  if (!uid) return LIGER_EINVAL;
  if (!nccl().ok) return fail(nullptr, LIGER_ENCCL, "NCCL library not loadable");
  ncclUniqueId id;
  if (nccl().GetUniqueId(&id) != ncclSuccess) return fail(nullptr, LIGER_ENCCL, "ncclGetUniqueId failed");
  memcpy(uid, &id, sizeof(id));
  return LIGER_OK;
}

int liger_init(int world, int rank, const liger_cfg* cfg, const uint8_t* nccl_uid, liger_ctx** out) {
  if (!cfg || !out || world < 1 || rank < 0 || rank >= world) return LIGER_EINVAL;
  if (int rc = check_device()) return rc;
  auto cp = std::make_unique<liger_ctx>();
  liger_ctx* c = cp.get();
  c->world = world;
  c->rank = rank;
  c->cfg = *cfg;
  c->h = cfg->hidden; c->a = cfg->n_heads; c->f = cfg->ffn; c->V = cfg->vocab; c->L = cfg->n_layers;
  c->pipe = cfg->mode == LIGER_MODE_PIPELINE || cfg->mode == LIGER_MODE_PIPELINE_TH;
  c->th_parts = cfg->mode == LIGER_MODE_PIPELINE_TH ? world : 1;
  c->tp = c->pipe ? 1 : world;
  c->tp_rank = c->pipe ? 0 : rank;
  const int tp = c->tp;
  if (c->a <= 0 || c->h % c->a || c->a % tp || c->f % tp || c->V % tp || c->h % 64)
    return fail(nullptr, LIGER_EINVAL, "liger_init: shapes not divisible by the TP degree");
  if (c->pipe && c->L < world) return fail(nullptr, LIGER_EINVAL, "liger_init: fewer layers than pipeline stages");
  c->d = c->h / c->a;
  if (c->d != 64 && c->d != 128) return fail(nullptr, LIGER_EINVAL, "liger_init: head_dim must be 64 or 128");
  c->hl = c->h / tp; c->al = c->a / tp; c->fl = c->f / tp; c->Vl = c->V / tp;
  // layers of this rank: all (TP) or an equal pipeline stage, the first L % world stages one more (AMB-29)
  if (c->pipe) {
    const int base = c->L / world, extra = c->L % world;
    c->l0 = rank * base + std::min(rank, extra);
    c->l1 = c->l0 + base + (rank < extra ? 1 : 0);
  } else {
    c->l0 = 0;
    c->l1 = c->L;
  }
  if (cfg->mode < LIGER_MODE_SERIAL || cfg->mode > LIGER_MODE_PIPELINE_TH)
    return fail(nullptr, LIGER_EINVAL, "liger_init: unknown mode");
  if (cfg->sync_mode < LIGER_SYNC_HYBRID || cfg->sync_mode > LIGER_SYNC_INTER_STREAM)
    return fail(nullptr, LIGER_EINVAL, "liger_init: unknown sync_mode");
  c->F = std::max(1, cfg->decomp_factor);
  c->cf = cfg->contention_factor > 0 ? cfg->contention_factor : 1.0;
  if (const char* sk = getenv("LIGER_DBG_SKIP")) {
    std::string all = std::string(",") + sk + ",";
    for (int o = 0; o < OP_COUNT; ++o)
      if (all.find(std::string(",") + kOpName[o] + ",") != std::string::npos) c->dbg_skip |= 1u << o;
  }
  if (const char* fa = getenv("LIGER_FUSED_AR")) c->fused_ar = atoi(fa) != 0;
  if (const char* sr = getenv("LIGER_GEMM_SM_RESERVE")) c->gemm_sm_reserve = atoi(sr);
  {
    const char* ts = getenv("LIGER_T1_STREAMS");
    c->t1_streams = (ts ? atoi(ts) != 0 : true) && c->tp == 1 && !c->pipe && cfg->mode == LIGER_MODE_INTERLEAVED;
  }
  {
    const char* lf = getenv("LIGER_LN_FOLD");
    c->ln_fold = (lf ? atoi(lf) != 0 : true) && c->tp == 1;
  }
  {
    int dev = 0, n = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && n > 0) c->n_sms = n;
  }
  const char* env = getenv("LIGER_AR_ATOMIC_CHUNKS");
  c->ar_atomic_chunks = env ? atoi(env) != 0 : (tp > 2);
  if (const char* e = getenv("LIGER_AR_DECOMP_MIN_KB")) c->ar_decomp_min_bytes = (size_t)atoll(e) * 1024;
  if (const char* e = getenv("LIGER_E1_LEAD_US")) c->e1_lead_us = atof(e);   // 0: the paper's placement
  if (world > 1) {
    if (!nccl_uid) return fail(nullptr, LIGER_EINVAL, "liger_init: nccl_uid required for world > 1");
    std::string err;
    c->comm = comm_create(world, rank, nccl_uid, &err);
    if (!c->comm) return fail(nullptr, LIGER_ENCCL, "liger_init: " + err);
  }
  int lo, hi;
  cudaDeviceGetStreamPriorityRange(&lo, &hi);
  // the communication stream gets the high priority (its kernels are short and gate the
  // other ranks); at t = 1 the two streams carry equal work (two batches): same priority
  // unless LIGER_T1_PRIO=1 (experiment)
  const bool t1_prio = getenv("LIGER_T1_PRIO") && atoi(getenv("LIGER_T1_PRIO")) != 0;
  CK(cudaStreamCreateWithPriority(&c->s_comp, cudaStreamNonBlocking, lo));
  CK(cudaStreamCreateWithPriority(&c->s_comm, cudaStreamNonBlocking, (c->t1_streams && !t1_prio) ? lo : hi));
  CK(cudaEventCreateWithFlags(&c->e1, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&c->e2, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&c->e_end[0], cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&c->e_end[1], cudaEventDisableTiming));

  // weights (this rank's shards, K-major [N_local, K])
  c->layers.resize(c->L);
  const size_t h = c->h;
  for (int l = c->l0; l < c->l1; ++l) {
    LayerW& W = c->layers[l];
    W.w_qkv = dalloc(c, (size_t)pad128(3 * c->hl) * h * 2);
    W.b_qkv = dalloc(c, 3 * c->hl * 2);
    W.w_o = dalloc(c, (size_t)pad128(c->h) * c->hl * 2);
    W.b_o = dalloc(c, h * 2);
    W.w_1 = dalloc(c, (size_t)pad128(c->fl) * h * 2);
    W.b_1 = dalloc(c, (size_t)c->fl * 2);
    W.w_2 = dalloc(c, (size_t)pad128(c->h) * c->fl * 2);
    W.b_2 = dalloc(c, h * 2);
    W.g1 = dalloc(c, h * 2); W.be1 = dalloc(c, h * 2); W.g2 = dalloc(c, h * 2); W.be2 = dalloc(c, h * 2);
    if (c->ln_fold) {
      W.w_qkv_f = dalloc(c, (size_t)pad128(3 * c->hl) * h * 2);
      W.w_1_f = dalloc(c, (size_t)pad128(c->fl) * h * 2);
      W.u_qkv = (float*)dalloc(c, (size_t)3 * c->hl * 4);
      W.c_qkv = (float*)dalloc(c, (size_t)3 * c->hl * 4);
      W.u_1 = (float*)dalloc(c, (size_t)c->fl * 4);
      W.c_1 = (float*)dalloc(c, (size_t)c->fl * 4);
      if (!W.w_qkv_f || !W.w_1_f || !W.c_1) return fail(nullptr, LIGER_ENOMEM, "liger_init: folded LN weights");
    }
    if (!W.w_qkv || !W.w_o || !W.w_1 || !W.w_2 || !W.be2)
      return fail(nullptr, LIGER_ENOMEM, "liger_init: out of device memory for weights");
  }
  c->e_tok = dalloc(c, (size_t)c->V * h * 2);
  c->e_pos = dalloc(c, (size_t)(cfg->max_pos + 2) * h * 2);
  c->lnf_g = dalloc(c, h * 2);
  c->lnf_b = dalloc(c, h * 2);
  if (!c->e_tok || !c->e_pos || !c->lnf_b) return fail(nullptr, LIGER_ENOMEM, "liger_init: embeddings");

  // slots and paged KV pool
  int nslots = (cfg->mode == LIGER_MODE_SERIAL ? 1 : std::max(1, cfg->max_inflight)) + 1;
  if (c->t1_streams) nslots += nslots & 1;   // slot parity picks the stream: keep the two balanced
  const int B = cfg->max_batch, Smax = cfg->max_seq;
  const int Mmax = B * Smax;
  c->max_pages = (Smax + cfg->max_new + LIGER_KV_BLOCK - 1) / LIGER_KV_BLOCK;
  c->n_pages = nslots * B * c->max_pages;
  c->kv_layer_elems = (size_t)c->n_pages * 2 * c->al * LIGER_KV_BLOCK * c->d;
  c->kv = dalloc(c, c->kv_layer_elems * 2 * (c->l1 - c->l0));
  if (!c->kv) return fail(nullptr, LIGER_ENOMEM, "liger_init: KV pool");
  // split-K workspace: the maximum over every token count a pass can have
  size_t ws = 0;
  for (int M = 1; M <= Mmax; ++M) {
    ws = std::max(ws, gemm_workspace_bytes(M, 3 * c->hl, c->h));
    ws = std::max(ws, gemm_workspace_bytes(M, c->h, c->hl));
    ws = std::max(ws, gemm_workspace_bytes(M, c->fl, c->h));
    ws = std::max(ws, gemm_workspace_bytes(M, c->h, c->fl));
    if (M <= B) ws = std::max(ws, gemm_workspace_bytes(M, c->Vl, c->h));
  }
  c->slots.resize(nslots);
  for (auto& S : c->slots) {
    S.x = dalloc(c, (size_t)Mmax * h * 2);
    S.y = dalloc(c, (size_t)Mmax * h * 2);
    S.qkv = dalloc(c, (size_t)Mmax * 3 * c->hl * 2);
    S.attn = dalloc(c, (size_t)Mmax * c->hl * 2);
    S.part = dalloc(c, (size_t)Mmax * h * 2);
    S.ln_stats = (float*)dalloc(c, 2 * 64 * sizeof(float));
    S.hbuf = dalloc(c, (size_t)Mmax * c->fl * 2);
    S.yhead = dalloc(c, (size_t)B * h * 2);
    S.xhead = dalloc(c, (size_t)B * h * 2);
    S.logits = (float*)dalloc(c, (size_t)B * c->Vl * 4);
    S.vals_all = (float*)dalloc(c, (size_t)tp * B * 4);
    S.idx_all = (int32_t*)dalloc(c, (size_t)tp * B * 4);
    S.cur_tok = (int32_t*)dalloc(c, (size_t)B * 4);
    S.tok_out = (int32_t*)dalloc(c, (size_t)B * cfg->max_new * 4);
    S.prompt = (int32_t*)dalloc(c, (size_t)Mmax * 4);
    S.page_table = (int32_t*)dalloc(c, (size_t)B * c->max_pages * 4);
    S.gemm_ws_bytes = ws;
    S.gemm_ws = dalloc(c, ws);
    S.attn_ws_bytes = attn_decode_workspace_bytes(B, c->al, c->d, Smax + cfg->max_new);
    S.attn_ws = dalloc(c, S.attn_ws_bytes);
    if (!S.x || !S.hbuf || !S.gemm_ws || !S.attn_ws || !S.page_table)
      return fail(nullptr, LIGER_ENOMEM, "liger_init: slot buffers");
    CK(cudaMemset(S.gemm_ws, 0, GEMM_COUNTER_BYTES));
    CK(cudaMemset(S.attn_ws, 0, ATTN_COUNTER_BYTES));
    CK(cudaMallocHost(&S.h_page_table, sizeof(int32_t) * B * c->max_pages));
    CK(cudaMallocHost(&S.h_prompt, sizeof(int32_t) * Mmax));
    CK(cudaMallocHost(&S.h_tok_out, sizeof(int32_t) * B * cfg->max_new));
    CK(cudaEventCreateWithFlags(&S.free_ev, cudaEventDisableTiming));
    CK(cudaEventRecord(S.free_ev, c->s_comp));
  }
  // function assembly template of one pass (§3.2) on this rank
  const bool first = c->l0 == 0, last = c->l1 == c->L;
  if (first) {
    if (c->pipe && world > 1) c->pass_ops.push_back({OP_RECV_TOK, -1});
    c->pass_ops.push_back({OP_EMBED, -1});
  } else {
    c->pass_ops.push_back({OP_RECV_X, -1});
  }
  for (int l = c->l0; l < c->l1; ++l) {
    c->pass_ops.push_back({OP_LN1, l});
    c->pass_ops.push_back({OP_QKV, l});
    c->pass_ops.push_back({OP_ATTN, l});
    c->pass_ops.push_back({OP_OUT, l});
    if (tp > 1) c->pass_ops.push_back({OP_AR1, l});
    c->pass_ops.push_back({OP_LN2, l});
    c->pass_ops.push_back({OP_FC1, l});
    c->pass_ops.push_back({OP_FC2, l});
    if (tp > 1) c->pass_ops.push_back({OP_AR2, l});
  }
  if (!last) {
    c->pass_ops.push_back({OP_SEND_X, -1});
  } else {
    c->pass_ops.push_back({OP_HEAD, -1});
    if (tp > 1) {
      c->pass_ops.push_back({OP_TOKG, -1});
      c->pass_ops.push_back({OP_PICK, -1});
    }
    if (c->pipe && world > 1) c->pass_ops.push_back({OP_SEND_TOK, -1});
  }
  if (device_sync_collective(c)) return fail(nullptr, LIGER_ECUDA, "liger_init: device synchronize failed");
  *out = cp.release();
  return LIGER_OK;
}

// Fold LN1 into QKV and LN2 into FC1 (decode passes at t = 1):
//   W x LN(x) = rstd * (W' x - mean * u) + c,   W' = W * gamma (per K column),
//   u = W' . 1 (row sums of the bf16 W'),        c = W . beta + bias
// (c and u by the library's own GEMM at M = 1 with fp32 output).
static int fold_layer_norms(liger_ctx* c, LayerW& W, cudaStream_t st) {
  const int h = c->h;
  Slot& S = c->slots[0];
  void* ones = S.yhead;   // [>= 1, h] bf16 scratch (unused outside the LM head)
  {
    std::vector<uint16_t> one((size_t)h, 0x3F80);   // bf16 1.0
    if (cudaMemcpyAsync(ones, one.data(), (size_t)h * 2, cudaMemcpyHostToDevice, st) != cudaSuccess) return LIGER_ECUDA;
    if (cudaStreamSynchronize(st) != cudaSuccess) return LIGER_ECUDA;
  }
  struct F { void *w, *wf, *g, *be, *b; float *u, *cc; int N; };
  const F fs[2] = {{W.w_qkv, W.w_qkv_f, W.g1, W.be1, W.b_qkv, W.u_qkv, W.c_qkv, 3 * c->hl},
                   {W.w_1, W.w_1_f, W.g2, W.be2, W.b_1, W.u_1, W.c_1, c->fl}};
  for (const F& f : fs) {
    GemmArgs g{};
    g.M = 1; g.K = h; g.N = f.N; g.n0 = 0; g.n1 = f.N; g.ldx = h; g.ldw = h; g.ldo = f.N; g.scale = 1.0f;
    g.out_f32 = 1; g.w_tiled = 1; g.workspace = S.gemm_ws; g.ws_bytes = S.gemm_ws_bytes;
    g.x = f.be; g.w = f.w; g.bias = f.b; g.out = f.cc;   // c = W . beta + bias
    if (int rc = gemm_launch(g, st)) return rc;
    if (int rc = fold_gamma_tiled_launch(f.w, f.wf, f.g, f.N, h, st)) return rc;
    g.x = ones; g.w = f.wf; g.bias = nullptr; g.out = f.u;   // u = W' . 1
    if (int rc = gemm_launch(g, st)) return rc;
  }
  return cudaStreamSynchronize(st) == cudaSuccess ? 0 : LIGER_ECUDA;
}

int liger_load_layer(liger_ctx* c, int l, uint64_t seed) {
  if (!c || l < 0 || l >= c->L) return LIGER_EINVAL;
  if (l < c->l0 || l >= c->l1) return LIGER_OK;   // another pipeline stage's layer
  const int r = c->tp_rank, t = c->tp;
  const int64_t h = c->h, hl = c->hl, fl = c->fl, f = c->f;
  LayerW& W = c->layers[l];
  cudaStream_t st = c->s_comp;
  const uint64_t tid = 16ull * l;
  // Projection weights are stored K-major in the tiled layout [N/128][K/64][128][64]
  // (LIGER_C0_TILED; the `ld` argument is then the first destination row).
  const int T = LIGER_C0_TILED;
  if (hl % 64 || fl % 64) return fail(c, LIGER_EINVAL, "liger_load_layer: h/t and 4h/t must be multiples of 64");
  CK(cudaMemsetAsync(W.w_qkv, 0, (size_t)pad128(3 * (int)hl) * h * 2, st));
  CK(cudaMemsetAsync(W.w_1, 0, (size_t)pad128((int)fl) * h * 2, st));
  // W_qkv logical [h, 3h]; local row j of block s in {q,k,v} = logical column s*h + r*hl + j
  for (int s = 0; s < 3; ++s) {
    CKR(c0_fill_launch(W.w_qkv, (int)hl, (int)h, s * hl, seed, tid + 0, s * h + r * hl, 0, 1, 3 * h,
                       weight_exp((int)h), T, st));
    CKR(c0_fill_launch((char*)W.b_qkv + s * hl * 2, 1, (int)hl, hl, seed, tid + 1, 0, s * h + r * hl, 0, 1, BIAS_EXP,
                       0, st));
  }
  // W_o logical [h_in, h_out]; local [h_out, hl_in]: (n, k) -> ((r*hl + k) * h + n)
  CKR(c0_fill_launch(W.w_o, (int)h, (int)hl, 0, seed, tid + 2, 0, r * hl, 1, h, weight_exp((int)h, true), T, st));
  CKR(c0_fill_launch(W.b_o, 1, (int)h, h, seed, tid + 3, 0, 0, 0, 1, BIAS_EXP, 0, st));
  // W_1 logical [h, f]; local [fl, h]: (n, k) -> (k * f + r*fl + n)
  CKR(c0_fill_launch(W.w_1, (int)fl, (int)h, 0, seed, tid + 4, r * fl, 0, 1, f, weight_exp((int)h), T, st));
  CKR(c0_fill_launch(W.b_1, 1, (int)fl, fl, seed, tid + 5, 0, r * fl, 0, 1, BIAS_EXP, 0, st));
  // W_2 logical [f, h]; local [h, fl]: (n, k) -> ((r*fl + k) * h + n)
  CKR(c0_fill_launch(W.w_2, (int)h, (int)fl, 0, seed, tid + 6, 0, r * fl, 1, h, weight_exp((int)f, true), T, st));
  CKR(c0_fill_launch(W.b_2, 1, (int)h, h, seed, tid + 7, 0, 0, 0, 1, BIAS_EXP, 0, st));
  CKR(c0_fill_launch(W.g1, 1, (int)h, h, seed, tid + 8, 0, 0, 0, 1, 0, 1, st));
  CKR(c0_fill_launch(W.be1, 1, (int)h, h, seed, tid + 9, 0, 0, 0, 1, 0, 2, st));
  CKR(c0_fill_launch(W.g2, 1, (int)h, h, seed, tid + 10, 0, 0, 0, 1, 0, 1, st));
  CKR(c0_fill_launch(W.be2, 1, (int)h, h, seed, tid + 11, 0, 0, 0, 1, 0, 2, st));
  (void)t;
  if (c->ln_fold) CKR(fold_layer_norms(c, W, st));
  CK(cudaStreamSynchronize(st));
  return LIGER_OK;
}

int liger_load_layer_weights(liger_ctx* c, int l, const liger_layer_weights* w) {
  if (!c || !w || l < 0 || l >= c->L) return LIGER_EINVAL;
  if (l < c->l0 || l >= c->l1) return LIGER_OK;   // another pipeline stage's layer
  const void* need[] = {w->w_qkv, w->b_qkv, w->w_o, w->b_o, w->w_1, w->b_1, w->w_2, w->b_2,
                        w->ln1_g, w->ln1_b, w->ln2_g, w->ln2_b};
  for (const void* q : need)
    if (!q) return fail(c, LIGER_EINVAL, "liger_load_layer_weights: null pointer");
  const int64_t h = c->h, hl = c->hl, fl = c->fl;
  LayerW& W = c->layers[l];
  cudaStream_t st = c->s_comp;
  CK(cudaMemsetAsync(W.w_qkv, 0, (size_t)pad128(3 * (int)hl) * h * 2, st));
  CK(cudaMemsetAsync(W.w_1, 0, (size_t)pad128((int)fl) * h * 2, st));
  CKR(tile_weight_launch(w->w_qkv, h, W.w_qkv, (int)(3 * hl), (int)h, st));
  CKR(tile_weight_launch(w->w_o, hl, W.w_o, (int)h, (int)hl, st));
  CKR(tile_weight_launch(w->w_1, h, W.w_1, (int)fl, (int)h, st));
  CKR(tile_weight_launch(w->w_2, fl, W.w_2, (int)h, (int)fl, st));
  CK(cudaMemcpyAsync(W.b_qkv, w->b_qkv, (size_t)3 * hl * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(W.b_o, w->b_o, (size_t)h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(W.b_1, w->b_1, (size_t)fl * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(W.b_2, w->b_2, (size_t)h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(W.g1, w->ln1_g, (size_t)h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(W.be1, w->ln1_b, (size_t)h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(W.g2, w->ln2_g, (size_t)h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(W.be2, w->ln2_b, (size_t)h * 2, cudaMemcpyDeviceToDevice, st));
  if (c->ln_fold) CKR(fold_layer_norms(c, W, st));
  CK(cudaStreamSynchronize(st));
  return LIGER_OK;
}

int liger_load_embed_weights(liger_ctx* c, const void* e_tok, const void* e_pos, const void* lnf_g,
                             const void* lnf_b) {
  if (!c || !e_tok || !e_pos || !lnf_g || !lnf_b) return LIGER_EINVAL;
  const size_t h = c->h;
  cudaStream_t st = c->s_comp;
  CK(cudaMemcpyAsync(c->e_tok, e_tok, (size_t)c->V * h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(c->e_pos, e_pos, (size_t)(c->cfg.max_pos + 2) * h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(c->lnf_g, lnf_g, h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(c->lnf_b, lnf_b, h * 2, cudaMemcpyDeviceToDevice, st));
  CK(cudaStreamSynchronize(st));
  return LIGER_OK;
}

int liger_set_streams(liger_ctx* c, void* compute_stream, void* comm_stream) {
  if (!c || !compute_stream || !comm_stream || compute_stream == comm_stream) return LIGER_EINVAL;
  if (!c->processing.empty() || !c->waiting.empty())
    return fail(c, LIGER_ESTATE, "liger_set_streams: batches in flight");
  CK(cudaStreamSynchronize(c->s_comp));
  CK(cudaStreamSynchronize(c->s_comm));
  if (c->own_streams) {
    cudaStreamDestroy(c->s_comp);
    cudaStreamDestroy(c->s_comm);
    c->own_streams = false;
  }
  c->s_comp = (cudaStream_t)compute_stream;
  c->s_comm = (cudaStream_t)comm_stream;
  c->have_round = false;
  return LIGER_OK;
}

int liger_load_embed(liger_ctx* c, uint64_t seed) {
  if (!c) return LIGER_EINVAL;
  const int64_t h = c->h;
  cudaStream_t st = c->s_comp;
  CKR(c0_fill_launch(c->e_tok, c->V, (int)h, h, seed, GID_ETOK, 0, 0, h, 1, emb_exp((int)h), 0, st));
  CKR(c0_fill_launch(c->e_pos, c->cfg.max_pos + 2, (int)h, h, seed, GID_EPOS, 0, 0, h, 1, emb_exp((int)h), 0, st));
  CKR(c0_fill_launch(c->lnf_g, 1, (int)h, h, seed, GID_LNFG, 0, 0, 0, 1, 0, 1, st));
  CKR(c0_fill_launch(c->lnf_b, 1, (int)h, h, seed, GID_LNFB, 0, 0, 0, 1, 0, 2, st));
  CK(cudaStreamSynchronize(st));
  return LIGER_OK;
}

int64_t liger_submit(liger_ctx* c, int batch, int seq_len, const int32_t* tokens, int tokens_on_device, int n_new,
                     double arrival_s) {
  if (!c || batch < 1 || batch > c->cfg.max_batch || seq_len < 1 || seq_len > c->cfg.max_seq || n_new < 1 ||
      n_new > c->cfg.max_new || !tokens || seq_len + n_new + 1 > c->cfg.max_pos + 2)
    return fail(c, LIGER_EINVAL, "liger_submit: batch/seq_len/n_new out of the configured range");
  auto bt = std::make_unique<Batch>();
  bt->id = c->next_id++;
  bt->b = batch;
  bt->s = seq_len;
  bt->n_new = n_new;
  bt->arrival_s = arrival_s;
  bt->submit_s = now_s();
  bt->eng = nullptr;
  if (tokens_on_device) {
    bt->dev_tokens = tokens;
    bt->results_to_host = false;
  } else {
    bt->host_tokens.assign(tokens, tokens + (size_t)batch * seq_len);
  }
  cudaEventCreateWithFlags(&bt->final_ev, cudaEventDisableTiming);
  const int64_t id = bt->id;
  c->all_batches.emplace_back(nullptr);
  c->waiting.push_back(std::move(bt));
  return id;
}

int liger_step(liger_ctx* c) {
  if (!c) return LIGER_EINVAL;
  const double t0 = now_s();
  // hybrid synchronization: wait for E1 of the running round (CPU-GPU sync);
  // the CPU_GPU ablation waits for the whole round, INTER_STREAM does not wait.
  if (c->have_round && c->cfg.sync_mode != LIGER_SYNC_INTER_STREAM) {
    const double w0 = now_s();
    if (c->cfg.sync_mode == LIGER_SYNC_CPU_GPU) {
      for (int i = 0; i < 2; ++i)
        while (cudaEventQuery(c->e_end[i]) == cudaErrorNotReady) {
        }
    } else {
      while (cudaEventQuery(c->e1) == cudaErrorNotReady) {
      }
    }
    c->st.wait_us += (now_s() - w0) * 1e6;
  }
  const double t_woke = now_s();
  update_list(c);
  if (c->processing.empty()) {
    c->st.host_us += (now_s() - t0) * 1e6;
    return c->waiting.empty() ? LIGER_IDLE : 0;
  }
  std::vector<Piece> pieces;
  int n = 0;
  if (c->pipe) {
    // Inter-operator pipeline: one pass of every in-flight batch, in arrival
    // order, on one stream; stages are decoupled by the send/recv of activations
    // and tokens, so consecutive batches occupy different stages concurrently.
    for (Batch* bt : c->processing) {
      if (bt->all_launched) continue;
      BatchCursor cur(c, bt, &pieces);
      const int pass = bt->pass;
      while (!cur.empty() && bt->pass == pass) cur.take(cur.head_left());
    }
    std::vector<int> all(pieces.size());
    for (size_t i = 0; i < pieces.size(); ++i) all[i] = (int)i;
    CKR(launch_run(c, pieces, all, 0));
    c->st.rounds++;
    c->have_round = false;
    n = (int)pieces.size();
  } else if (c->t1_streams && !c->timing) {
    // t = 1: one pass of every in-flight batch per step, in turn, each on the stream of
    // its slot (per-launch kernel timing runs the batches one at a time instead).  A
    // stream's launch queue is bounded: enqueueing one batch's whole list at once blocked
    // the host on that stream until the batch had nearly finished, so the other stream
    // stayed empty and the two batches' kernels never overlapped (in-kernel trace,
    // tools/timeline_capacity.py); pass by pass, both streams always hold work.
    for (Batch* bt : c->processing) {
      if (bt->all_launched) continue;
      const size_t p0 = pieces.size();
      BatchCursor cur(c, bt, &pieces);
      const int pass = bt->pass;
      while (!cur.empty() && bt->pass == pass) cur.take(cur.head_left());
      std::vector<int> mine;
      for (size_t i = p0; i < pieces.size(); ++i) mine.push_back((int)i);
      CKR(launch_run(c, pieces, mine, bt->slot & 1));
    }
    c->st.rounds++;
    c->have_round = false;
    n = (int)pieces.size();
  } else if (c->cfg.mode == LIGER_MODE_SERIAL) {
    // Intra-Op baseline: the single batch's whole remaining list, in order,
    // on one stream (computation then all-reduce, serially).
    Batch* bt = c->processing[0];
    BatchCursor cur(c, bt, &pieces);
    while (!cur.empty()) cur.take(cur.head_left());
    std::vector<int> all(pieces.size());
    for (size_t i = 0; i < pieces.size(); ++i) all[i] = (int)i;
    CKR(launch_run(c, pieces, all, 0));
    c->st.rounds++;
    c->have_round = false;
    n = (int)pieces.size();
  } else {
    std::vector<std::unique_ptr<BatchCursor>> curs;
    std::vector<Cursor*> pl;
    for (Batch* bt : c->processing) {
      curs.emplace_back(new BatchCursor(c, bt, &pieces));
      pl.push_back(curs.back().get());
    }
    RoundPlan plan;
    plan_round(pl, c->cf, &plan);
    std::vector<int> w0, w1;
    for (auto& p : plan.sub0) w0.push_back((int)p.token);
    for (auto& p : plan.sub1) w1.push_back((int)p.token);
    const int s0 = plan.type == KT_COMM ? 1 : 0;   // SubSet0 on the stream of its type
    const int s1 = 1 - s0;
    // gate both subsets on E2 of the previous round (inter-stream sync)
    if (c->have_round) {
      cudaStreamWaitEvent(c->s_comp, c->e2, 0);
      cudaStreamWaitEvent(c->s_comm, c->e2, 0);
    }
    // E1 placement.  The paper records E1 before the switch kernel (the last of SubSet0,
    // P:236) so the host plans and launches the next round while that kernel runs -- on
    // its V100s kernels took milliseconds.  B200 decode kernels take 3-30 us, the order of
    // the host's own work per round, so E1 goes before the first SubSet0 kernel from which
    // the profiled durations of the kernels still to run cover the host's measured time
    // per round (x1.5), and never after the switch kernel.  Only the time at which the
    // host wakes up moves: plans and kernels are the same (they depend on the launch state
    // alone, identical on every rank).
    size_t e1_at = w0.empty() ? 0 : w0.size() - 1;
    {
      const double lead = c->e1_lead_us >= 0 ? c->e1_lead_us : 1.5 * c->host_round_us;
      double rem = 0.0;
      for (size_t i = w0.size(); i-- > 0;) {
        const Piece& p = pieces[w0[i]];
        rem += 1e6 * op_dur(c, p.bt, p.pass, c->pass_ops[p.idx].op, p.u1 - p.u0);   // s -> us
        if (i < e1_at) e1_at = i;
        if (rem >= lead) break;
      }
    }
    // communication subset first
    auto launch_sub0 = [&]() -> int {
      if (w0.empty()) return 0;
      std::vector<int> head(w0.begin(), w0.begin() + e1_at), tail(w0.begin() + e1_at, w0.end());
      int rc = launch_run(c, pieces, head, s0);
      if (rc < 0) return rc;
      cudaEventRecord(c->e1, stream_of(c, s0));   // E1: before the kernels that cover the host's round
      rc = launch_run(c, pieces, tail, s0);
      if (rc < 0) return rc;
      cudaEventRecord(c->e2, stream_of(c, s0));   // E2: after the switch kernel
      return 0;
    };
    if (s1 == 1) {
      CKR(launch_run(c, pieces, w1, s1));
      CKR(launch_sub0());
    } else {
      CKR(launch_sub0());
      CKR(launch_run(c, pieces, w1, s1));
    }
    c->have_round = !w0.empty();
    if (c->cfg.sync_mode == LIGER_SYNC_CPU_GPU) {
      cudaEventRecord(c->e_end[0], c->s_comp);
      cudaEventRecord(c->e_end[1], c->s_comm);
    }
    c->st.rounds++;
    if (!w1.empty()) c->st.overlapped_rounds++;
    n = (int)pieces.size();
    const double us = (now_s() - t_woke) * 1e6;
    c->host_round_us = c->host_round_us > 0 ? 0.9 * c->host_round_us + 0.1 * us : us;
  }
  c->st.host_us += (now_s() - t0) * 1e6;
  (void)n;
  return LIGER_OK;   // pieces launched this round: liger_stats().kernels
}

int liger_drain(liger_ctx* c) {
  if (!c) return LIGER_EINVAL;
  for (;;) {
    int rc = liger_step(c);
    if (rc < 0) return rc;
    if (rc == LIGER_IDLE) break;
  }
  CK(cudaStreamSynchronize(c->s_comp));
  CK(cudaStreamSynchronize(c->s_comm));
  reap(c);
  return LIGER_OK;
}

int liger_poll(liger_ctx* c, int64_t id, liger_result* out, int32_t* tokens_out) {
  if (!c || id < 0 || id >= (int64_t)c->all_batches.size()) return LIGER_EINVAL;
  Batch* bt = c->all_batches[id].get();
  if (!bt) {   // still in the waiting queue
    for (auto& w : c->waiting)
      if (w->id == id) bt = w.get();
    if (!bt) return LIGER_EINVAL;
  }
  if (!bt->finished) reap(c);
  if (out) {
    out->id = bt->id;
    out->batch = bt->b;
    out->seq_len = bt->s;
    out->n_new = bt->n_new;
    out->done = bt->finished ? 1 : 0;
    out->arrival_s = bt->arrival_s;
    out->submit_s = bt->submit_s;
    out->start_s = bt->start_s;
    out->finish_s = bt->finish_s.load();
  }
  if (!bt->finished) return LIGER_PENDING;
  if (tokens_out) {
    if (!bt->results_copied) return fail(c, LIGER_ESTATE, "liger_poll: results of this batch stay on the device");
    memcpy(tokens_out, bt->tokens.data(), sizeof(int32_t) * bt->tokens.size());
  }
  return LIGER_OK;
}

int liger_result_tokens_device(liger_ctx* c, int64_t id, const int32_t** dev_tokens) {
  if (!c || id < 0 || id >= (int64_t)c->all_batches.size() || !dev_tokens) return LIGER_EINVAL;
  Batch* bt = c->all_batches[id].get();
  if (!bt || bt->slot < 0) return LIGER_PENDING;
  if (!bt->finished) reap(c);
  if (!bt->finished) return LIGER_PENDING;
  if (c->slots[bt->slot].owner != bt)
    return fail(c, LIGER_ESTATE, "liger_result_tokens_device: the batch's slot was reused by a later batch");
  *dev_tokens = c->slots[bt->slot].tok_out;
  return LIGER_OK;
}

int liger_op_allreduce(liger_ctx* c, void* buf, size_t count, int u0, int u1, int F, void* stream) {
  if (!c || !buf || F < 1 || u0 < 0 || u1 > F || u0 > u1) return LIGER_EINVAL;
  if (!c->comm || u0 == u1 || !count) return LIGER_OK;   // t = 1: the sum of one partial
  cudaStream_t st = stream ? (cudaStream_t)stream : c->s_comm;
  if (issue_ar(c, buf, count, u0, u1, F, st)) return fail(c, LIGER_ENCCL, c->comm->err);
  c->st.comm_kernels++;
  return LIGER_OK;
}

const char* liger_scheduler_name(const liger_ctx* c) {
  if (!c) return "none";
  if (c->cfg.mode == LIGER_MODE_PIPELINE) return "pipeline";
  if (c->cfg.mode == LIGER_MODE_PIPELINE_TH) return "pipeline_th";
  if (c->cfg.mode == LIGER_MODE_SERIAL) return "serial";
  if (c->t1_streams) return "t1_two_stream";
  if (c->tp == 1) return "t1_algorithm1";   // t = 1 without the two-stream schedule (LIGER_T1_STREAMS=0)
  switch (c->cfg.sync_mode) {
    case LIGER_SYNC_CPU_GPU: return "algorithm1_cpu_gpu";
    case LIGER_SYNC_INTER_STREAM: return "algorithm1_inter_stream";
  }
  return "algorithm1_hybrid";
}

int liger_set_debug_capture(liger_ctx* c, size_t arena_bytes) {
  if (!c) return LIGER_EINVAL;
  if (arena_bytes > c->dbg_arena_bytes) {
    if (!c->processing.empty()) return fail(c, LIGER_ESTATE, "liger_set_debug_capture: batches in flight");
    if (c->dbg_arena) cudaFree(c->dbg_arena);
    c->dbg_arena = nullptr;
    c->dbg_arena_bytes = c->dbg_arena_used = 0;
    if (cudaMalloc((void**)&c->dbg_arena, arena_bytes) != cudaSuccess) {
      cudaGetLastError();
      c->dbg_arena = nullptr;
    } else {
      c->dbg_arena_bytes = arena_bytes;
    }
  }
  // [collective]: nobody starts serving (and spinning on peers) before every rank has allocated
  if (c->comm) c->comm->barrier();
  if (arena_bytes && !c->dbg_arena) return fail(c, LIGER_ENOMEM, "liger_set_debug_capture: capture arena");
  c->dbg_capture = arena_bytes != 0;
  return LIGER_OK;
}

int liger_debug_read(liger_ctx* c, int64_t id, int what, void* host_buf, size_t bytes) {
  if (!c || id < 0 || id >= (int64_t)c->all_batches.size() || !host_buf) return LIGER_EINVAL;
  if (what != LIGER_DBG_LOGITS && what != LIGER_DBG_RESID) return LIGER_EINVAL;
  Batch* bt = c->all_batches[id].get();
  if (!bt) return LIGER_PENDING;
  if (!bt->finished) reap(c);
  if (!bt->finished) return LIGER_PENDING;
  if (!bt->captured) return fail(c, LIGER_ESTATE, "liger_debug_read: no capture for this batch on this rank");
  const size_t need = what == LIGER_DBG_LOGITS ? (size_t)bt->n_new * bt->b * c->Vl * 4
                                                : (size_t)bt->n_new * bt->b * c->h * 2;
  if (bytes < need) return fail(c, LIGER_EINVAL, "liger_debug_read: host buffer too small");
  CK(cudaMemcpy(host_buf, what == LIGER_DBG_LOGITS ? (const void*)bt->dbg_logits : bt->dbg_resid, need,
                cudaMemcpyDeviceToHost));
  return LIGER_OK;
}

int liger_stats(liger_ctx* c, liger_stats_t* out) {
  if (!c || !out) return LIGER_EINVAL;
  *out = c->st;
  return LIGER_OK;
}

int liger_reset_stats(liger_ctx* c) {
  if (!c) return LIGER_EINVAL;
  c->st = liger_stats_t{};
  return LIGER_OK;
}

int liger_set_gemm_sm_reserve(liger_ctx* c, int reserve) {
  if (!c || reserve < 0 || reserve >= c->n_sms) return LIGER_EINVAL;
  c->gemm_sm_reserve = reserve;
  return LIGER_OK;
}

int liger_set_kernel_timing(liger_ctx* c, int on) {
  if (!c) return LIGER_EINVAL;
  timing_flush(c);
  c->timing = on != 0;
  for (int i = 0; i < LIGER_KT_CLASSES; ++i) c->tcount[i] = 0, c->tms[i] = c->tbytes[i] = c->tflops[i] = 0;
  return LIGER_OK;
}

int liger_kernel_timing(liger_ctx* c, int64_t* count, double* ms, double* bytes, double* flops) {
  if (!c) return LIGER_EINVAL;
  timing_flush(c);
  for (int i = 0; i < LIGER_KT_CLASSES; ++i) {
    if (count) count[i] = c->tcount[i];
    if (ms) ms[i] = c->tms[i];
    if (bytes) bytes[i] = c->tbytes[i];
    if (flops) flops[i] = c->tflops[i];
  }
  return LIGER_OK;
}

int liger_set_duration(liger_ctx* c, int op, int m_tokens, int k_of_F, double us) {
  if (!c || op < 0 || op >= OP_COUNT || m_tokens <= 0 || k_of_F < 0 || k_of_F > c->F) return LIGER_EINVAL;
  DurTable& T = c->dur;
  auto it = std::lower_bound(T.mgrid.begin(), T.mgrid.end(), m_tokens);
  size_t mi = it - T.mgrid.begin();
  if (it == T.mgrid.end() || *it != m_tokens) {
    T.mgrid.insert(it, m_tokens);
    for (int o = 0; o < OP_COUNT; ++o)
      if (!T.t[o].empty()) T.t[o].insert(T.t[o].begin() + mi, std::vector<double>(c->F + 1, 0.0));
  }
  if (T.t[op].empty()) T.t[op].assign(T.mgrid.size(), std::vector<double>(c->F + 1, 0.0));
  T.t[op][mi][k_of_F] = us * 1e-6;
  T.have = true;
  return LIGER_OK;
}

// Contention-factor calibration (§3.5): profile the lengthy
// computation kernels (the projection GEMMs at the given token counts) running
// concurrently with communication kernels (all-reduces of the matching
// [M, h] partial) on the two streams, with different inputs, and take the
// maximum slowdown of either side relative to its no-load duration (reading
// R4).  At t = 1 there is no tensor-parallel all-reduce; the calibration then
// uses a 1-rank NCCL communicator whose all-reduce kernel moves the same bytes
// locally (a proxy, reported as such).  Sets the context's cf when set_cf != 0.
int liger_calibrate_cf(liger_ctx* c, const int32_t* m_list, int n_m, int set_cf, double* cf_out,
                       double* detail /* [n_m][4][2] slowdowns (gemm, ar) or NULL */) {
  if (!c || !m_list || n_m <= 0) return LIGER_EINVAL;
  if (!c->processing.empty() || !c->waiting.empty()) return fail(c, LIGER_ESTATE, "liger_calibrate_cf: batches in flight");
  CKR(device_sync_collective(c));
  Comm* comm = c->comm;
  Comm* own = nullptr;
  if (!comm) {   // t = 1: a 1-rank NCCL communicator's all-reduce kernel as the proxy
    if (!nccl().ok) return fail(c, LIGER_ENCCL, "NCCL library not loadable");
    ncclUniqueId id;
    if (nccl().GetUniqueId(&id) != ncclSuccess) return fail(c, LIGER_ENCCL, "ncclGetUniqueId failed");
    std::string err;
    own = comm_create(1, 0, reinterpret_cast<const uint8_t*>(&id), &err);
    if (!own) return fail(c, LIGER_ENCCL, "liger_calibrate_cf: " + err);
    comm = own;
  }
  CKR(device_sync_collective(c));
  Slot& S = c->slots[0];
  const int Mmax = c->cfg.max_batch * c->cfg.max_seq;
  cudaEvent_t ev[4];
  for (auto& e : ev) CK(cudaEventCreate(&e));
  const bool saved_timing = c->timing;
  c->timing = false;
  c->calibrating = true;
  Batch fake;
  fake.slot = 0;
  fake.n_new = 1;
  fake.b = 1;
  double cf = 1.0;
  auto ar = [&](size_t elems) { comm->allreduce(S.part, elems, CD_BF16, CO_SUM, c->s_comm); };
  for (int mi = 0; mi < n_m; ++mi) {
    const int M = std::min<int>(m_list[mi], Mmax);
    fake.s = M;
    int oi = 0;
    for (int op : {OP_QKV, OP_OUT, OP_FC1, OP_FC2}) {
      int pidx = 0;
      while (c->pass_ops[pidx].op != op) ++pidx;
      const size_t elems = (size_t)M * c->h;
      auto gemm = [&] { launch_piece(c, &fake, 0, pidx, 0, op_units(c, op, M), c->s_comp); };
      float tg = 1e30f, ta = 1e30f, tgc = 1e30f, tac = 1e30f;
      for (int rep = 0; rep < 4; ++rep) {
        float x;
        cudaEventRecord(ev[0], c->s_comp); gemm(); cudaEventRecord(ev[1], c->s_comp);
        cudaEventSynchronize(ev[1]); cudaEventElapsedTime(&x, ev[0], ev[1]); if (rep) tg = std::min(tg, x);
        cudaEventRecord(ev[2], c->s_comm); ar(elems); cudaEventRecord(ev[3], c->s_comm);
        cudaEventSynchronize(ev[3]); cudaEventElapsedTime(&x, ev[2], ev[3]); if (rep) ta = std::min(ta, x);
        // concurrent: both streams released together
        cudaEventRecord(ev[0], c->s_comp);
        cudaStreamWaitEvent(c->s_comm, ev[0], 0);
        cudaEventRecord(ev[2], c->s_comm);
        ar(elems);
        cudaEventRecord(ev[3], c->s_comm);
        gemm();
        cudaEventRecord(ev[1], c->s_comp);
        cudaEventSynchronize(ev[1]);
        cudaEventSynchronize(ev[3]);
        float g2, a2;
        cudaEventElapsedTime(&g2, ev[0], ev[1]);
        cudaEventElapsedTime(&a2, ev[2], ev[3]);
        if (rep) {
          tgc = std::min(tgc, g2);
          tac = std::min(tac, a2);
        }
      }
      const double sg = tgc / tg, sa = tac / ta;
      if (detail) {
        detail[(mi * 4 + oi) * 2 + 0] = sg;
        detail[(mi * 4 + oi) * 2 + 1] = sa;
      }
      cf = std::max(cf, std::max(sg, sa));
      ++oi;
    }
  }
  c->timing = saved_timing;
  c->calibrating = false;
  for (auto& e : ev) cudaEventDestroy(e);
  delete own;
  if (c->world > 1) {   // all ranks must use the same cf (identical plans)
    float* dv = nullptr;
    float v = (float)cf;
    CK(cudaMalloc(&dv, 4));
    CK(cudaMemcpy(dv, &v, 4, cudaMemcpyHostToDevice));
    if (c->comm->allreduce(dv, 1, CD_F32, CO_MAX, c->s_comp)) return fail(c, LIGER_ENCCL, c->comm->err);
    CK(cudaMemcpyAsync(&v, dv, 4, cudaMemcpyDeviceToHost, c->s_comp));
    CK(cudaStreamSynchronize(c->s_comp));
    cudaFree(dv);
    cf = v;
  }
  if (set_cf) c->cf = cf;
  if (cf_out) *cf_out = cf;
  CKR(device_sync_collective(c));
  return LIGER_OK;
}

// Offline profiling: no-load durations of every kernel
// class over a token grid and for every k/F piece, on slot 0's buffers.
int liger_profile(liger_ctx* c, const int32_t* m_list, int n_m) {
  if (!c || !m_list || n_m <= 0) return LIGER_EINVAL;
  if (!c->processing.empty() || !c->waiting.empty()) return fail(c, LIGER_ESTATE, "liger_profile: batches in flight");
  CKR(device_sync_collective(c));
  Slot& S = c->slots[0];
  cudaStream_t st = c->s_comp;
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  const int Mmax = c->cfg.max_batch * c->cfg.max_seq;
  const bool saved_timing = c->timing;
  c->timing = false;
  auto time_it = [&](auto&& fn) -> double {
    for (int i = 0; i < 2; ++i) fn();
    float best[5];
    for (int r = 0; r < 5; ++r) {
      cudaEventRecord(a, st);
      fn();
      cudaEventRecord(b, st);
      cudaEventSynchronize(b);
      cudaEventElapsedTime(&best[r], a, b);
    }
    std::sort(best, best + 5);
    return best[2] * 1e-3;
  };
  Batch fake;
  fake.slot = 0;
  fake.n_new = 1;
  for (int mi = 0; mi < n_m; ++mi) {
    const int M = std::min<int>(m_list[mi], Mmax);
    fake.b = 1;          // GEMM shapes depend on the token count M = b * s only
    fake.s = M;
    const int F = std::max(1, c->F);
    for (int op : {OP_QKV, OP_OUT, OP_FC1, OP_FC2}) {
      int pidx = 0;
      while (c->pass_ops[pidx].op != op) ++pidx;
      const int units = op_units(c, op, M);
      for (int k = 1; k <= units; ++k) {
        const int kk = units > 1 ? k : F;
        const double t = time_it([&] { launch_piece(c, &fake, 0, pidx, 0, k, st); });
        liger_set_duration(c, op, M, kk, t * 1e6);
      }
    }
    // memory-bound ops
    const double tln = time_it([&] {
      add_layernorm_launch(S.x, S.part, c->layers[c->l0].b_o, S.x, S.y, c->layers[c->l0].g2, c->layers[c->l0].be2, M,
                           c->h, 1, 0, c->cfg.ln_eps, st);
    });
    liger_set_duration(c, OP_LN1, M, F, tln * 1e6);
    liger_set_duration(c, OP_LN2, M, F, tln * 1e6);
    liger_set_duration(c, OP_EMBED, M, F, tln * 1e6);
    if (c->tp > 1) {
      const size_t E = (size_t)M * c->h;
      const int ua = op_units(c, OP_AR1, M);
      for (int k = 1; k <= ua; ++k) {
        const int kk = ua > 1 ? k : F;
        const double t = time_it([&] { issue_ar(c, S.part, E, 0, k, ua, st); });
        liger_set_duration(c, OP_AR1, M, kk, t * 1e6);
        liger_set_duration(c, OP_AR2, M, kk, t * 1e6);
      }
    }
  }
  // LM head at batch sizes (last stage only)
  if (c->l1 == c->L) {
    int pidx = 0;
    while (c->pass_ops[pidx].op != OP_HEAD) ++pidx;
    for (int bb : {1, c->cfg.max_batch}) {
      fake.b = bb;
      fake.s = 1;
      const double t = time_it([&] { launch_piece(c, &fake, 1, pidx, 0, 1, st); });
      liger_set_duration(c, OP_HEAD, bb, std::max(1, c->F), t * 1e6);
    }
  }
  // attention: calibrate the analytical model at one prefill and one decode point
  {
    int pidx = 0;
    while (c->pass_ops[pidx].op != OP_ATTN) ++pidx;
    fake.b = 1;
    fake.s = std::min(512, c->cfg.max_seq);
    fake.pages.clear();
    for (int p = 0; p < c->max_pages; ++p) S.h_page_table[p] = p;   // pages 0.. (no batch in flight)
    cudaMemcpyAsync(S.page_table, S.h_page_table, sizeof(int32_t) * c->max_pages, cudaMemcpyHostToDevice, st);
    const double tp = time_it([&] { launch_piece(c, &fake, 0, pidx, 0, 1, st); });
    c->attn_scale[0] = tp / model_dur(c, OP_ATTN, fake.s, 1, fake.s, fake.s);
    if (c->cfg.max_new > 1) {
      fake.n_new = c->cfg.max_new;
      const int pass = std::min(c->cfg.max_new - 1, 8);
      const double td = time_it([&] { launch_piece(c, &fake, pass, pidx, 0, 1, st); });
      c->attn_scale[1] = td / model_dur(c, OP_ATTN, 1, 1, fake.s + pass, 0);
    }
  }
  c->timing = saved_timing;
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  // ranks must plan identically (NCCL ordering): take the max of every entry over ranks
  if (c->world > 1) {
    std::vector<float> flat;
    for (int o = 0; o < OP_COUNT; ++o)
      for (auto& row : c->dur.t[o])
        for (double v : row) flat.push_back((float)v);
    flat.push_back((float)c->attn_scale[0]);
    flat.push_back((float)c->attn_scale[1]);
    float* dv = nullptr;
    CK(cudaMalloc(&dv, flat.size() * 4));
    CK(cudaMemcpy(dv, flat.data(), flat.size() * 4, cudaMemcpyHostToDevice));
    if (c->comm->allreduce(dv, flat.size(), CD_F32, CO_MAX, st)) return fail(c, LIGER_ENCCL, c->comm->err);
    CK(cudaMemcpyAsync(flat.data(), dv, flat.size() * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    cudaFree(dv);
    size_t i = 0;
    for (int o = 0; o < OP_COUNT; ++o)
      for (auto& row : c->dur.t[o])
        for (double& v : row) v = flat[i++];
    c->attn_scale[0] = flat[i++];
    c->attn_scale[1] = flat[i++];
  }
  CKR(device_sync_collective(c));
  return LIGER_OK;
}

const char* liger_last_error(const liger_ctx* c) { return c ? c->err.c_str() : global_error(); }

int liger_finalize(liger_ctx* c) {
  if (!c) return LIGER_EINVAL;
  // [collective]: every rank has finished enqueueing before anyone frees memory
  // or events a peer's pending work may reference
  if (c->comm) c->comm->barrier();
  cudaDeviceSynchronize();
  if (c->comm) c->comm->barrier();
  delete c->comm;
  for (void* p : c->allocs) cudaFree(p);
  for (auto& S : c->slots) {
    cudaFreeHost(S.h_page_table);
    cudaFreeHost(S.h_prompt);
    cudaFreeHost(S.h_tok_out);
    cudaEventDestroy(S.free_ev);
  }
  for (auto e : c->ev_pool) cudaEventDestroy(e);
  for (auto e : c->timing_pool) cudaEventDestroy(e);
  for (auto& b : c->all_batches)
    if (b && b->final_ev) cudaEventDestroy(b->final_ev);
  if (c->dbg_arena) cudaFree(c->dbg_arena);
  for (auto& b : c->waiting) cudaEventDestroy(b->final_ev);
  cudaEventDestroy(c->e1);
  cudaEventDestroy(c->e2);
  cudaEventDestroy(c->e_end[0]);
  cudaEventDestroy(c->e_end[1]);
  if (c->own_streams) {
    cudaStreamDestroy(c->s_comp);
    cudaStreamDestroy(c->s_comm);
  }
  gemm_forget_pointer_range(nullptr, ~size_t(0));
  delete c;
  return LIGER_OK;
}

}  // extern "C"
