/* liger.h — C ABI of the B200-native Liger hot path (libliger.so).
 *
 * Liger (Du et al., PPoPP'24; /root/reference/PAPER.md, cited as P:<line>)
 * serves pre-packed request batches on a model sharded with intra-operator
 * (Megatron tensor) parallelism and interleaves the
 * computation kernels of one batch with the communication kernels of another
 * (interleaved parallelism, §3.1), scheduled by Algorithm 1 (§3.4
 * P:178-226) with hybrid CPU-GPU / inter-stream synchronization,
 * a contention factor (§3.5) and runtime decomposition of long
 * GEMMs and all-reduces into k/F pieces (§3.6).
 *
 * Conventions
 *  - Every call returns an int status: 0 = LIGER_OK, > 0 informational,
 *    < 0 error.  No C++ exception crosses this boundary.  liger_last_error()
 *    returns a description of the last error of a context (or the global one
 *    for ctx == NULL).
 *  - Pointers documented "device" are CUDA device pointers (e.g. a torch
 *    tensor's data_ptr()); "host" are ordinary host pointers.  The library
 *    never frees memory it did not allocate (borrowed pointers).
 *  - `stream` arguments are cudaStream_t handles (NULL = legacy default stream).
 *  - All bf16 tensors are row-major and 16-byte aligned; fp32 accumulation.
 *  - Calls marked [collective] must be made by every rank of a context, in the
 *    same order and with the same arguments (NCCL ordering).
 *  - One host thread per context; nothing is re-entrant.
 *  - There is no CPU fallback: without a usable sm_100 device every compute
 *    entry point returns LIGER_ENODEV.
 */
#ifndef LIGER_H_
#define LIGER_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------ status */
#define LIGER_OK 0
#define LIGER_PENDING 1   /* liger_poll: batch not finished yet              */
#define LIGER_IDLE 2      /* liger_step: nothing to schedule                 */
#define LIGER_EINVAL (-22)
#define LIGER_ENOMEM (-12)
#define LIGER_ECUDA (-1000)
#define LIGER_ENCCL (-1001)
#define LIGER_ESTATE (-1002)
#define LIGER_ETIMEOUT (-1003)
#define LIGER_ENODEV (-1004)

/* ------------------------------------------------------------------ enums */
#define LIGER_ACT_NONE 0
#define LIGER_ACT_RELU 1      /* OPT (reading R13)                          */
#define LIGER_ACT_GELU_TANH 2 /* tiny and GLM-shaped configs                */

#define LIGER_MODE_SERIAL 0      /* Intra-Op baseline: compute then all-reduce, in order */
#define LIGER_MODE_INTERLEAVED 1 /* Liger: Algorithm 1 + hybrid sync; at t = 1
                                    (nothing to interleave) the in-flight batches run
                                    concurrently on the two streams (LIGER_T1_STREAMS=0: one) */
/* Numerics note (t = 1): decode passes of <= 16 tokens fold LayerNorm into the QKV / FC1
 * GEMMs and the residual adds into the out-proj / FC2 epilogues (LIGER_LN_FOLD=0
 * restores the add + LN kernels).  Every mode and schedule of a context computes the
 * same bits; the two settings differ by rounding only (both meet the oracle). */
/* Synchronisation of Algorithm 1 rounds (§3.4, Fig. 8; ablation §4.5):
 * HYBRID      the host waits for E1 (recorded before the running round's last
 *             primary kernel), then launches the next round's subsets -- comm
 *             first -- gated on E2 (after that kernel) by inter-stream waits;
 * CPU_GPU     the host waits until every kernel of the running round has
 *             finished, then launches (launch latency exposed);
 * INTER_STREAM no host wait: every round is launched ahead and ordered only by
 *             the E2 inter-stream waits (the paper's "lag" variant). */
#define LIGER_SYNC_HYBRID 0
#define LIGER_SYNC_CPU_GPU 1
#define LIGER_SYNC_INTER_STREAM 2
#define LIGER_MODE_PIPELINE 2    /* Inter-Op baseline: rank r holds an equal stage of unsharded
                                    layers, activations / tokens travel by send/recv;
                                    generated tokens are reported by the last stage */
#define LIGER_MODE_PIPELINE_TH 3 /* Inter-Th baseline: the Inter-Op pipeline whose every
                                    projection GEMM runs as `world` partitioned kernels (1/world
                                    of the output columns each, as intra-op partitions them);
                                    bit-identical to LIGER_MODE_PIPELINE */

/* ------------------------------------------------------------------ config */
typedef struct {
  int32_t n_layers, hidden, n_heads, ffn, vocab, max_pos; /* model shape, Table 1  */
  int32_t act;              /* LIGER_ACT_*                                                     */
  float ln_eps;             /* LayerNorm epsilon (1e-5, reading R26)                           */
  int32_t max_batch;        /* max sequences per submitted batch                               */
  int32_t max_seq;          /* max prompt length                                               */
  int32_t max_new;          /* max generated tokens per sequence                               */
  int32_t mode;             /* LIGER_MODE_*                                                    */
  int32_t max_inflight;     /* processing-list size; 1 => serial order         */
  int32_t decomp_factor;    /* F (P:254, 8 in the paper); 1 => no decomposition               */
  float contention_factor;  /* cf scaling secondary durations; <= 0 => 1.0            */
  uint64_t seed;            /* seed of the counter-based weight generator (C0)       */
  int32_t sync_mode;        /* LIGER_SYNC_* (interleaved mode; §3.4 Fig. 8, §4.5)    */
} liger_cfg;

typedef struct liger_ctx liger_ctx;

typedef struct {
  int64_t id;
  int32_t batch, seq_len, n_new;
  int32_t done;             /* 1 when finished                                                */
  double arrival_s;         /* trace arrival time (seconds, caller's clock)                   */
  double submit_s;          /* host monotonic time of liger_submit                            */
  double start_s;           /* host monotonic time the first kernel was launched              */
  double finish_s;          /* host monotonic time the final event was observed complete      */
} liger_result;

typedef struct {
  int64_t rounds;           /* Algorithm 1 iterations                                          */
  int64_t kernels;          /* kernel launches (compute + comm pieces)                         */
  int64_t comm_kernels;
  int64_t split_pieces;     /* decomposed pieces launched (k/F < 1)                            */
  int64_t overlapped_rounds;/* rounds with a non-empty secondary subset                        */
  double host_us;           /* host time spent in liger_step (plan + launch + waits)          */
  double wait_us;           /* host time spent waiting on E1 events                            */
  int64_t gpu_launches;     /* CUDA kernel launches issued by the library                     */
  double comm_host_us;      /* host time inside communication calls (NCCL enqueue; the loopback
                               backend's rendezvous) -- part of host_us                          */
} liger_stats_t;

/* ------------------------------------------------------------------ lifecycle */

/* Create a context for rank `rank` of `world` tensor-parallel ranks on the
 * current CUDA device.  nccl_uid: host pointer to the 128-byte ncclUniqueId
 * produced by liger_nccl_unique_id() on rank 0 and broadcast by the caller
 * (e.g. torch.distributed); ignored (may be NULL) when world == 1.
 * Allocates weights (uninitialised), the paged KV pool and per-slot
 * activation buffers with cudaMalloc; creates a compute and a communication
 * stream (CUDA_DEVICE_MAX_CONNECTIONS=2 is recommended).
 * [collective]  Returns LIGER_ENODEV without an sm_100 device. */
int liger_init(int world, int rank, const liger_cfg* cfg, const uint8_t* nccl_uid, liger_ctx** out);

/* Write a fresh ncclUniqueId (128 bytes) to host buffer `uid`. */
int liger_nccl_unique_id(uint8_t* uid);

/* Write a 128-byte id selecting the LOOPBACK communicator: the `world` ranks
 * are threads of one process sharing the current GPU (each calls liger_init
 * with this id and its rank from its own host thread); collectives are a host
 * rendezvous plus rank-ordered device reductions.  A test vehicle that runs
 * the complete t > 1 path (comm stream, Algorithm 1 secondaries,
 * decomposition, hybrid sync, token all-gather) on a single GPU; world <= 8. */
int liger_loopback_unique_id(uint8_t* uid);

/* Initialise this rank's shard of layer `layer` on the device with the
 * counter-based generator C0 (global indices, so every rank gets
 * its slice of the same logical weights).  seed overrides cfg->seed when != 0
 * is not desired: pass cfg->seed for the configured model. [collective] */
int liger_load_layer(liger_ctx* ctx, int layer, uint64_t seed);

/* Initialise embeddings (token + learned positions), final LN. [collective] */
int liger_load_embed(liger_ctx* ctx, uint64_t seed);

/* Load caller-owned weights instead of the seeded init (e.g. torch tensors; the library
 * copies them into its own layout -- the tiled projection weights, the folded-LN copies
 * at t = 1 -- and never keeps or frees the caller's pointers; the copies are complete
 * when the call returns).  All device pointers, bf16, row-major, THIS RANK's shard in the
 * nn.Linear layout of the Megatron partition (C8):
 *   w_qkv [3h/t, h]: rows = this rank's q heads | k heads | v heads (h/t rows each);
 *   b_qkv [3h/t] (same order); w_o [h, h/t] (columns = this rank's heads); b_o [h];
 *   w_1 [f/t, h] (rows = this rank's FFN columns); b_1 [f/t]; w_2 [h, f/t]; b_2 [h];
 *   ln1_g, ln1_b, ln2_g, ln2_b [h] (replicated).
 * In the pipeline modes t = 1 and the rank loads only its stage's layers (others: no-op).
 * LIGER_EINVAL for a null pointer or a layer out of range. [collective] */
typedef struct {
  const void *w_qkv, *b_qkv, *w_o, *b_o, *w_1, *b_1, *w_2, *b_2, *ln1_g, *ln1_b, *ln2_g, *ln2_b;
} liger_layer_weights;
int liger_load_layer_weights(liger_ctx* ctx, int layer, const liger_layer_weights* w);
/* Caller-owned embeddings: e_tok [V, h], e_pos [max_pos + 2, h] (OPT's offset 2 included),
 * lnf_g, lnf_b [h]; device bf16, replicated on every rank; copied. [collective] */
int liger_load_embed_weights(liger_ctx* ctx, const void* e_tok, const void* e_pos, const void* lnf_g,
                             const void* lnf_b);

/* Run on caller-owned CUDA streams (e.g. torch streams) instead of the two the context
 * created: compute_stream carries the computation kernels, comm_stream the collectives
 * (Algorithm 1's two streams).  Borrowed: the library never destroys them; they must
 * outlive the context and be distinct, non-null streams.  Only while no batch is in flight
 * (LIGER_ESTATE otherwise); the context's own streams are synchronised first. */
int liger_set_streams(liger_ctx* ctx, void* compute_stream, void* comm_stream);

/* Enqueue one pre-packed batch in the waiting queue.
 * tokens: [batch * seq_len] int32 prompt ids, sequence-major; host pointer
 * (copied to the device inside the library) or device pointer when
 * tokens_on_device != 0 (must stay valid until the batch finishes).
 * n_new: tokens to generate greedily (1 prefill pass + n_new - 1 decode passes,
 * reading R22).  arrival_s: the request's arrival time on the caller's clock.
 * Returns the batch id (>= 0) or an error (< 0). [collective] */
int64_t liger_submit(liger_ctx* ctx, int batch, int seq_len, const int32_t* tokens, int tokens_on_device,
                     int n_new, double arrival_s);

/* One scheduling round (one iteration of Algorithm 1): update the
 * processing list, wait for the running round's E1 event (hybrid sync,
 * P:236), plan SubSet0/SubSet1 and launch them (communication first) gated
 * on the running round's E2 event.  Returns LIGER_OK after a round (or while
 * waiting batches cannot be admitted yet), LIGER_IDLE when no batch is
 * pending, or an error; launched pieces are counted in liger_stats().
 * [collective] */
int liger_step(liger_ctx* ctx);

/* Run liger_step until every submitted batch has been launched and finished. */
int liger_drain(liger_ctx* ctx);

/* Query a batch.  Returns LIGER_PENDING while unfinished, LIGER_OK when done.
 * tokens_out: optional host buffer [batch * n_new] for the generated ids
 * (copied device -> host on the first successful poll that passes it). */
int liger_poll(liger_ctx* ctx, int64_t id, liger_result* out, int32_t* tokens_out);

/* Device pointer to a finished batch's generated tokens [batch * n_new] int32.
 * LIGER_PENDING until the batch has finished; LIGER_ESTATE once its slot has been
 * reused by a later batch (the pointer is valid only until then). */
int liger_result_tokens_device(liger_ctx* ctx, int64_t id, const int32_t** dev_tokens);

/* The per-layer all-reduce (§8(a) a6 / a10) as a standalone call on the
 * context's communicator, decomposed as the engine decomposes it (§3.6; a13):
 * in-place bf16 sum over the tensor-parallel ranks of units [u0, u1) of F, unit u
 * being the contiguous element range [count*u/F, count*(u+1)/F) of device buffer
 * `buf` (bf16 [count]).  With atomic chunks (t > 2, R9) every unit is its
 * own collective, so any split of [0, F) into pieces gives the bits of the whole.
 * Messages up to the one-shot cap use the peer-memory kernel when the backend has
 * it (rank-ordered fp32 sum, RNE to bf16).  stream: cudaStream_t or NULL (the
 * context's communication stream).  A no-op at world == 1.  [collective] */
int liger_op_allreduce(liger_ctx* ctx, void* buf, size_t count, int u0, int u1, int F, void* stream);

/* CUDA-IPC peer regions and the one-shot all-reduce kernel on them (§8(a) a6/a10 decode
 * transport; what the NCCL backend sets up with LIGER_ONESHOT_AR=1, exposed so that the
 * transport can be tested across processes with any bootstrap).  A region holds
 * [2 staging buffers of cap bytes][epoch flag][counters] (zeroed at creation);
 * liger_ipc_region_create allocates one on the current device and writes its 64-byte
 * cudaIpcMemHandle to `handle`; liger_ipc_region_open maps a peer process's region.
 * liger_op_oneshot_allreduce: in-place bf16 sum of buf[count] over `world` ranks whose
 * regions are regions[0..world) (regions[rank] = this rank's own), call number `epoch`
 * (1, 2, ... in the same order on every rank): stage, publish the epoch (system-scope
 * release), wait for every peer's flag (10 s watchdog trap), sum in rank order in fp32,
 * round to bf16.  count * 2 <= cap, 16-byte multiples.  LIGER_EINVAL / LIGER_ECUDA.
 * phases selects the kernel's halves: LIGER_AR_PHASE_STAGE (copy buf into this rank's
 * staging buffer of the epoch and publish the flag), LIGER_AR_PHASE_REDUCE (wait for all
 * flags, sum), or both (what the serving path runs, one launch per rank with the ranks on
 * different GPUs).  Ranks that share ONE GPU must not run kernels that wait on each other
 * concurrently (nothing guarantees they are co-scheduled; B200_PROFILING.md): there every
 * rank runs STAGE, the host synchronises, then every rank runs REDUCE (whose waits are
 * then already satisfied) -- the same kernel code, the same bits. */
#define LIGER_AR_PHASE_STAGE 1
#define LIGER_AR_PHASE_REDUCE 2
/* Test vehicle for the one-shot kernel's cross-rank protocol on ONE GPU: the `world` ranks of
 * call `epoch` -- rank q's buffer bufs[q] (bf16 [count], summed in place) and region
 * regions[q] (as above: liger_ipc_region_create'd or any zeroed device allocation of
 * liger's region size) -- run as ONE cooperative launch whose block group q executes rank
 * q's device code (stage, publish, spin on every flag, rank-ordered sum): the ranks' spins
 * run concurrently with every block co-resident, as ranks on different GPUs do.
 * LIGER_EINVAL if the blocks cannot all be co-resident. */
int liger_ipc_region_create(size_t cap, void** region, uint8_t* handle);
int liger_ipc_region_open(const uint8_t* handle, void** peer);
int liger_ipc_region_close(void* peer);
int liger_ipc_region_free(void* region);
int liger_op_oneshot_allreduce(void* buf, size_t count, void* const* regions, int world, int rank, size_t cap,
                               uint64_t epoch, int phases, void* stream);
int liger_op_oneshot_allreduce_emulated(void* const* bufs, size_t count, void* const* regions, int world, size_t cap,
                                        uint64_t epoch, void* stream);

/* The fused row-parallel GEMM + all-reduce of serial TP (§8(f) next row 4; DESIGN.md §8
 * "Fused row-parallel GEMM + all-reduce"), its two halves on explicit regions, call number
 * `epoch` as above (one epoch per fused all-reduce, the same sequence as the one-shot's).
 * liger_op_gemm_fused_ar_stage: the split-K GEMM P = x[M, K] . W^T (W tiled as for
 * liger_op_gemm_tiled, no bias / activation: the row-parallel partial) whose
 * split-K fixup writes bf16(P) row-major [M, N] into this rank's staging buffer of the
 * epoch and, once every fixup CTA's stores are visible, publishes the epoch flag.
 * LIGER_EINVAL unless the plan of (M, N, K) splits K (the fixup is the producer) and
 * M * N * 2 <= cap.
 * liger_op_add_layernorm_fused_ar: waits for every rank's flag, then for each row i < rows
 *   r = x[i] + sum_{q = 0..world-1} staged_q[i] (fp32, in rank order, bf16 of the sum as
 *       the one-shot all-reduce rounds it) + add_bias,
 * and x_out / y as liger_op_add_layernorm (h = N).  Same one-GPU rule as the one-shot:
 * every rank's stage call completes before any rank's add + LN call is launched. */
int liger_op_gemm_fused_ar_stage(const void* x, int64_t ldx, const void* w_tiled, int M, int N, int K,
                                 void* const* regions, int world, int rank, size_t cap, uint64_t epoch,
                                 void* workspace, size_t ws_bytes, void* stream);
int liger_op_add_layernorm_fused_ar(void* const* regions, int world, int rank, size_t cap, uint64_t epoch,
                                    const void* x, const void* add_bias, void* x_out, void* y, const void* gamma,
                                    const void* beta, int rows, int h, float eps, void* stream);

/* Debug readback for parity tests (not part of the serving path).
 * liger_set_debug_capture(ctx, arena_bytes) [collective]: arena_bytes > 0 turns capture
 * on with a device arena of that size (allocated here, before serving: nothing is
 * allocated while peers may spin in one-shot all-reduce kernels; freed by
 * liger_finalize), 0 turns it off.  For a batch admitted while capture is on, every
 * LM-head pass (pass j = 0 prefill, j >= 1 decode step j, reading R22) copies, after the
 * argmax, this rank's fp32 logits shard and the LM-head input residual into the batch's
 * part of the arena (device-to-device copies on the pass's stream; no kernel and no
 * change to any computed value); a batch that no longer fits is not captured.  liger_debug_read copies
 * a finished batch's capture to host_buf:
 *   LIGER_DBG_LOGITS  fp32 [n_new][batch][V/t]: logits of vocabulary columns
 *                     [tp_rank*V/t, (tp_rank+1)*V/t) (C7: LN_f(x_L) . E_tok^T)
 *   LIGER_DBG_RESID   bf16 [n_new][batch][h]: the last token's residual stream x_L
 *                     after the last decoder layer, before the final LayerNorm (C6)
 * Errors: LIGER_PENDING (not finished), LIGER_ESTATE (the batch ran without capture or
 * on a pipeline stage without the LM head), LIGER_EINVAL (bytes smaller than the
 * capture: n_new * batch * 4 V/t resp. n_new * batch * 2 h bytes). */
#define LIGER_DBG_LOGITS 1
#define LIGER_DBG_RESID 2
int liger_set_debug_capture(liger_ctx* ctx, size_t arena_bytes);
int liger_debug_read(liger_ctx* ctx, int64_t id, int what, void* host_buf, size_t bytes);

int liger_stats(liger_ctx* ctx, liger_stats_t* out);
int liger_reset_stats(liger_ctx* ctx);

/* Contention control (§3.5): at t > 1
 * (and inside liger_calibrate_cf) every projection GEMM's persistent grid leaves
 * `reserve` SMs free for a concurrently running all-reduce kernel.  The grid size
 * never changes a GEMM's bits.  0 <= reserve < #SMs, else LIGER_EINVAL.  Default 0
 * (or LIGER_GEMM_SM_RESERVE).  Local (not collective), but every rank should use
 * the same value, since it changes the profiled durations the plans are made from. */
int liger_set_gemm_sm_reserve(liger_ctx* ctx, int reserve);

/* Enable (1) / disable (0) CUDA-event timing of every GEMM, attention,
 * layernorm and all-reduce launch on the stream it runs on;
 * liger_kernel_timing returns, per kernel class (LIGER_KT_*), the launch
 * count, the summed device milliseconds, and the summed algorithmic bytes and
 * flops.  Host arrays of LIGER_KT_CLASSES. */
#define LIGER_KT_GEMM_DECODE 0   /* projection GEMMs with M <= 64 tokens (HBM-bound) */
#define LIGER_KT_ATTN 1
#define LIGER_KT_LN 2
#define LIGER_KT_ALLREDUCE 3
#define LIGER_KT_GEMM_PREFILL 4  /* projection GEMMs with M > 64 tokens (tensor-bound) */
#define LIGER_KT_LMHEAD 5
#define LIGER_KT_FIXUP 6         /* split-K fixup kernels */
#define LIGER_KT_CLASSES 7
int liger_set_kernel_timing(liger_ctx* ctx, int on);
int liger_kernel_timing(liger_ctx* ctx, int64_t* count, double* ms, double* bytes, double* flops);

/* Timeline trace (diagnostics, not part of the serving path).  liger_trace_start
 * installs a device buffer of `capacity` records; from then on thread 0 of every
 * CTA of the GEMM, split-K fixup, add+LN and attention kernels appends one
 * LIGER_TRACE_REC_BYTES-byte record {uint32 kernel id, CTA index, SM id, pad;
 * uint64 %globaltimer ns at entry, after the PDL wait, at exit}.  Kernel ids:
 * 1 GEMM, 2 fixup, 3 decode attention (0x103 = its merging CTA), 5 add+LN.
 * liger_trace_stop synchronises the device, copies min(n, capacity) records to
 * host_records (caller-owned), stores the number recorded in *n_out and frees the
 * buffer.  Records beyond the capacity are dropped.  Process-global; not
 * thread-safe.  Errors: LIGER_EINVAL (capacity 0), LIGER_ESTATE (not started),
 * LIGER_ECUDA. */
#define LIGER_TRACE_REC_BYTES 40
int liger_trace_start(unsigned int capacity);
int liger_trace_stop(void* host_records, unsigned int capacity, unsigned int* n_out);

/* Set the per-kernel duration table used by Algorithm 1:
 * durations in microseconds for a kernel class at a token count, piecewise
 * linear in M between profiled points.  Called by the offline profiler
 * (bench.py / liger_profile) or loaded from JSON by the binding. */
int liger_set_duration(liger_ctx* ctx, int kclass, int m_tokens, int k_of_F, double us);

/* Offline profiling: measure no-load durations of every
 * kernel class at token counts m_list[0..n_m) for every piece size k/F and
 * store them in the duration table.  Returns LIGER_OK. */
int liger_profile(liger_ctx* ctx, const int32_t* m_list, int n_m);

/* Contention-factor calibration (§8(a) a16): run each projection
 * GEMM at token counts m_list concurrently with an all-reduce of the matching
 * [M, h] partial on the communication stream, and return in *cf_out the
 * maximum slowdown of either kernel versus its no-load duration (ranks agree
 * by max).  detail (optional, host [n_m][4][2]): slowdowns (GEMM, all-reduce)
 * per token count and GEMM (QKV, out, FC1, FC2).  At world == 1 a 1-rank NCCL
 * all-reduce (a local copy kernel of the same bytes) is the proxy.
 * set_cf != 0 installs the result as the scheduler's cf. [collective] */
int liger_calibrate_cf(liger_ctx* ctx, const int32_t* m_list, int n_m, int set_cf, double* cf_out,
                       double* detail);

/* The schedule this context actually runs (a static string): "serial" (Intra-Op),
 * "algorithm1_hybrid" / "algorithm1_cpu_gpu" / "algorithm1_inter_stream" (Liger at
 * t > 1, by sync mode), "t1_two_stream" (interleaved mode at t = 1, reading R31:
 * there is no communication to interleave, the in-flight batches' kernel lists run
 * concurrently on the two streams), "t1_algorithm1" (t = 1 with LIGER_T1_STREAMS=0),
 * "pipeline", "pipeline_th". */
const char* liger_scheduler_name(const liger_ctx* ctx);

const char* liger_last_error(const liger_ctx* ctx);
int liger_finalize(liger_ctx* ctx); /* [collective] */

/* ------------------------------------------------------------------ kernel entry points
 * The single kernels of the hot path, exposed for parity tests and roofline
 * measurement.  All pointers are device pointers unless stated.  They launch
 * asynchronously on `stream` and return LIGER_EINVAL on bad shapes. */

/* GEMM with fused epilogue (§8(a) a3/a5/a8/a9, decomposition a13):
 *   out[m, n] = act( (sum_k x[m,k] * w[n,k]) + bias[n] ) * (n < scale_cols ? scale : 1)
 * for m < M and n in the slice [n0, n1) of the N output columns (PAPER.md
 * §3.6 "vertical" split, Fig. 9).  x bf16 [M, K] row stride ldx; w bf16
 * [N, K] row stride ldw; bias bf16 [N] or NULL; out bf16 (or fp32 if out_f32)
 * with row stride ldo (columns n0..n1 written at their global index n).
 * Scaling is applied after the bias and before the activation.
 * workspace: device scratch of liger_gemm_workspace_bytes(M, N, K) bytes whose
 * first 16 KiB must be zero before the first use (the kernel leaves them zero).
 * The result for any column is bit-identical for every slice containing it. */
int liger_op_gemm(const void* x, int64_t ldx, const void* w, int64_t ldw, void* out, int64_t ldo, int M, int N,
                  int K, int n0, int n1, const void* bias, int act, int scale_cols, float scale, int out_f32,
                  void* workspace, size_t ws_bytes, void* stream);
/* Same, with W in the tiled layout liger_load_layer uses for the projection
 * weights: [ceil(N/128)][K/64][128][64] bf16 (every 16 KiB TMA box contiguous in
 * HBM); requires K % 64 == 0 and n0 % 128 == 0. */
int liger_op_gemm_tiled(const void* x, int64_t ldx, const void* w_tiled, void* out, int64_t ldo, int M, int N,
                        int K, int n0, int n1, const void* bias, int act, int scale_cols, float scale, int out_f32,
                        void* workspace, size_t ws_bytes, void* stream);
/* Convert a row-major bf16 W [N, K] (row stride ld) to the tiled layout
 * (dst holds ceil(N/128)*128*K elements; padding rows are zero). */
int liger_op_tile_weight(const void* w, int64_t ld, void* w_tiled, int N, int K, void* stream);
size_t liger_gemm_workspace_bytes(int M, int N, int K);
/* The tiling plan liger_op_gemm uses for a GEMM of full size (M, N, K) (host
 * only; a function of (M, N, K), identical for every column slice):
 * out[5] = {token tile bn, m tiles, split-K chunk kc, splits, pipeline stages};
 * splits > 1: a split-K fixup kernel sums the chunks' fp32 partials in chunk order. */
int liger_gemm_plan(int M, int N, int K, int32_t* out);

/* Fused residual add + LayerNorm (§8(a) a2/a7/a11; C2):
 *   r    = x[in_row(i)] + (add ? add[in_row(i)] : 0) + (add_bias ? add_bias : 0)     (fp32)
 *   x_out[i] = bf16(r)           (if x_out != NULL; may alias x when in_row(i) == i)
 *   y[i] = bf16( (r' - mean(r')) / sqrt(var(r') + eps) * gamma + beta ),  r' = bf16(r)
 * for i < rows, in_row(i) = i * in_row_step + in_row_off (gather of the last
 * token of each sequence for the LM head).  All [*, h] bf16. */
int liger_op_add_layernorm(const void* x, const void* add, const void* add_bias, void* x_out, void* y,
                           const void* gamma, const void* beta, int rows, int h, int in_row_step,
                           int in_row_off, float eps, void* stream);

/* Embedding (§8(a) a1; C1): out[i] = E_tok[ids[i]] + E_pos[pos(i) + 2] with
 * pos(i) = start_pos + (seq_len > 0 ? i % seq_len : 0); bf16 [rows, h]. */
int liger_op_embed(const int32_t* ids, const void* e_tok, const void* e_pos, void* out, int rows, int h,
                   int seq_len, int start_pos, void* stream);

/* Paged KV cache geometry: page = kv_block (16) tokens; pool layout
 * [n_pages][2 (K,V)][heads][16][d] bf16.  page_table: int32 [b][max_pages]. */
#define LIGER_KV_BLOCK 16

/* Prefill causal attention (§8(a) a4; C4) over qkv [b*s, 3*heads*d] bf16
 * (row = token, columns [q heads | k heads | v heads], q pre-scaled),
 * writing o [b*s, heads*d] bf16 and the K/V of all s positions into the pages. */
int liger_op_attn_prefill(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages,
                          int b, int s, int heads, int d, void* stream);

/* Decode attention (§8(a) a4) for one new token per sequence at position
 * `pos` (cache holds positions [0, pos)): qkv [b, 3*heads*d]; appends the
 * token's K/V to the cache page; o [b, heads*d].  workspace: device scratch
 * of liger_attn_decode_workspace_bytes(b, heads, d, pos + 1) bytes (enough for
 * every launch with at most b sequences and context at most pos + 1), first
 * 16 KiB zero before first use (left zero).  LIGER_EINVAL if pos >= max_pages * 16
 * (the page table row cannot hold the new token) or d not in {64, 128}. */
int liger_op_attn_decode(const void* qkv, void* o, void* kv_pool, const int32_t* page_table, int max_pages, int b,
                         int pos, int heads, int d, void* workspace, size_t ws_bytes, void* stream);
size_t liger_attn_decode_workspace_bytes(int b, int heads, int d, int ctx);

/* Row-wise argmax over fp32 logits [rows, n] (row stride ld): writes the
 * maximum value and its index + idx_offset (lowest index on ties, C7). */
int liger_op_argmax(const float* logits, int64_t ld, int rows, int n, int idx_offset, float* max_out,
                    int32_t* idx_out, void* stream);

/* Fill a bf16 [rows, cols] (row stride ld) device tensor with C0 values of
 * logical tensor `tensor_id`: element (r, c) takes global index
 * (r + row_off) * idx_row_stride + (c + col_off) * idx_col_stride, scale 2^exp;
 * kind 0 = plain, 1 = gamma (1 + v/16), 2 = beta (v/16); kind | LIGER_C0_TILED writes
 * element (r, c) as row ld + r, column c of a tiled-layout matrix with K = cols
 * (see liger_op_gemm_tiled; ld then means "first destination row"). */
#define LIGER_C0_TILED 16
int liger_op_c0_fill(void* dst, int rows, int cols, int64_t ld, uint64_t seed, uint64_t tensor_id,
                     int64_t row_off, int64_t col_off, int64_t idx_row_stride, int64_t idx_col_stride, int exp,
                     int kind, void* stream);

/* ------------------------------------------------------------------ host-only scheduler (no GPU needed)
 * Algorithm 1 planner (§3.4, readings R1-R5 of DESIGN.md)
 * exposed for CPU tests of the host logic; the engine runs the same plan_round.
 * liger_planner_submit: one batch of n_kernels kernels, types[i] 0 = compute,
 * 1 = communication, units[i] = pieces (1 = not decomposable, else F), durs =
 * concatenation over kernels of units[i] durations (duration of a k-unit piece,
 * k = 1..units[i]).  liger_plan_round: update_list() + one round; writes
 * *n_out entries {batch, kernel index, unit begin, unit end, subset (0/1)}
 * (LIGER_EINVAL if more than cap), the round's type and SubSet0 time; returns
 * LIGER_OK, or LIGER_IDLE when nothing is left. */
typedef struct liger_planner liger_planner;
int liger_planner_create(int list_size, double cf, liger_planner** out);
int liger_planner_submit(liger_planner* p, int64_t batch, int n_kernels, const int32_t* types,
                         const int32_t* units, const double* durs /* per kernel: units entries */);
int liger_plan_round(liger_planner* p, int32_t* entries /* [cap][5] */, int cap, int32_t* n_out,
                     int32_t* round_type, double* time0);
int liger_planner_destroy(liger_planner* p);

#ifdef __cplusplus
}
#endif
#endif /* LIGER_H_ */
