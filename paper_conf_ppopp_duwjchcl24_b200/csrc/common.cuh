// Shared device helpers for the sm_100a kernels (PTX wrappers, bf16 packing).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include <stdlib.h>

#include <mutex>
#include <unordered_set>
#include <utility>

#define LIGER_DEV __device__ __forceinline__

namespace liger {

LIGER_DEV uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---------------------------------------------------------------- mbarrier
LIGER_DEV void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
LIGER_DEV void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
LIGER_DEV void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
LIGER_DEV void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
LIGER_DEV void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t a = smem_u32(bar);
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "LIGER_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra LIGER_DONE_%=;\n\t"
      "bra LIGER_WAIT_%=;\n"
      "LIGER_DONE_%=:\n\t}" ::"r"(a),
      "r"(parity)
      : "memory");
}

// ---------------------------------------------------------------- clusters / DSMEM
LIGER_DEV uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// All threads of every CTA of the cluster (aligned: whole warps).
LIGER_DEV void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cta address -> the same offset in CTA `rank` of the cluster (shared::cluster window)
LIGER_DEV uint32_t dsmem_map(uint32_t local_addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(local_addr), "r"(rank));
  return r;
}
// Release-arrive (cluster scope) on an mbarrier of CTA `rank` (cumulative over
// writes that happen-before it, e.g. other lanes' smem stores ordered by __syncwarp).
LIGER_DEV void mbar_arrive_remote(uint64_t* local_bar, uint32_t rank) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(
                   dsmem_map(smem_u32(local_bar), rank))
               : "memory");
}
LIGER_DEV void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  uint32_t a = smem_u32(bar);
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "LIGER_CWAIT_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra LIGER_CDONE_%=;\n\t"
      "bra LIGER_CWAIT_%=;\n"
      "LIGER_CDONE_%=:\n\t}" ::"r"(a),
      "r"(parity)
      : "memory");
}
LIGER_DEV float4 ld_dsmem_f4(uint32_t cluster_addr) {
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"(cluster_addr)
               : "memory");
  return v;
}

// ---------------------------------------------------------------- TMA
LIGER_DEV void tma_prefetch_desc(const void* desc) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(desc) : "memory");
}
// 2-D tiled load: coordinates (c0 = innermost element index, c1 = row).
LIGER_DEV void tma_load_2d(void* smem_dst, const void* desc, uint64_t* bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(smem_dst)),
      "l"(desc), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}
LIGER_DEV void tma_load_2d_hint(void* smem_dst, const void* desc, uint64_t* bar, int c0, int c1,
                                uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%2, %3}], [%4], %5;" ::"r"(smem_u32(smem_dst)),
      "l"(desc), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
// 1-D bulk copy global -> shared completing on an mbarrier (TMA bulk engine).
LIGER_DEV void bulk_load(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(smem_dst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// Fire-and-forget L2 prefetch of [gsrc, gsrc + bytes) (TMA bulk engine; 16-B aligned, bytes % 16 == 0).
LIGER_DEV void bulk_prefetch_l2(const void* gsrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(gsrc), "r"(bytes) : "memory");
}
LIGER_DEV uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
LIGER_DEV uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// ---------------------------------------------------------------- tcgen05
LIGER_DEV void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
LIGER_DEV void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// Must be executed by one full warp.
LIGER_DEV void tmem_alloc(uint32_t* smem_slot, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(smem_slot)),
               "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
LIGER_DEV void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}

// D[tmem] (+)= A[smem] * B[smem]^T, kind::f16 (bf16 in, fp32 accumulate).
LIGER_DEV void umma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// Arrive on an mbarrier when all previously issued tcgen05.mma of this thread complete.
LIGER_DEV void umma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}

// 32 lanes x 32 bit, 16 consecutive columns per thread.
LIGER_DEV void tmem_ld_32x32b_x16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr)
      : "memory");
}
LIGER_DEV void tmem_ld_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// UMMA shared-memory descriptor for a K-major tile written by TMA with
// SWIZZLE_128B: rows of 128 B (64 bf16), 8-row atoms of 1024 B (SBO), version 1.
LIGER_DEV uint64_t umma_desc_sw128(uint32_t smem_addr) {
  uint64_t d = 0;
  d |= (uint64_t)((smem_addr >> 4) & 0x3FFF);
  d |= (uint64_t)(1024 >> 4) << 32;   // stride byte offset
  d |= (uint64_t)1 << 46;             // descriptor version (sm_100)
  d |= (uint64_t)2 << 61;             // SWIZZLE_128B
  return d;
}

LIGER_DEV void named_bar_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Programmatic dependent launch: wait for the preceding grid in the stream
// (no-op when launched without the PDL attribute).
LIGER_DEV void grid_dependency_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// Allow the next PDL kernel in the stream to be scheduled (its CTAs wait in
// grid_dependency_wait until this grid has completed).
LIGER_DEV void grid_dependency_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
// For kernels whose whole body depends on upstream data.  The trigger comes
// AFTER the wait: the next kernel's pre-wait code (weight / KV-cache prefetch)
// then overlaps only this kernel, never an older one still running.
LIGER_DEV void pdl_enter() {
  grid_dependency_wait();
  grid_dependency_trigger();
}

// ---------------------------------------------------------------- timeline trace
// Development diagnostics (liger_trace_start / liger_trace_stop): thread 0 of every
// CTA of a traced kernel writes {kernel id, CTA, SM, entry, after-PDL-wait, exit}
// %globaltimer stamps.  Off (one predicated load) unless a buffer is installed.
// Each translation unit holds its own copy of the buffer descriptor.
struct TraceRec {
  uint32_t kid, cta, smid, pad;
  uint64_t t0, t1, t2;
};
struct TraceBuf {
  TraceRec* rec;
  unsigned int* n;
  unsigned int cap;
};
static __device__ TraceBuf g_trace = {nullptr, nullptr, 0};
LIGER_DEV uint64_t trace_now() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Entry stamp; thread 0 of a traced CTA also reserves its record slot here, so the atomic's
// round trip overlaps the kernel's work instead of delaying the CTA's exit.
struct TraceStart {
  uint64_t t0;
  unsigned int slot;
};
LIGER_DEV TraceStart trace_begin() {
  TraceStart r{trace_now(), 0xFFFFFFFFu};
  if (threadIdx.x == 0 && g_trace.rec != nullptr) r.slot = atomicAdd(g_trace.n, 1u);
  return r;
}
LIGER_DEV void trace_write(uint32_t kid, TraceStart s0, uint64_t t1) {
  if (g_trace.rec == nullptr || s0.slot >= g_trace.cap) return;
  const uint64_t t0 = s0.t0;
  const uint64_t t2 = trace_now();
  const unsigned int i = s0.slot;
  uint32_t sm;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
  TraceRec r;
  r.kid = kid;
  r.cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  r.smid = sm;
  r.pad = 0;
  r.t0 = t0;
  r.t1 = t1;
  r.t2 = t2;
  g_trace.rec[i] = r;
}
#define LIGER_TRACE_SETTER(name) \
  void trace_set_##name(TraceRec* rec, unsigned int* n, unsigned int cap) { \
    TraceBuf b{rec, n, cap};                                                \
    cudaMemcpyToSymbol(g_trace, &b, sizeof(b));                             \
  }
enum TraceKid : uint32_t { TK_GEMM = 1, TK_FIXUP, TK_ATTN_DEC, TK_ATTN_PRE, TK_ADDLN, TK_EMBED, TK_ARGMAX, TK_PICK, TK_FUSED };

LIGER_DEV float bf16_bits_to_f32(uint16_t b) { return __uint_as_float(((uint32_t)b) << 16); }

LIGER_DEV float gelu_tanh_f(float x) {
  const float k0 = 0.7978845608028654f, k1 = 0.044715f;
  return 0.5f * x * (1.0f + tanhf(k0 * (x + k1 * x * x * x)));
}

// Every kernel of the library prefers the maximal shared-memory carveout.  An SM's
// L1/shared split can only change while it is idle, so a kernel that stays resident
// (the all-reduce kernels spinning on peers' flags) would otherwise pin a small-smem
// configuration and keep a persistent GEMM CTA (up to 217 KB) off that SM -- with
// static unit assignment that GEMM then never completes (a TP = 4 loopback hang).
inline void prefer_max_smem(const void* fn);
// Load a kernel now (CUDA lazy module loading would otherwise load it at its first launch,
// which can wait for running kernels -- a deadlock when those spin on peers whose host
// thread is the one loading; see preload_kernels in kernels.h).
template <typename K>
inline void preload_kernel(K k) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, reinterpret_cast<const void*>(k));
  prefer_max_smem(reinterpret_cast<const void*>(k));
}
inline void prefer_max_smem(const void* fn) {
  static std::mutex mu;
  static std::unordered_set<const void*> done;
  static const bool off = getenv("LIGER_NO_CARVEOUT") != nullptr;   // experiments only
  if (off) return;
  std::lock_guard<std::mutex> g(mu);
  if (done.insert(fn).second) cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
}

// Launch with programmatic stream serialization so the kernel's prologue overlaps
// the tail of the previous kernel on the stream (the kernel calls
// grid_dependency_wait() before touching data produced or consumed upstream).
// SMs of the current device (host).
inline int sm_count() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

template <typename... KArgs, typename... Args>
inline int launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t stream,
                      Args&&... args) {
  prefer_max_smem(reinterpret_cast<const void*>(kernel));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  static const int pdl_on = getenv("LIGER_NO_PDL") ? 0 : 1;   // experiments: LIGER_NO_PDL=1
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_on;
  cudaError_t e = cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
  return e == cudaSuccess ? 0 : -1000;
}

template <typename... KArgs, typename... Args>
inline int launch_pdl_cluster(void (*kernel)(KArgs...), dim3 grid, dim3 block, int cluster_x, size_t smem,
                              cudaStream_t stream, Args&&... args) {
  prefer_max_smem(reinterpret_cast<const void*>(kernel));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  static const int pdl_on = getenv("LIGER_NO_PDL") ? 0 : 1;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = cluster_x;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1 + pdl_on;
  cudaError_t e = cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
  return e == cudaSuccess ? 0 : -1000;
}

}  // namespace liger
