// One-shot all-reduce over peer memory (§8(f) next row 4):
// the per-layer all-reduce of the row-parallel partials for decode-size messages,
// where a ring/tree collective is latency-bound (2(t-1) dependent steps).
//
// Every rank owns a peer-visible staging region [2 buffers][cap bytes] + one epoch
// flag.  Call e (all ranks issue all-reduces in the same order) runs ONE kernel:
//   A  copy the local bf16 input into staging buffer e % 2;
//   -  the last block to finish A (device counter) publishes flag = e with a
//      system-scope release;
//   B  every block waits until all t flags reach e (acquire, system scope), then
//      sums element i over ranks q = 0..t-1 IN ORDER in fp32 (peer loads over
//      NVLink: ld.global.cv) and writes bf16(sum) in place.
// The sum order is the same on every rank and for every element, so all ranks get
// identical bits, and an all-reduce split into contiguous pieces (Liger's runtime
// decomposition) is bit-identical to the whole one.  Buffer e % 2 is
// rewritten at call e + 2 only after this rank passed call e + 1's flag wait, i.e.
// after every peer finished call e (stream order), so two buffers suffice.
//
// Transport: NVLink peers map each other's staging with CUDA IPC handles
// (exchanged by the NCCL communicator), one rank per GPU.  The loopback test
// backend (t ranks sharing one GPU) never uses it: kernels that wait on each other
// are not guaranteed to be co-scheduled on one GPU.  There the kernel is tested
// phase by phase (`phases`): every rank's STAGE launch, a host sync, then every
// rank's REDUCE launch, whose flag waits are already satisfied.
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <string.h>
#include <stdio.h>
#include <stdlib.h>

#include "comm.h"
#include "common.cuh"
#include "kernels.h"

namespace liger {

namespace {

constexpr int PAR_MAX_WORLD = 8;
constexpr int PAR_THREADS = 256;

struct PeerPtrs {
  const uint4* data[PAR_MAX_WORLD];                  // staging buffer e % 2 of rank q
  const unsigned long long* flag[PAR_MAX_WORLD];     // epoch flag of rank q
};

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// One rank's one-shot all-reduce, run by `nblk` blocks (block index `bid` of them).
// n8 = number of 8-element (16-byte) vectors
__device__ __forceinline__ void oneshot_rank(uint4* buf, size_t n8, uint4* my_stage, unsigned long long* my_flag,
                                             unsigned int* counter, const PeerPtrs& peers, int world,
                                             unsigned long long epoch, int phases, int bid, int nblk) {
  const size_t stride = (size_t)nblk * blockDim.x;
  // The partials come from the preceding GEMM.  Dependents are released only after
  // every peer has arrived (below): a kernel parked at its griddepcontrol.wait
  // must not hold SM resources while this one spins on other ranks -- on the
  // loopback backend those ranks share this GPU and would need them to progress.
  grid_dependency_wait();
  if (phases & LIGER_AR_PHASE_STAGE) {
    for (size_t i = (size_t)bid * blockDim.x + threadIdx.x; i < n8; i += stride) my_stage[i] = buf[i];
    __threadfence_system();   // every thread's staging stores before the block's publish
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence_system();
      const unsigned int prev = atomicAdd(counter, 1u);
      if (prev == (unsigned int)nblk - 1) {   // every block's staging copy is done: publish
        *counter = 0;
        __threadfence_system();
        st_release_sys(my_flag, epoch);
      }
    }
  }
  if (!(phases & LIGER_AR_PHASE_REDUCE)) {
    grid_dependency_trigger();
    return;
  }
  if (threadIdx.x == 0) {
    const uint64_t t0 = trace_now();
    for (int q = 0; q < world; ++q)
      while (ld_acquire_sys(peers.flag[q]) < epoch) {
        __nanosleep(64);
        if (trace_now() - t0 > 10000000000ull) {   // a peer never arrived: fail, do not hang
          printf("liger one-shot all-reduce: epoch %llu, waited 10 s for peer %d (flag %llu), block %d of %d\n",
                 epoch, q, ld_acquire_sys(peers.flag[q]), bid, nblk);
          __trap();
        }
      }
  }
  __syncthreads();
  grid_dependency_trigger();
  for (size_t i = (size_t)bid * blockDim.x + threadIdx.x; i < n8; i += stride) {
    uint4 v[PAR_MAX_WORLD];
#pragma unroll
    for (int q = 0; q < PAR_MAX_WORLD; ++q)
      if (q < world) v[q] = __ldcv(peers.data[q] + i);
    float acc[8];
    {
      const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&v[0]);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 f = __bfloat1622float2(h[e]);
        acc[2 * e] = f.x;
        acc[2 * e + 1] = f.y;
      }
    }
#pragma unroll
    for (int q = 1; q < PAR_MAX_WORLD; ++q) {
      if (q < world) {
        const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&v[q]);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float2 f = __bfloat1622float2(h[e]);
          acc[2 * e] += f.x;
          acc[2 * e + 1] += f.y;
        }
      }
    }
    uint4 o;
    __nv_bfloat162* oh = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
    for (int e = 0; e < 4; ++e) oh[e] = __floats2bfloat162_rn(acc[2 * e], acc[2 * e + 1]);
    buf[i] = o;
  }
}


__global__ void __launch_bounds__(PAR_THREADS) oneshot_ar_bf16_kernel(uint4* buf, size_t n8, uint4* my_stage,
                                                                      unsigned long long* my_flag,
                                                                      unsigned int* counter, PeerPtrs peers,
                                                                      int world, unsigned long long epoch,
                                                                      int phases) {
  oneshot_rank(buf, n8, my_stage, my_flag, counter, peers, world, epoch, phases, blockIdx.x, gridDim.x);
}

// Test vehicle: the `world` ranks of one all-reduce as ONE cooperative launch on one GPU
// (block group q = blocks [q nblk, (q + 1) nblk) runs rank q's oneshot_rank), so the ranks'
// spins on each other's flags run concurrently with every block co-resident -- the way
// ranks on different GPUs run, which separate launches on one GPU cannot guarantee.
struct EmuRanks {
  uint4* buf[PAR_MAX_WORLD];
  uint4* stage[PAR_MAX_WORLD];
  unsigned long long* flag[PAR_MAX_WORLD];
  unsigned int* counter[PAR_MAX_WORLD];
};
__global__ void __launch_bounds__(PAR_THREADS) oneshot_ar_emulated_kernel(EmuRanks r, size_t n8, PeerPtrs peers,
                                                                          int world, unsigned long long epoch,
                                                                          int nblk) {
  const int q = blockIdx.x / nblk;
  oneshot_rank(r.buf[q], n8, r.stage[q], r.flag[q], r.counter[q], peers, world, epoch,
               LIGER_AR_PHASE_STAGE | LIGER_AR_PHASE_REDUCE, blockIdx.x % nblk, nblk);
}
}  // namespace

// [2 buffers][cap] | epoch flag (+0) | one-shot block counter (+128) | fused-producer
// counter (+256): the counters live in the zeroed region so that nothing is
// allocated after the ranks' setup rendezvous -- on the loopback backend a
// cudaMalloc / cudaMemset there can wait for a peer's kernel that is spinning on
// this rank's flag (seen as a TP = 4 hang).
size_t peer_ar_region_bytes(size_t cap) { return 2 * cap + 512; }

int PeerAR::init(int world_, int rank_, size_t cap_, void* local_region, void* const* peer_regions) {
  if (world_ < 1 || world_ > PAR_MAX_WORLD || cap_ % 256) return LIGER_EINVAL;
  world = world_;
  rank = rank_;
  cap = cap_;
  local = local_region;
  for (int q = 0; q < world; ++q) peer[q] = peer_regions[q];
  counter = reinterpret_cast<unsigned int*>(static_cast<char*>(local) + 2 * cap + 128);
  fused_counter = reinterpret_cast<unsigned int*>(static_cast<char*>(local) + 2 * cap + 256);
  return 0;
}

PeerAR::~PeerAR() {}

static bool dbg_epochs() {
  static const bool on = getenv("LIGER_DBG_EPOCH") != nullptr;
  return on;
}

int PeerAR::fused_begin(size_t bytes, FusedARDesc* out) {
  if (bytes > cap || bytes % 16) return LIGER_EINVAL;
  ++epoch;
  if (dbg_epochs()) fprintf(stderr, "[rank %d] epoch %llu fused %zu B\n", rank, (unsigned long long)epoch, bytes);
  const int b = (int)(epoch & 1);
  FusedARDesc d{};
  d.stage = static_cast<char*>(local) + (size_t)b * cap;
  d.flag = reinterpret_cast<unsigned long long*>(static_cast<char*>(local) + 2 * cap);
  d.counter = fused_counter;
  for (int q = 0; q < world; ++q) {
    d.peer_stage[q] = static_cast<const char*>(peer[q]) + (size_t)b * cap;
    d.peer_flag[q] = reinterpret_cast<const unsigned long long*>(static_cast<const char*>(peer[q]) + 2 * cap);
  }
  d.world = world;
  d.epoch = epoch;
  *out = d;
  return 0;
}

int PeerAR::allreduce_bf16(void* buf, size_t count, cudaStream_t st, int phases) {
  const size_t bytes = count * 2;
  if (bytes > cap || bytes % 16 || reinterpret_cast<uintptr_t>(buf) % 16 || phases < 1 || phases > 3)
    return LIGER_EINVAL;
  if (!count) return 0;
  ++epoch;
  if (dbg_epochs()) fprintf(stderr, "[rank %d] epoch %llu one-shot %zu B\n", rank, (unsigned long long)epoch, bytes);
  const int b = (int)(epoch & 1);
  PeerPtrs pp{};
  for (int q = 0; q < world; ++q) {
    pp.data[q] = reinterpret_cast<const uint4*>(static_cast<const char*>(peer[q]) + (size_t)b * cap);
    pp.flag[q] = reinterpret_cast<const unsigned long long*>(static_cast<const char*>(peer[q]) + 2 * cap);
  }
  const size_t n8 = bytes / 16;
  int blocks = (int)((n8 + PAR_THREADS - 1) / PAR_THREADS);
  if (blocks > 64) blocks = 64;
  if (blocks < 1) blocks = 1;
  uint4* stage = reinterpret_cast<uint4*>(static_cast<char*>(local) + (size_t)b * cap);
  unsigned long long* flag = reinterpret_cast<unsigned long long*>(static_cast<char*>(local) + 2 * cap);
  return launch_pdl(oneshot_ar_bf16_kernel, dim3(blocks), dim3(PAR_THREADS), 0, st, reinterpret_cast<uint4*>(buf),
                    n8, stage, flag, counter, pp, world, (unsigned long long)epoch, phases)
             ? LIGER_ECUDA
             : 0;
}

// world ranks' regions[q] (each [2 staging buffers of cap][flag][counters], zeroed before the
// first use) and buffers bufs[q]; call number `epoch`: one cooperative launch
int oneshot_allreduce_emulated(void* const* bufs, size_t count, void* const* regions, int world, size_t cap,
                               uint64_t epoch, cudaStream_t st) {
  const size_t bytes = count * 2;
  if (world < 1 || world > PAR_MAX_WORLD || bytes > cap || bytes % 16 || cap % 256 || epoch == 0) return LIGER_EINVAL;
  if (!count) return 0;
  const int b = (int)(epoch & 1);
  EmuRanks r{};
  PeerPtrs pp{};
  for (int q = 0; q < world; ++q) {
    if (!bufs[q] || !regions[q] || reinterpret_cast<uintptr_t>(bufs[q]) % 16) return LIGER_EINVAL;
    char* reg = static_cast<char*>(regions[q]);
    r.buf[q] = static_cast<uint4*>(bufs[q]);
    r.stage[q] = reinterpret_cast<uint4*>(reg + (size_t)b * cap);
    r.flag[q] = reinterpret_cast<unsigned long long*>(reg + 2 * cap);
    r.counter[q] = reinterpret_cast<unsigned int*>(reg + 2 * cap + 128);
    pp.data[q] = r.stage[q];
    pp.flag[q] = r.flag[q];
  }
  const size_t n8 = bytes / 16;
  int nblk = (int)((n8 + PAR_THREADS - 1) / PAR_THREADS);
  nblk = nblk < 1 ? 1 : (nblk > 8 ? 8 : nblk);
  int dev = 0, per_sm = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, oneshot_ar_emulated_kernel, PAR_THREADS, 0);
  if (world * nblk > per_sm * sms) return LIGER_EINVAL;   // every block must be co-resident
  unsigned long long ep = epoch;
  int w = world;
  void* args[] = {&r, (void*)&n8, &pp, &w, &ep, &nblk};
  return cudaLaunchCooperativeKernel((const void*)oneshot_ar_emulated_kernel, dim3(world * nblk), dim3(PAR_THREADS),
                                     args, 0, st) == cudaSuccess
             ? 0
             : LIGER_ECUDA;
}

void preload_peer_ar_kernel() {
  preload_kernel(oneshot_ar_bf16_kernel);
  preload_kernel(oneshot_ar_emulated_kernel);
}

}  // namespace liger
