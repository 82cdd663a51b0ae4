// Communication backends of the tensor-parallel ranks.
//
//  * NcclComm: NCCL over NVLink/NVSwitch (the product path; libnccl is loaded with
//    dlopen and bootstrapped with a caller-broadcast ncclUniqueId).
//  * LoopbackComm: the ranks of a group are threads of ONE process sharing one
//    GPU; a collective is a host rendezvous plus device kernels that read every
//    rank's buffer (rank order, deterministic).  It exists so the whole t > 1
//    path -- communication stream, Algorithm 1 rounds with real secondary
//    subsets, decomposition, hybrid E1/E2 sync, token all-gather -- can be run
//    and checked on a single GPU.  Selected by a uid from
//    liger_loopback_unique_id().
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <dlfcn.h>
#include <nccl.h>
#include <stdint.h>
#include <string.h>

#include <condition_variable>
#include <map>
#include <mutex>
#include <random>
#include <string>
#include <vector>

#include "comm.h"
#include "common.cuh"
#include "kernels.h"

namespace liger {

// ------------------------------------------------------------------ NCCL (dlopen)
NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* names[] = {"libnccl.so.2", "libnccl.so",
                           "/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/lib/libnccl.so.2"};
    void* h = nullptr;
    for (const char* n : names)
      if ((h = dlopen(n, RTLD_NOW | RTLD_GLOBAL))) break;
    if (!h) return;
#define LIGER_SYM(field, name) api.field = reinterpret_cast<decltype(api.field)>(dlsym(h, name))
    LIGER_SYM(GetUniqueId, "ncclGetUniqueId");
    LIGER_SYM(CommInitRank, "ncclCommInitRank");
    LIGER_SYM(AllReduce, "ncclAllReduce");
    LIGER_SYM(AllGather, "ncclAllGather");
    LIGER_SYM(Send, "ncclSend");
    LIGER_SYM(Recv, "ncclRecv");
    LIGER_SYM(GroupStart, "ncclGroupStart");
    LIGER_SYM(GroupEnd, "ncclGroupEnd");
    LIGER_SYM(CommDestroy, "ncclCommDestroy");
    LIGER_SYM(CommGetAsyncError, "ncclCommGetAsyncError");
    LIGER_SYM(GetErrorString, "ncclGetErrorString");
#undef LIGER_SYM
    api.ok = api.GetUniqueId && api.CommInitRank && api.AllReduce && api.AllGather && api.GroupStart &&
             api.GroupEnd && api.CommDestroy && api.GetErrorString;
  });
  return api;
}

static ncclDataType_t nccl_dt(CommDType d) {
  return d == CD_BF16 ? ncclBfloat16 : d == CD_F32 ? ncclFloat32 : ncclInt32;
}
static size_t dt_size(CommDType d) { return d == CD_BF16 ? 2 : 4; }

// One-shot peer all-reduce for decode-size bf16 sums (LIGER_ONESHOT_AR=0/1 overrides
// the backend default; LIGER_ONESHOT_MAX_KB the largest message, default 1024).
static bool oneshot_enabled(bool dflt) {
  const char* e = getenv("LIGER_ONESHOT_AR");
  return e ? atoi(e) != 0 : dflt;
}
static size_t oneshot_cap() {
  const char* e = getenv("LIGER_ONESHOT_MAX_KB");
  const size_t kb = e ? (size_t)atoll(e) : 1024;
  return (kb * 1024 + 255) / 256 * 256;
}
static bool oneshot_eligible(size_t count, CommDType dt, CommOp op, const void* buf) {
  return dt == CD_BF16 && op == CO_SUM && count * 2 <= oneshot_cap() && (count * 2) % 16 == 0 &&
         reinterpret_cast<uintptr_t>(buf) % 16 == 0;
}

struct NcclComm : Comm {
  ncclComm_t comm = nullptr;
  int world = 1, rank = 0;
  bool oneshot = false;
  PeerAR* par = nullptr;
  void* region = nullptr;
  void* mapped[8] = {};
  ~NcclComm() override {
    cudaDeviceSynchronize();
    delete par;
    for (int q = 0; q < world && q < 8; ++q)
      if (mapped[q] && q != rank) cudaIpcCloseMemHandle(mapped[q]);
    if (region) cudaFree(region);
    if (comm) nccl().CommDestroy(comm);
  }
  // all ranks' min of a local flag (a collective every rank reaches, whatever its flag)
  int agree_min(int v, cudaStream_t st, int* out) {
    int32_t* d = nullptr;
    if (cudaMalloc(&d, sizeof(int32_t)) != cudaSuccess) return LIGER_ENOMEM;
    cudaMemcpy(d, &v, sizeof(int32_t), cudaMemcpyHostToDevice);
    ncclResult_t r = nccl().AllReduce(d, d, 1, ncclInt32, ncclMin, comm, st);
    if (r == ncclSuccess && cudaStreamSynchronize(st) == cudaSuccess)
      cudaMemcpy(out, d, sizeof(int32_t), cudaMemcpyDeviceToHost);
    cudaFree(d);
    return r == ncclSuccess ? 0 : LIGER_ENCCL;
  }
  // [collective, at communicator creation] map every rank's staging region: CUDA IPC
  // handles exchanged with an NCCL all-gather (same-node NVLink / NVSwitch peers).  Every
  // rank takes part in every collective whatever its local outcome, and the ranks agree
  // (NCCL min) first on the allocation and then on every rank having mapped every peer;
  // if any step failed anywhere, all of them use NCCL all-reduces (no rank returns early
  // while its peers wait in a collective).
  int setup_oneshot(cudaStream_t st) {
    const size_t cap = oneshot_cap(), rb = peer_ar_region_bytes(cap);
    int ok = world <= 8 ? 1 : 0;
    if (ok && (cudaMalloc(&region, rb) != cudaSuccess || cudaMemset(region, 0, rb) != cudaSuccess)) {
      cudaGetLastError();
      if (region) cudaFree(region);
      region = nullptr;
      ok = 0;
    }
    cudaIpcMemHandle_t h{};
    if (ok && cudaIpcGetMemHandle(&h, region) != cudaSuccess) {
      cudaGetLastError();
      ok = 0;
    }
    int all_ok = 0;
    if (int rc = agree_min(ok, st, &all_ok)) return rc;
    if (all_ok) {
      char* d = nullptr;
      if (cudaMalloc(&d, (size_t)64 * (world + 1)) != cudaSuccess) return LIGER_ENOMEM;
      cudaMemcpy(d + (size_t)64 * world, &h, 64, cudaMemcpyHostToDevice);
      ncclResult_t r = nccl().AllGather(d + (size_t)64 * world, d, 64, ncclUint8, comm, st);
      std::vector<cudaIpcMemHandle_t> all(world);
      if (r == ncclSuccess && cudaStreamSynchronize(st) == cudaSuccess)
        cudaMemcpy(all.data(), d, (size_t)64 * world, cudaMemcpyDeviceToHost);
      cudaFree(d);
      if (r != ncclSuccess) return LIGER_ENCCL;
      for (int q = 0; q < world && ok; ++q) {
        if (q == rank) {
          mapped[q] = region;
          continue;
        }
        if (cudaIpcOpenMemHandle(&mapped[q], all[q], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
          cudaGetLastError();
          mapped[q] = nullptr;
          ok = 0;
        }
      }
      if (int rc = agree_min(ok, st, &all_ok)) return rc;
    }
    if (!all_ok) {   // agreed fallback: NCCL for every all-reduce
      for (int q = 0; q < world; ++q)
        if (mapped[q] && q != rank) cudaIpcCloseMemHandle(mapped[q]);
      for (int q = 0; q < world; ++q) mapped[q] = nullptr;
      oneshot = false;
      err = "one-shot all-reduce disabled: a rank could not set up or map the peers' staging buffers";
      return 0;
    }
    par = new PeerAR();
    return par->init(world, rank, cap, region, mapped);
  }
  int init_peer(cudaStream_t st) override { return oneshot ? setup_oneshot(st) : 0; }
  PeerAR* peer_ar(cudaStream_t) override { return oneshot ? par : nullptr; }
  int allreduce(void* buf, size_t count, CommDType dt, CommOp op, cudaStream_t st) override {
    if (!count) return 0;
    if (oneshot && par && oneshot_eligible(count, dt, op, buf)) return par->allreduce_bf16(buf, count, st);
    ncclResult_t r = nccl().AllReduce(buf, buf, count, nccl_dt(dt), op == CO_SUM ? ncclSum : ncclMax, comm, st);
    if (r != ncclSuccess) {
      err = std::string("ncclAllReduce: ") + nccl().GetErrorString(r);
      return LIGER_ENCCL;
    }
    return 0;
  }
  int allgather2(const void* s0, void* r0, size_t n0, CommDType d0, const void* s1, void* r1, size_t n1,
                 CommDType d1, cudaStream_t st) override {
    nccl().GroupStart();
    nccl().AllGather(s0, r0, n0, nccl_dt(d0), comm, st);
    nccl().AllGather(s1, r1, n1, nccl_dt(d1), comm, st);
    ncclResult_t r = nccl().GroupEnd();
    if (r != ncclSuccess) {
      err = std::string("ncclAllGather: ") + nccl().GetErrorString(r);
      return LIGER_ENCCL;
    }
    return 0;
  }
  int send(const void* buf, size_t bytes, int peer, cudaStream_t st) override {
    if (!nccl().Send) return LIGER_ENCCL;
    ncclResult_t r = nccl().Send(buf, bytes, ncclUint8, peer, comm, st);
    if (r != ncclSuccess) {
      err = std::string("ncclSend: ") + nccl().GetErrorString(r);
      return LIGER_ENCCL;
    }
    return 0;
  }
  int recv(void* buf, size_t bytes, int peer, cudaStream_t st) override {
    if (!nccl().Recv) return LIGER_ENCCL;
    ncclResult_t r = nccl().Recv(buf, bytes, ncclUint8, peer, comm, st);
    if (r != ncclSuccess) {
      err = std::string("ncclRecv: ") + nccl().GetErrorString(r);
      return LIGER_ENCCL;
    }
    return 0;
  }
  int check_async() override {
    if (!nccl().CommGetAsyncError) return 0;
    ncclResult_t a = ncclSuccess;
    nccl().CommGetAsyncError(comm, &a);
    if (a != ncclSuccess && a != ncclInProgress) {
      err = std::string("NCCL async error: ") + nccl().GetErrorString(a);
      return LIGER_ENCCL;
    }
    return 0;
  }
};

// ------------------------------------------------------------------ loopback (ranks = threads, one GPU)
// Point-to-point mailbox of one directed pair (src -> dst): a ring of device
// slots.  send copies into slot k % NSLOT and records a per-slot event; recv
// waits for it and copies out, recording a per-slot "consumed" event that the
// sender waits on before reusing the slot.  The host only blocks when a sender
// is NSLOT messages ahead of its receiver's host (no cyclic wait: the
// receiver of a full ring is never waiting for that sender).
constexpr int P2P_SLOTS = 4;
struct P2PBox {
  std::mutex mu;
  std::condition_variable cv;
  uint64_t sent = 0, recvd = 0;              // messages enqueued by the two hosts
  void* slot[P2P_SLOTS] = {};
  size_t cap[P2P_SLOTS] = {};
  size_t len[P2P_SLOTS] = {};
  cudaEvent_t full[P2P_SLOTS] = {}, empty[P2P_SLOTS] = {};
  bool empty_recorded[P2P_SLOTS] = {};
};
struct P2PTable {
  std::mutex mu;
  std::map<std::pair<int, int>, P2PBox*> boxes;
  P2PBox* get(int s, int d) {
    std::lock_guard<std::mutex> l(mu);
    P2PBox*& b = boxes[{s, d}];
    if (!b) {
      b = new P2PBox();
      for (int i = 0; i < P2P_SLOTS; ++i) {
        cudaEventCreateWithFlags(&b->full[i], cudaEventDisableTiming);
        cudaEventCreateWithFlags(&b->empty[i], cudaEventDisableTiming);
      }
    }
    return b;
  }
  ~P2PTable() {
    for (auto& kv : boxes) {
      for (int i = 0; i < P2P_SLOTS; ++i) {
        if (kv.second->slot[i]) cudaFree(kv.second->slot[i]);
        cudaEventDestroy(kv.second->full[i]);
        cudaEventDestroy(kv.second->empty[i]);
      }
      delete kv.second;
    }
  }
};

struct LoopGroup {
  int world;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  // per-rank operands, double-buffered by generation parity: a rank can deposit
  // for generation g+1 while slower ranks still read generation g, and cannot
  // reach g+2 before every rank has left g.
  std::vector<const void*> a[2], b[2];
  std::vector<cudaEvent_t> ev[2];
  int members = 0;
  P2PTable p2p;
};

static std::mutex g_groups_mu;
static std::map<std::string, LoopGroup*> g_groups;

constexpr int LOOP_MAX_WORLD = 8;
template <typename T>
struct RankPtrs {
  const T* p[LOOP_MAX_WORLD];
};

// out[i] = reduce over ranks q = 0..world-1 (in order) of in_q[i]
template <typename T, bool MAX>
__global__ void loop_reduce_kernel(const RankPtrs<T> in, int world, T* out, size_t n) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    float acc = (float)in.p[0][i];
    for (int q = 1; q < world; ++q) acc = MAX ? fmaxf(acc, (float)in.p[q][i]) : acc + (float)in.p[q][i];
    out[i] = (T)acc;
  }
}
template <bool MAX>
__global__ void loop_reduce_bf16_kernel(const RankPtrs<__nv_bfloat16> in, int world, __nv_bfloat16* out, size_t n) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    float acc = __bfloat162float(in.p[0][i]);
    for (int q = 1; q < world; ++q) {
      const float v = __bfloat162float(in.p[q][i]);
      acc = MAX ? fmaxf(acc, v) : acc + v;
    }
    out[i] = __float2bfloat16_rn(acc);
  }
}

struct LoopbackComm : Comm {
  LoopGroup* g = nullptr;
  std::string key;
  int world = 1, rank = 0;
  cudaEvent_t ev_ready = nullptr, ev_done = nullptr;
  void* scratch = nullptr;
  size_t scratch_bytes = 0;
  ~LoopbackComm() override {
    cudaDeviceSynchronize();
    if (ev_ready) cudaEventDestroy(ev_ready);
    if (ev_done) cudaEventDestroy(ev_done);
    if (scratch) cudaFree(scratch);
    std::lock_guard<std::mutex> l(g_groups_mu);
    if (g && --g->members == 0) {
      g_groups.erase(key);
      delete g;
    }
  }
  // host rendezvous: deposit (x, y, e) for this rank, wait for all ranks, return everyone's
  void rendezvous(const void* x, const void* y, cudaEvent_t e, std::vector<const void*>* xs,
                  std::vector<const void*>* ys, std::vector<cudaEvent_t>* es) {
    std::unique_lock<std::mutex> l(g->mu);
    const uint64_t my_gen = g->gen;
    const int par = (int)(my_gen & 1);
    g->a[par][rank] = x;
    g->b[par][rank] = y;
    g->ev[par][rank] = e;
    if (++g->arrived == world) {
      g->arrived = 0;
      ++g->gen;
      g->cv.notify_all();
    } else {
      g->cv.wait(l, [&] { return g->gen != my_gen; });
    }
    *xs = g->a[par];
    *ys = g->b[par];
    *es = g->ev[par];
  }
  void wait_all(const std::vector<cudaEvent_t>& es, cudaStream_t st) {
    for (int q = 0; q < world; ++q) cudaStreamWaitEvent(st, es[q], 0);
  }
  int ensure_scratch(size_t bytes) {
    if (bytes <= scratch_bytes) return 0;
    cudaDeviceSynchronize();
    if (scratch) cudaFree(scratch);
    if (cudaMalloc(&scratch, bytes) != cudaSuccess) return LIGER_ENOMEM;
    scratch_bytes = bytes;
    return 0;
  }
  // No peer-memory kernels on this backend: its ranks share one GPU, and kernels that
  // wait on each other are not guaranteed to be co-scheduled there (B200_PROFILING.md).
  // The one-shot / fused kernels are tested phase by phase through the op-level C-ABI.
  int init_peer(cudaStream_t) override { return 0; }
  PeerAR* peer_ar(cudaStream_t) override { return nullptr; }
  int allreduce(void* buf, size_t count, CommDType dt, CommOp op, cudaStream_t st) override {
    if (!count) return 0;
    const size_t bytes = count * dt_size(dt);
    if (int rc = ensure_scratch(bytes)) return rc;
    std::vector<const void*> xs, ys;
    std::vector<cudaEvent_t> es;
    cudaEventRecord(ev_ready, st);
    rendezvous(buf, nullptr, ev_ready, &xs, &ys, &es);
    wait_all(es, st);
    const int blocks = (int)std::min<size_t>((count + 255) / 256, 148 * 8);
    if (dt == CD_BF16) {
      RankPtrs<__nv_bfloat16> in{};
      for (int q = 0; q < world; ++q) in.p[q] = (const __nv_bfloat16*)xs[q];
      if (op == CO_SUM)
        loop_reduce_bf16_kernel<false><<<blocks, 256, 0, st>>>(in, world, (__nv_bfloat16*)scratch, count);
      else
        loop_reduce_bf16_kernel<true><<<blocks, 256, 0, st>>>(in, world, (__nv_bfloat16*)scratch, count);
    } else if (dt == CD_F32) {
      RankPtrs<float> in{};
      for (int q = 0; q < world; ++q) in.p[q] = (const float*)xs[q];
      if (op == CO_SUM)
        loop_reduce_kernel<float, false><<<blocks, 256, 0, st>>>(in, world, (float*)scratch, count);
      else
        loop_reduce_kernel<float, true><<<blocks, 256, 0, st>>>(in, world, (float*)scratch, count);
    } else {
      return LIGER_EINVAL;
    }
    // every rank has read every input before anyone overwrites its buffer
    cudaEventRecord(ev_done, st);
    rendezvous(nullptr, nullptr, ev_done, &xs, &ys, &es);
    wait_all(es, st);
    cudaMemcpyAsync(buf, scratch, bytes, cudaMemcpyDeviceToDevice, st);
    return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
  }
  int allgather2(const void* s0, void* r0, size_t n0, CommDType d0, const void* s1, void* r1, size_t n1,
                 CommDType d1, cudaStream_t st) override {
    std::vector<const void*> xs, ys;
    std::vector<cudaEvent_t> es;
    cudaEventRecord(ev_ready, st);
    rendezvous(s0, s1, ev_ready, &xs, &ys, &es);
    wait_all(es, st);
    const size_t b0 = n0 * dt_size(d0), b1 = n1 * dt_size(d1);
    for (int q = 0; q < world; ++q) {
      if (xs[q] != (char*)r0 + q * b0) cudaMemcpyAsync((char*)r0 + q * b0, xs[q], b0, cudaMemcpyDeviceToDevice, st);
      if (ys[q] != (char*)r1 + q * b1) cudaMemcpyAsync((char*)r1 + q * b1, ys[q], b1, cudaMemcpyDeviceToDevice, st);
    }
    cudaEventRecord(ev_done, st);
    rendezvous(nullptr, nullptr, ev_done, &xs, &ys, &es);
    wait_all(es, st);
    return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
  }
  int send(const void* buf, size_t bytes, int peer, cudaStream_t st) override {
    P2PBox* b = g->p2p.get(rank, peer);
    std::unique_lock<std::mutex> l(b->mu);
    b->cv.wait(l, [&] { return b->sent - b->recvd < (uint64_t)P2P_SLOTS; });   // ring has room (host)
    const int k = (int)(b->sent % P2P_SLOTS);
    if (b->cap[k] < bytes) {
      if (b->slot[k]) {
        cudaEventSynchronize(b->empty[k]);
        cudaFree(b->slot[k]);
      }
      if (cudaMalloc(&b->slot[k], bytes) != cudaSuccess) return LIGER_ENOMEM;
      b->cap[k] = bytes;
    }
    if (b->empty_recorded[k]) cudaStreamWaitEvent(st, b->empty[k], 0);   // receiver done with the slot
    cudaMemcpyAsync(b->slot[k], buf, bytes, cudaMemcpyDeviceToDevice, st);
    cudaEventRecord(b->full[k], st);
    b->len[k] = bytes;
    ++b->sent;
    b->cv.notify_all();
    return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
  }
  int recv(void* buf, size_t bytes, int peer, cudaStream_t st) override {
    P2PBox* b = g->p2p.get(peer, rank);
    std::unique_lock<std::mutex> l(b->mu);
    b->cv.wait(l, [&] { return b->sent > b->recvd; });   // the matching send was enqueued (host)
    const int k = (int)(b->recvd % P2P_SLOTS);
    if (b->len[k] != bytes) {
      err = "loopback recv: size mismatch";
      return LIGER_EINVAL;
    }
    cudaStreamWaitEvent(st, b->full[k], 0);
    cudaMemcpyAsync(buf, b->slot[k], bytes, cudaMemcpyDeviceToDevice, st);
    cudaEventRecord(b->empty[k], st);
    b->empty_recorded[k] = true;
    ++b->recvd;
    b->cv.notify_all();
    return cudaGetLastError() == cudaSuccess ? 0 : LIGER_ECUDA;
  }
  int check_async() override { return 0; }
  void barrier() override {
    std::vector<const void*> xs, ys;
    std::vector<cudaEvent_t> es;
    rendezvous(nullptr, nullptr, nullptr, &xs, &ys, &es);
  }
};

static const char kLoopMagic[16] = {'L', 'I', 'G', 'E', 'R', '-', 'L', 'O', 'O', 'P', 'B', 'A', 'C', 'K', ':', 0};

bool uid_is_loopback(const uint8_t* uid) { return uid && memcmp(uid, kLoopMagic, 16) == 0; }

void make_loopback_uid(uint8_t* uid) {
  memset(uid, 0, 128);
  memcpy(uid, kLoopMagic, 16);
  std::random_device rd;
  for (int i = 16; i < 48; ++i) uid[i] = (uint8_t)(rd() & 0xff);
}

Comm* comm_create(int world, int rank, const uint8_t* uid, std::string* err) {
  if (uid_is_loopback(uid)) {
    auto* c = new LoopbackComm();
    c->world = world;
    c->rank = rank;
    c->key.assign((const char*)uid, 48);
    {
      std::lock_guard<std::mutex> l(g_groups_mu);
      LoopGroup*& g = g_groups[c->key];
      if (!g) {
        g = new LoopGroup();
        g->world = world;
        for (int i = 0; i < 2; ++i) {
          g->a[i].assign(world, nullptr);
          g->b[i].assign(world, nullptr);
          g->ev[i].assign(world, nullptr);
        }
      }
      if (g->world != world) {
        *err = "loopback group world size mismatch";
        delete c;
        return nullptr;
      }
      ++g->members;
      c->g = g;
    }
    if (world > LOOP_MAX_WORLD) {
      *err = "loopback communicator: at most 8 ranks";
      delete c;
      return nullptr;
    }
    if (cudaEventCreateWithFlags(&c->ev_ready, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_done, cudaEventDisableTiming) != cudaSuccess) {
      *err = "loopback communicator: CUDA allocation failed";
      delete c;
      return nullptr;
    }
    if (c->init_peer(nullptr)) {
      *err = "loopback communicator: one-shot setup failed";
      delete c;
      return nullptr;
    }
    return c;
  }
  if (!nccl().ok) {
    *err = "NCCL library not loadable";
    return nullptr;
  }
  ncclUniqueId id;
  memcpy(&id, uid, sizeof(id));
  auto* c = new NcclComm();
  c->world = world;
  c->rank = rank;
  c->oneshot = oneshot_enabled(false);   // IPC path: opt-in (LIGER_ONESHOT_AR=1) until measured on NVLink
  ncclResult_t r = nccl().CommInitRank(&c->comm, world, id, rank);
  if (r != ncclSuccess) {
    *err = std::string("ncclCommInitRank: ") + nccl().GetErrorString(r);
    c->comm = nullptr;
    delete c;
    return nullptr;
  }
  // the one-shot staging buffers are set up here, eagerly (a collective of every rank),
  // never lazily inside a serving call
  cudaStream_t st = nullptr;
  int rc = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) == cudaSuccess ? c->init_peer(st) : LIGER_ECUDA;
  if (st) cudaStreamDestroy(st);
  if (rc) {
    *err = "NCCL communicator: one-shot all-reduce setup failed (" + c->err + ")";
    delete c;
    return nullptr;
  }
  return c;
}

void preload_peer_ar_kernel();
void preload_comm_kernels() {
  preload_kernel(loop_reduce_bf16_kernel<false>);
  preload_kernel(loop_reduce_bf16_kernel<true>);
  preload_kernel(loop_reduce_kernel<float, false>);
  preload_kernel(loop_reduce_kernel<float, true>);
  preload_peer_ar_kernel();
}

}  // namespace liger
