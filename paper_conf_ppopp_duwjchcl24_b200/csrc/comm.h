// Communication backend interface of the tensor-parallel ranks (see comm.cu).
#pragma once
#include <cuda_runtime.h>
#include <nccl.h>
#include <stddef.h>
#include <stdint.h>

#include <string>

#include "kernels.h"

namespace liger {

struct NcclApi {
  bool ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi& nccl();


// One-shot all-reduce over peer memory (peer_ar.cu): every rank's staging region
// (peer_ar_region_bytes(cap) bytes, zeroed; [2 buffers][cap] + epoch flag) is
// mapped by every rank; calls must be issued in the same order on all ranks.
struct PeerAR {
  int world = 1, rank = 0;
  size_t cap = 0;
  void* local = nullptr;      // this rank's region (owned by the backend)
  void* peer[8] = {};         // every rank's region as seen from this rank (peer[rank] = local)
  unsigned int* counter = nullptr;
  uint64_t epoch = 0;
  int init(int world, int rank, size_t cap, void* local_region, void* const* peer_regions);
  // in place, sum in rank order; phases = LIGER_AR_PHASE_STAGE (stage + publish) |
  // LIGER_AR_PHASE_REDUCE (wait for every flag + sum); the serving path runs both
  int allreduce_bf16(void* buf, size_t count, cudaStream_t st, int phases = 3);
  unsigned int* fused_counter = nullptr;
  // take the next epoch for a fused producer/consumer pair (same order on all ranks)
  int fused_begin(size_t bytes, FusedARDesc* out);
  ~PeerAR();
};
size_t peer_ar_region_bytes(size_t cap);
// test vehicle: `world` ranks' one-shot all-reduces (call `epoch`) as one cooperative launch
int oneshot_allreduce_emulated(void* const* bufs, size_t count, void* const* regions, int world, size_t cap,
                               uint64_t epoch, cudaStream_t st);

enum CommDType { CD_BF16, CD_F32, CD_I32 };
enum CommOp { CO_SUM, CO_MAX };

struct Comm {
  std::string err;
  virtual ~Comm() {}
  // in-place all-reduce of `count` elements
  virtual int allreduce(void* buf, size_t count, CommDType dt, CommOp op, cudaStream_t st) = 0;
  // two all-gathers issued as one group: recv[q * n + i] = send_q[i]
  virtual int allgather2(const void* s0, void* r0, size_t n0, CommDType d0, const void* s1, void* r1, size_t n1,
                         CommDType d1, cudaStream_t st) = 0;
  // point-to-point (inter-operator pipeline baseline): `bytes` from this rank to `peer`
  virtual int send(const void* buf, size_t bytes, int peer, cudaStream_t st) = 0;
  virtual int recv(void* buf, size_t bytes, int peer, cudaStream_t st) = 0;
  virtual int check_async() = 0;
  // host-side barrier of the group (loopback: every rank's thread has arrived)
  virtual void barrier() {}
  // [collective] set up the one-shot peer all-reduce (called once by comm_create)
  virtual int init_peer(cudaStream_t) { return 0; }
  // the one-shot peer all-reduce state, or nullptr when this backend does not use it
  virtual PeerAR* peer_ar(cudaStream_t) { return nullptr; }
};

Comm* comm_create(int world, int rank, const uint8_t* uid, std::string* err);
bool uid_is_loopback(const uint8_t* uid);
void make_loopback_uid(uint8_t* uid);

}  // namespace liger
