// a10: communication for sharded states (world_size = 2^g GPUs, one process per GPU, NCCL over
// NVLink / NVSwitch). NCCL is loaded with dlopen only when world_size > 1 (the torch-bundled
// libnccl.so.2, located through $QGPU_NCCL_LIB by the Python binding).
//
// Batched global-local swap: s rank bits j[k] are exchanged with s local positions
// l[k] in ONE all-to-all among the 2^s ranks of a group (the ranks that differ only in the j[k]):
// block d of a rank's live amplitudes (its bits at the l[k] = d) goes to the peer whose rank bits
// are d, and comes back from that peer into the same slots. It is an all-to-all of grouped
// ncclSend / ncclRecv (NCCL's own all-to-all is the same grouped point-to-point; here the group
// is a subset of the ranks whenever s < g, and the rank's own block never moves). Slabs of every
// block go through two staging sets: pack (state's stream) -> send/recv (communication stream) ->
// unpack (state's stream), so NVLink transfers slab k while the SMs pack k+1 and unpack k-1.
#include "comm.h"

#include <dlfcn.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

namespace qgpu {

namespace {

typedef struct ncclComm* ncclComm_t;
typedef struct {
  char internal[128];
} ncclUniqueId;
typedef int ncclResult_t;
constexpr int kNcclUint64 = 5;
constexpr int kNcclFloat64 = 8;
constexpr int kNcclSum = 0;
constexpr ncclResult_t kNcclInProgress = 7;

struct NcclLib {
  bool tried = false, ok = false;
  std::string err;
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*commGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
  ncclResult_t (*groupStart)() = nullptr;
  ncclResult_t (*groupEnd)() = nullptr;
  ncclResult_t (*send)(const void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*recv)(void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*allReduce)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*allGather)(const void*, void*, size_t, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*errStr)(ncclResult_t) = nullptr;
};

NcclLib& nccl() {
  static NcclLib L;
  if (L.tried) return L;
  L.tried = true;
  void* h = nullptr;
  if (const char* ev = std::getenv("QGPU_NCCL_LIB")) h = dlopen(ev, RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    L.err = "libnccl.so.2 not found (set QGPU_NCCL_LIB)";
    return L;
  }
#define QGPU_NSYM(f, name)                                     \
  L.f = reinterpret_cast<decltype(L.f)>(dlsym(h, name));        \
  if (!L.f) {                                                  \
    L.err = std::string("missing ") + name;                    \
    return L;                                                  \
  }
  QGPU_NSYM(getUniqueId, "ncclGetUniqueId")
  QGPU_NSYM(commInitRank, "ncclCommInitRank")
  QGPU_NSYM(commDestroy, "ncclCommDestroy")
  QGPU_NSYM(commGetAsyncError, "ncclCommGetAsyncError")
  QGPU_NSYM(groupStart, "ncclGroupStart")
  QGPU_NSYM(groupEnd, "ncclGroupEnd")
  QGPU_NSYM(send, "ncclSend")
  QGPU_NSYM(recv, "ncclRecv")
  QGPU_NSYM(allReduce, "ncclAllReduce")
  QGPU_NSYM(allGather, "ncclAllGather")
  QGPU_NSYM(errStr, "ncclGetErrorString")
#undef QGPU_NSYM
  L.ok = true;
  return L;
}

}  // namespace

struct Comm {
  ncclComm_t comm = nullptr;
  int rank = 0, world = 1;
  cudaStream_t s_comm = nullptr;       // NCCL transfers of the pipelined swap
  cudaEvent_t ev_packed[2] = {}, ev_xfer[2] = {}, ev_join = nullptr;
  double2* send[2] = {};               // staging sets: (world - 1) blocks of `slab` amplitudes
  double2* recv[2] = {};
  uint64_t slab_cap = 0;               // amplitudes per block per staging set
};

#define QGPU_NCCL(call)                                                                    \
  do {                                                                                      \
    ncclResult_t _r = (call);                                                               \
    if (_r != 0) {                                                                          \
      *err = std::string("NCCL: ") + #call + ": " + (L.errStr ? L.errStr(_r) : "error");    \
      return QGPU_ERR_NCCL;                                                                 \
    }                                                                                       \
  } while (0)

#define QGPU_CUDA(call)                                                                     \
  do {                                                                                      \
    cudaError_t _e = (call);                                                                \
    if (_e != cudaSuccess) {                                                                \
      *err = std::string(#call) + ": " + cudaGetErrorString(_e);                            \
      return QGPU_ERR_CUDA;                                                                 \
    }                                                                                       \
  } while (0)

qgpu_status comm_unique_id(void* out128, std::string* err) {
  NcclLib& L = nccl();
  if (!L.ok) {
    *err = L.err;
    return QGPU_ERR_UNSUPPORTED;
  }
  ncclUniqueId id;
  QGPU_NCCL(L.getUniqueId(&id));
  std::memcpy(out128, &id, sizeof(id));
  return QGPU_OK;
}

int comm_world(const Comm* c) { return c ? c->world : 1; }

qgpu_status comm_create(Comm** out, const qgpu_config& cfg, cudaStream_t, uint64_t local_amps,
                        std::string* err) {
  *out = nullptr;
  NcclLib& L = nccl();
  if (!L.ok) {
    *err = L.err;
    return QGPU_ERR_NCCL;
  }
  auto* c = new Comm();
  c->rank = cfg.rank;
  c->world = cfg.world_size;
  ncclUniqueId id;
  std::memcpy(&id, cfg.nccl_unique_id, sizeof(id));
  ncclResult_t r = L.commInitRank(&c->comm, cfg.world_size, id, cfg.rank);
  if (r != 0) {
    *err = std::string("ncclCommInitRank: ") + L.errStr(r);
    delete c;
    return QGPU_ERR_NCCL;
  }
  // staging: per set (world - 1) blocks of slab_cap amplitudes; swap_slab_bytes bounds one set
  const uint64_t slab_bytes = std::max<uint64_t>(cfg.swap_slab_bytes, 1u << 20);
  const uint64_t blocks = uint64_t(std::max(1, c->world - 1));
  c->slab_cap = std::max<uint64_t>(1, std::min<uint64_t>(slab_bytes / 16 / blocks, std::max<uint64_t>(local_amps / 2, 1)));
  bool ok = cudaStreamCreateWithFlags(&c->s_comm, cudaStreamNonBlocking) == cudaSuccess &&
            cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming) == cudaSuccess;
  for (int i = 0; i < 2 && ok; ++i) {
    ok = cudaEventCreateWithFlags(&c->ev_packed[i], cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&c->ev_xfer[i], cudaEventDisableTiming) == cudaSuccess &&
         cudaMalloc(&c->send[i], c->slab_cap * blocks * 16) == cudaSuccess &&
         cudaMalloc(&c->recv[i], c->slab_cap * blocks * 16) == cudaSuccess;
  }
  if (!ok) {
    cudaGetLastError();
    *err = "swap staging / stream allocation failed";
    comm_destroy(c);
    return QGPU_ERR_OUT_OF_MEMORY;
  }
  *out = c;
  return QGPU_OK;
}

void comm_destroy(Comm* c) {
  if (!c) return;
  NcclLib& L = nccl();
  if (c->s_comm) cudaStreamSynchronize(c->s_comm);
  if (c->comm && L.ok) L.commDestroy(c->comm);
  for (int i = 0; i < 2; ++i) {
    if (c->send[i]) cudaFree(c->send[i]);
    if (c->recv[i]) cudaFree(c->recv[i]);
    if (c->ev_packed[i]) cudaEventDestroy(c->ev_packed[i]);
    if (c->ev_xfer[i]) cudaEventDestroy(c->ev_xfer[i]);
  }
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  if (c->s_comm) cudaStreamDestroy(c->s_comm);
  delete c;
}

qgpu_status comm_check(Comm* c, std::string* err) {
  if (!c) return QGPU_OK;
  NcclLib& L = nccl();
  ncclResult_t st = 0;
  QGPU_NCCL(L.commGetAsyncError(c->comm, &st));
  if (st != 0 && st != kNcclInProgress) {
    *err = std::string("NCCL asynchronous error: ") + L.errStr(st);
    return QGPU_ERR_NCCL;
  }
  return QGPU_OK;
}

qgpu_status comm_swap(Comm* c, double2* psi, const SwapGeom& g, uint64_t slab_amps, cudaStream_t st,
                      uint64_t* bytes_sent, std::string* err) {
  NcclLib& L = nccl();
  if (g.nb == 0 || g.rest == 0) return QGPU_OK;
  const uint64_t slab = std::max<uint64_t>(1, std::min({slab_amps, c->slab_cap * uint64_t(std::max(1, c->world - 1)) /
                                                                        uint64_t(g.nb), g.rest}));
  // the communication stream starts after everything enqueued so far on the state's stream
  QGPU_CUDA(cudaEventRecord(c->ev_join, st));
  QGPU_CUDA(cudaStreamWaitEvent(c->s_comm, c->ev_join, 0));
  BlockArgs a{};
  a.psi = psi;
  a.nins = g.nins;
  for (int k = 0; k < g.nins; ++k) a.ins[k] = g.ins[k];
  a.nb = g.nb;
  for (int b = 0; b < g.nb; ++b) a.pat[b] = g.pat[b];
  const uint64_t nslab = (g.rest + slab - 1) / slab;
  auto unpack = [&](uint64_t k) -> qgpu_status {
    const int i = int(k & 1);
    QGPU_CUDA(cudaStreamWaitEvent(st, c->ev_xfer[i], 0));
    a.buf = c->recv[i];
    a.t0 = k * slab;
    a.cnt = std::min(slab, g.rest - a.t0);
    QGPU_CUDA(launch_unpack_blocks(st, a));
    return QGPU_OK;
  };
  for (uint64_t k = 0; k < nslab; ++k) {
    const int i = int(k & 1);
    // pack slab k into set i (set i's previous transfer, slab k-2, was waited for by unpack(k-2))
    a.buf = c->send[i];
    a.t0 = k * slab;
    a.cnt = std::min(slab, g.rest - a.t0);
    const uint64_t cnt = a.cnt;
    QGPU_CUDA(launch_pack_blocks(st, a));
    QGPU_CUDA(cudaEventRecord(c->ev_packed[i], st));
    QGPU_CUDA(cudaStreamWaitEvent(c->s_comm, c->ev_packed[i], 0));
    QGPU_NCCL(L.groupStart());
    for (int b = 0; b < g.nb; ++b) {
      QGPU_NCCL(L.send(c->send[i] + uint64_t(b) * cnt, 2 * cnt, kNcclFloat64, g.peer[b], c->comm, c->s_comm));
      QGPU_NCCL(L.recv(c->recv[i] + uint64_t(b) * cnt, 2 * cnt, kNcclFloat64, g.peer[b], c->comm, c->s_comm));
    }
    QGPU_NCCL(L.groupEnd());
    QGPU_CUDA(cudaEventRecord(c->ev_xfer[i], c->s_comm));
    *bytes_sent += 16 * cnt * uint64_t(g.nb);
    // unpack the previous slab while this one is on the wire
    if (k >= 1)
      if (qgpu_status s = unpack(k - 1)) return s;
  }
  if (qgpu_status s = unpack(nslab - 1)) return s;
  return comm_check(c, err);
}

qgpu_status comm_activate_copy(Comm* c, double2* psi, int kg_from, int kg, uint64_t L_amps, cudaStream_t st,
                               std::string* err) {
  NcclLib& L = nccl();
  const int lo = 1 << kg_from, hi = 1 << kg;
  if (!L_amps) return QGPU_OK;
  QGPU_NCCL(L.groupStart());
  for (int step = lo; step < hi; step <<= 1) {
    // one new rank bit per step: ranks [step, 2 step) receive from r - step
    if (c->rank < step && c->rank + step < hi)
      QGPU_NCCL(L.send(psi, 2 * L_amps, kNcclFloat64, c->rank + step, c->comm, st));
    if (c->rank >= step && c->rank < 2 * step)
      QGPU_NCCL(L.recv(psi, 2 * L_amps, kNcclFloat64, c->rank - step, c->comm, st));
  }
  QGPU_NCCL(L.groupEnd());
  return comm_check(c, err);
}

qgpu_status comm_allreduce_sum(Comm* c, double* buf, size_t count, cudaStream_t st, std::string* err) {
  NcclLib& L = nccl();
  QGPU_NCCL(L.allReduce(buf, buf, count, kNcclFloat64, kNcclSum, c->comm, st));
  return comm_check(c, err);
}

qgpu_status comm_allgather_u64(Comm* c, const uint64_t* in, uint64_t* out, cudaStream_t st, std::string* err) {
  NcclLib& L = nccl();
  QGPU_NCCL(L.allGather(in, out, 1, kNcclUint64, c->comm, st));
  return comm_check(c, err);
}

qgpu_status comm_exchange(Comm* c, int n, const int* peer, const double* const* send, const size_t* scount,
                          double* const* recv, const size_t* rcount, cudaStream_t st, std::string* err) {
  NcclLib& L = nccl();
  QGPU_NCCL(L.groupStart());
  for (int i = 0; i < n; ++i) {
    if (scount[i]) QGPU_NCCL(L.send(send[i], scount[i], kNcclFloat64, peer[i], c->comm, st));
    if (rcount[i]) QGPU_NCCL(L.recv(recv[i], rcount[i], kNcclFloat64, peer[i], c->comm, st));
  }
  QGPU_NCCL(L.groupEnd());
  return comm_check(c, err);
}

}  // namespace qgpu
