// a10: communication for sharded states (world_size = 2^g GPUs, one process per GPU, NCCL over
// NVLink / NVSwitch). NCCL is loaded with dlopen only when world_size > 1 (the torch-bundled
// libnccl.so.2, located through $QGPU_NCCL_LIB by the Python binding).
//
// Global-local swap of rank bit j with local position lp: rank r (bit j = b) keeps
// its amplitudes with local bit lp = b and exchanges the half with lp = 1-b with its partner
// r ^ 2^j, whose half lands in the same slots (in place). The half is moved in slabs through
// two bounded staging buffers: pack (gather) -> ncclSend/ncclRecv (grouped) -> unpack (scatter).
#include "comm.h"

#include <dlfcn.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "kernels.h"

namespace qgpu {

namespace {

typedef struct ncclComm* ncclComm_t;
typedef struct {
  char internal[128];
} ncclUniqueId;
typedef int ncclResult_t;
constexpr int kNcclFloat64 = 8;
constexpr int kNcclSum = 0;

struct NcclLib {
  bool tried = false, ok = false;
  std::string err;
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*groupStart)() = nullptr;
  ncclResult_t (*groupEnd)() = nullptr;
  ncclResult_t (*send)(const void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*recv)(void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*allReduce)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
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
  QGPU_NSYM(groupStart, "ncclGroupStart")
  QGPU_NSYM(groupEnd, "ncclGroupEnd")
  QGPU_NSYM(send, "ncclSend")
  QGPU_NSYM(recv, "ncclRecv")
  QGPU_NSYM(allReduce, "ncclAllReduce")
  QGPU_NSYM(errStr, "ncclGetErrorString")
#undef QGPU_NSYM
  L.ok = true;
  return L;
}

}  // namespace

struct Comm {
  ncclComm_t comm = nullptr;
  int rank = 0, world = 1;
  double2* sendbuf = nullptr;
  double2* recvbuf = nullptr;
  uint64_t slab = 0;  // amplitudes per slab
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
  const uint64_t slab_bytes = std::max<uint64_t>(cfg.swap_slab_bytes, 1u << 20);
  c->slab = std::min<uint64_t>(slab_bytes / 16, std::max<uint64_t>(local_amps / 2, 1));
  if (cudaMalloc(&c->sendbuf, c->slab * 16) != cudaSuccess || cudaMalloc(&c->recvbuf, c->slab * 16) != cudaSuccess) {
    *err = "swap staging allocation failed";
    comm_destroy(c);
    return QGPU_ERR_OUT_OF_MEMORY;
  }
  *out = c;
  return QGPU_OK;
}

void comm_destroy(Comm* c) {
  if (!c) return;
  NcclLib& L = nccl();
  if (c->comm && L.ok) L.commDestroy(c->comm);
  if (c->sendbuf) cudaFree(c->sendbuf);
  if (c->recvbuf) cudaFree(c->recvbuf);
  delete c;
}

qgpu_status comm_swap_bit(Comm* c, double2* psi, int m, int rank, int j, int lp, cudaStream_t st,
                          std::string* err) {
  NcclLib& L = nccl();
  const int b = (rank >> j) & 1;
  const int partner = rank ^ (1 << j);
  const uint64_t half = 1ull << (m - 1);
  for (uint64_t t0 = 0; t0 < half; t0 += c->slab) {
    const uint64_t cnt = std::min(c->slab, half - t0);
    QGPU_CUDA(launch_pack_half(st, psi, c->sendbuf, lp, 1 - b, t0, cnt));
    QGPU_NCCL(L.groupStart());
    QGPU_NCCL(L.send(c->sendbuf, 2 * cnt, kNcclFloat64, partner, c->comm, st));
    QGPU_NCCL(L.recv(c->recvbuf, 2 * cnt, kNcclFloat64, partner, c->comm, st));
    QGPU_NCCL(L.groupEnd());
    QGPU_CUDA(launch_unpack_half(st, psi, c->recvbuf, lp, 1 - b, t0, cnt));
  }
  return QGPU_OK;
}

qgpu_status comm_allreduce_sum(Comm* c, double* buf, size_t count, cudaStream_t st, std::string* err) {
  NcclLib& L = nccl();
  QGPU_NCCL(L.allReduce(buf, buf, count, kNcclFloat64, kNcclSum, c->comm, st));
  return QGPU_OK;
}

}  // namespace qgpu
