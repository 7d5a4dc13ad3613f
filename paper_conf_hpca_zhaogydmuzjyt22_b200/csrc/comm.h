// a10: communication for sharded states (world_size = 2^g GPUs, one process per GPU).
// NCCL is loaded at run time (dlopen) only when world_size > 1 with an NCCL unique id.
#pragma once

#include <cuda_runtime.h>

#include <algorithm>
#include <string>

#include "kernels.h"
#include "qgpu_internal.h"

namespace qgpu {

struct Comm;

// Geometry of one batched global-local swap as seen by one rank:
// rank bits j[k] <-> local positions l[k], k < s. The rank's live local amplitudes [0, L) split
// into 2^s blocks by their bits at the l[k]; block d (bit k of d = the bit at l[k]) goes to the
// group peer whose rank bits j[k] equal d, and the peer's block for this rank lands in the same
// slots (in place). The rank keeps its own block e (its rank bits at j[k]).
struct SwapGeom {
  int s = 0;
  int nins = 0;
  int ins[8] = {};                 // l[k] ascending (rest index -> live index deposit)
  int e = 0;                       // this rank's own block
  int nb = 0;                      // blocks exchanged = 2^s - 1
  int dlist[kMaxSwapBlocks] = {};  // block patterns, ascending, e skipped
  int peer[kMaxSwapBlocks] = {};   // rank receiving block dlist[b] (and sending its block e back)
  uint64_t pat[kMaxSwapBlocks] = {};
  uint64_t rest = 0;               // rest indices per block: L >> s
  void init(int rank, int s_, const int* j, const int* l, uint64_t L) {
    s = s_;
    nins = s;
    for (int k = 0; k < s; ++k) ins[k] = l[k];
    std::sort(ins, ins + s);
    e = 0;
    int jmask = 0;
    for (int k = 0; k < s; ++k) {
      e |= ((rank >> j[k]) & 1) << k;
      jmask |= 1 << j[k];
    }
    nb = 0;
    for (int d = 0; d < (1 << s); ++d) {
      if (d == e) continue;
      int pr = rank & ~jmask;
      uint64_t pt = 0;
      for (int k = 0; k < s; ++k)
        if (d >> k & 1) {
          pr |= 1 << j[k];
          pt |= 1ull << l[k];
        }
      dlist[nb] = d;
      peer[nb] = pr;
      pat[nb] = pt;
      ++nb;
    }
    rest = L >> s;
  }
  // slot of block pattern d in this rank's staging (d != e)
  int slot(int d) const { return d < e ? d : d - 1; }
};

qgpu_status comm_unique_id(void* out128, std::string* err);
qgpu_status comm_create(Comm** out, const qgpu_config& cfg, cudaStream_t stream, uint64_t local_amps,
                        std::string* err);
void comm_destroy(Comm* c);
// Batched in-place global-local swap (geometry g) of this rank's live local amplitudes, slabbed
// through two staging sets: pack (state's stream) -> grouped ncclSend/ncclRecv with every group
// peer (a communication stream) -> unpack (state's stream), so the transfer of slab k overlaps
// the pack of slab k+1 and the unpack of slab k-1. *bytes_sent += amplitude bytes sent.
qgpu_status comm_swap(Comm* c, double2* psi, const SwapGeom& g, uint64_t slab_amps, cudaStream_t st,
                      uint64_t* bytes_sent, std::string* err);
// Cross-rank first-touch expand (PK_ACTIVATE with act_copy): ranks [2^kg_from, 2^kg) receive the
// live prefix [0, L) of rank r - 2^kg_from.
qgpu_status comm_activate_copy(Comm* c, double2* psi, int kg_from, int kg, uint64_t L, cudaStream_t st,
                               std::string* err);
// In-place all-reduce (sum) of `count` doubles on the device.
qgpu_status comm_allreduce_sum(Comm* c, double* buf, size_t count, cudaStream_t st, std::string* err);
// All-gather of one uint64 per rank (device buffers: in[1], out[world]).
qgpu_status comm_allgather_u64(Comm* c, const uint64_t* in, uint64_t* out, cudaStream_t st, std::string* err);
// Grouped point-to-point: send[i] (count[i] doubles) to peer[i] and recv[i] from peer[i].
qgpu_status comm_exchange(Comm* c, int n, const int* peer, const double* const* send, const size_t* scount,
                          double* const* recv, const size_t* rcount, cudaStream_t st, std::string* err);
// Non-blocking poll of the communicator's asynchronous error state (ncclCommGetAsyncError).
qgpu_status comm_check(Comm* c, std::string* err);
int comm_world(const Comm* c);

}  // namespace qgpu
