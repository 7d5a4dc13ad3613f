// a10: communication for sharded states (world_size = 2^g GPUs, one process per GPU).
// NCCL is loaded at run time (dlopen) only when world_size > 1 with an NCCL unique id.
#pragma once

#include <cuda_runtime.h>

#include <string>

#include "qgpu_internal.h"

namespace qgpu {

struct Comm;

qgpu_status comm_unique_id(void* out128, std::string* err);
qgpu_status comm_create(Comm** out, const qgpu_config& cfg, cudaStream_t stream, uint64_t local_amps,
                        std::string* err);
void comm_destroy(Comm* c);
// In-place global-local swap of rank bit j with local position lp (pairwise exchange with
// rank ^ 2^j, slabbed through bounded staging).
qgpu_status comm_swap_bit(Comm* c, double2* psi, int m, int rank, int j, int lp, cudaStream_t st,
                          std::string* err);
// In-place all-reduce (sum) of `count` doubles on the device.
qgpu_status comm_allreduce_sum(Comm* c, double* buf, size_t count, cudaStream_t st, std::string* err);

}  // namespace qgpu
