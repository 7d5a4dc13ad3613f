// a10: communication for sharded states (world_size = 2^g GPUs, one process per GPU).
// NCCL is loaded at run time (dlopen) only when world_size > 1.
#pragma once

#include <cuda_runtime.h>

#include <string>

#include "qgpu_internal.h"

struct qgpu_state;

namespace qgpu {

struct Comm;

qgpu_status comm_create(Comm** out, const qgpu_config& cfg, cudaStream_t stream, std::string* err);
void comm_destroy(Comm* c);
// all-reduce (sum) of the 2^m probability buckets held in dev_buf (in place), after folding
// the rank-bit qubits (rank_fixed: bit j set = requested qubit j is a rank bit equal to 1 here)
qgpu_status comm_probabilities_finish(Comm* c, double* dev_buf, int m, uint64_t rank_fixed,
                                      cudaStream_t stream);
qgpu_status comm_get_amplitudes(Comm* c, qgpu_state* st, uint64_t start, uint64_t count,
                                double* out);

}  // namespace qgpu
