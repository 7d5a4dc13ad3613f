// a10: sharded-state communication (placeholder until the NCCL path lands).
#include "comm.h"

namespace qgpu {

struct Comm {
  int dummy;
};

qgpu_status comm_create(Comm** out, const qgpu_config&, cudaStream_t, std::string* err) {
  *out = nullptr;
  *err = "world_size > 1 is not available in this build yet";
  return QGPU_ERR_UNSUPPORTED;
}
void comm_destroy(Comm* c) { delete c; }
qgpu_status comm_probabilities_finish(Comm*, double*, int, uint64_t, cudaStream_t) {
  return QGPU_ERR_UNSUPPORTED;
}
qgpu_status comm_get_amplitudes(Comm*, qgpu_state*, uint64_t, uint64_t, double*) {
  return QGPU_ERR_UNSUPPORTED;
}

}  // namespace qgpu
