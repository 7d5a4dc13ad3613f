// Per-pass NVRTC specialisation of the fused tile kernel (jit.cpp).
#pragma once

#include <cuda_runtime.h>

#include <string>
#include <vector>

#include "qgpu_internal.h"

namespace qgpu {

// CUDA source of the specialised kernel for one tile pass (host-only, deterministic).
// hist_mode >= 0: fused-measurement variant (TileArgs::hacc); mode 2 with hist_key != ~0u: the
// compile-time reduce-scatter epilogue for unrequested lane bits (hist_key & 0xff) and dead
// register bits (hist_key >> 8), see hist_rs_key()
std::string tile_jit_source(const Pass& p, int hist_mode = -1, uint32_t hist_key = ~0u);
// Compile source to an sm_100a cubin with NVRTC (works without a GPU).
bool jit_compile_cubin(const std::string& src, std::string* cubin, std::string* log);
// Same, through the on-disk cubin cache ($QGPU_JIT_CACHE or <lib dir>/build/jitcache).
bool jit_cubin_cached(const std::string& src, std::string* cubin, std::string* log, bool* hit);
// NVRTC and the driver API could be loaded.
bool jit_available(std::string* why);
// Load (disk cache) or compile in parallel the kernels of the given passes; returns #loaded.
int jit_prepare(const std::vector<const Pass*>& passes, double* compile_ms);
// Compile-or-fetch and launch; cudaErrorNotSupported when the JIT is unavailable.
cudaError_t launch_tile_jit(cudaStream_t st, const Pass& p, const TileArgs& a, size_t smem, int num_sms,
                            double* compile_ms);

}  // namespace qgpu
