// Per-pass NVRTC specialisation of the fused tile kernel (jit.cpp).
#pragma once

#include <cuda_runtime.h>

#include <string>

#include "qgpu_internal.h"

namespace qgpu {

// CUDA source of the specialised kernel for one tile pass (host-only, deterministic).
std::string tile_jit_source(const Pass& p);
// Compile source to an sm_100a cubin with NVRTC (works without a GPU).
bool jit_compile_cubin(const std::string& src, std::string* cubin, std::string* log);
// NVRTC and the driver API could be loaded.
bool jit_available(std::string* why);
// Compile-or-fetch and launch; cudaErrorNotSupported when the JIT is unavailable.
cudaError_t launch_tile_jit(cudaStream_t st, const Pass& p, const TileArgs& a, size_t smem, int num_sms,
                            double* compile_ms);

}  // namespace qgpu
