// Store-path probe 2: write-only bandwidth of a persistent grid (the fused pass's launch shape)
// as a function of the tile order across CTAs and of CTAs per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/st_probe2 scripts/st_probe2.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

// ORDER 0: round-robin tile = bid + k*G; 1: chunks of CH consecutive tiles per CTA per round;
// 2: one contiguous range per CTA
template <int ORDER, int CH>
__global__ void wprobe(double2* psi, uint64_t ntiles, int tile_amps) {
  const int nthr = blockDim.x;
  const int per = tile_amps / nthr;
  const uint64_t G = gridDim.x;
  const uint64_t per_cta = (ntiles + G - 1) / G;
  for (uint64_t k = 0;; ++k) {
    uint64_t t;
    if (ORDER == 0) t = blockIdx.x + k * G;
    else if (ORDER == 1) t = ((k / CH) * G + blockIdx.x) * CH + (k % CH);
    else t = blockIdx.x * per_cta + k;
    if (ORDER == 2 ? (k >= per_cta || t >= ntiles) : t >= ntiles) break;
    double2* base = psi + t * tile_amps;
    for (int r = 0; r < per; ++r) __stcs(base + uint64_t(r) * nthr + threadIdx.x, make_double2(r, t));
  }
}

template <int ORDER, int CH>
float run(double2* psi, uint64_t amps, int grid, int block, int tile_amps) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const uint64_t ntiles = amps / tile_amps;
  wprobe<ORDER, CH><<<grid, block>>>(psi, ntiles, tile_amps);
  float best = 1e30f;
  for (int i = 0; i < 5; ++i) {
    cudaEventRecord(e0);
    wprobe<ORDER, CH><<<grid, block>>>(psi, ntiles, tile_amps);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  return best;
}

int main() {
  const uint64_t amps = 1ull << 28;
  double2* psi;
  cudaMalloc(&psi, amps * 16);
  const double GB = amps * 16 / 1e9;
  for (int cps : {1, 2, 4})
    for (int block : {256, 128})
      for (int tile : {4096, 2048}) {
        const int g = 148 * cps;
        printf("ctas/SM %d blk %4d tile %5d  rr %5.0f  ch4 %5.0f  ch16 %5.0f  ch64 %5.0f  range %5.0f GB/s\n", cps,
               block, tile, GB / run<0, 1>(psi, amps, g, block, tile) * 1e3,
               GB / run<1, 4>(psi, amps, g, block, tile) * 1e3, GB / run<1, 16>(psi, amps, g, block, tile) * 1e3,
               GB / run<1, 64>(psi, amps, g, block, tile) * 1e3, GB / run<2, 1>(psi, amps, g, block, tile) * 1e3);
      }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
