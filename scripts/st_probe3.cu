// Store-path probe 3: write-only bandwidth when a 64 KiB tile is 2^(12-r) runs of 2^r amplitudes
// spread over high address bits (the QFT_28 last pass: 8 runs of 8 KiB at 2^25-amplitude strides)
// vs one contiguous 64 KiB tile. Persistent grid, 1 CTA of 256 threads per SM, 16-byte stores.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/st_probe3 scripts/st_probe3.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void wprobe(double2* psi, uint64_t ntiles, int lowbits, int hipos, int nhi) {
  const int nthr = blockDim.x;
  for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    // tile index bits fill positions [lowbits, hipos) then >= hipos + nhi
    const uint64_t tlo = t & ((1ull << (hipos - lowbits)) - 1), thi = t >> (hipos - lowbits);
    const uint64_t base = (tlo << lowbits) | (thi << (hipos + nhi));
    for (int r = 0; r < 4096 / nthr; ++r) {
      const uint32_t j = uint32_t(r) * nthr + threadIdx.x;  // tile-local index
      const uint64_t lo = j & ((1u << lowbits) - 1), hi = j >> lowbits;
      __stcs(psi + (base | lo | (hi << hipos)), make_double2(r, t));
    }
  }
}

int main() {
  const int n = 28;
  const uint64_t amps = 1ull << n;
  double2* psi;
  cudaMalloc(&psi, amps * 16);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const double GB = amps * 16 / 1e9;
  for (int lowbits : {12, 11, 10, 9, 8, 7, 5}) {
    const int nhi = 12 - lowbits;
    for (int hipos : {lowbits, n - nhi}) {
      float best = 1e30f;
      for (int i = 0; i < 6; ++i) {
        cudaEventRecord(e0);
        wprobe<<<148, 256>>>(psi, amps / 4096, lowbits, hipos, nhi);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (i && ms < best) best = ms;
      }
      printf("runs of 2^%2d amps, high tile bits at %2d..%2d: %6.0f GB/s\n", lowbits, hipos, hipos + nhi - 1,
             GB / best * 1e3);
    }
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
