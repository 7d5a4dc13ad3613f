// Store-path probe: write-only HBM bandwidth by cache hint and width, for the fused pass's store
// shape (lanes contiguous, 16 slots per thread per 64 KiB tile, persistent grid).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/st_probe scripts/st_probe.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

template <int HINT, int W>
__device__ __forceinline__ void st(double2* p, double x, double y) {
  if constexpr (W == 16) {
    if constexpr (HINT == 0) asm volatile("st.global.v2.f64 [%0], {%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
    if constexpr (HINT == 1) asm volatile("st.global.cs.v2.f64 [%0], {%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
    if constexpr (HINT == 2) asm volatile("st.global.cg.v2.f64 [%0], {%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
    if constexpr (HINT == 3) asm volatile("st.global.L1::no_allocate.v2.f64 [%0], {%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
  } else {
    if constexpr (HINT == 0) asm volatile("st.global.v4.f64 [%0], {%1,%2,%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
    if constexpr (HINT == 1) asm volatile("st.global.cs.v4.f64 [%0], {%1,%2,%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
    if constexpr (HINT == 2) asm volatile("st.global.cg.v4.f64 [%0], {%1,%2,%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
    if constexpr (HINT == 3) asm volatile("st.global.L1::no_allocate.v4.f64 [%0], {%1,%2,%1,%2};" ::"l"(p), "d"(x), "d"(y) : "memory");
  }
}

// one tile = 4096 amplitudes; thread t stores slots r*nthr + t (W/16 amps per access)
template <int HINT, int W>
__global__ void wprobe(double2* psi, uint64_t ntiles) {
  constexpr int A = W / 16;
  const int nthr = blockDim.x;
  const int per = 4096 / A / nthr;
  for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    double2* base = psi + t * 4096;
    for (int r = 0; r < per; ++r) st<HINT, W>(base + (uint64_t(r) * nthr + threadIdx.x) * A, double(r), double(t));
  }
}

template <int HINT, int W>
float run(double2* psi, uint64_t ntiles, int grid, int block) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  wprobe<HINT, W><<<grid, block>>>(psi, ntiles);
  float best = 1e30f;
  for (int i = 0; i < 5; ++i) {
    cudaEventRecord(e0);
    wprobe<HINT, W><<<grid, block>>>(psi, ntiles);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  return best;
}

int main() {
  const uint64_t amps = 1ull << 28;  // 4 GiB
  double2* psi;
  cudaMalloc(&psi, amps * 16);
  const uint64_t ntiles = amps / 4096;
  const double GB = amps * 16 / 1e9;
  const char* hn[4] = {"wb", "cs", "cg", "na"};
  for (int block : {256, 512, 1024})
    for (int g : {148, 296, 592, 148 * 16}) {
      printf("grid %5d blk %4d ", g, block);
      float r[8] = {run<0, 16>(psi, ntiles, g, block), run<1, 16>(psi, ntiles, g, block),
                    run<2, 16>(psi, ntiles, g, block), run<3, 16>(psi, ntiles, g, block),
                    run<0, 32>(psi, ntiles, g, block), run<1, 32>(psi, ntiles, g, block),
                    run<2, 32>(psi, ntiles, g, block), run<3, 32>(psi, ntiles, g, block)};
      for (int i = 0; i < 8; ++i) printf(" %s%d %5.0f", hn[i & 3], i < 4 ? 16 : 32, GB / r[i] * 1e3);
      printf(" GB/s\n");
    }
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int i = 0; i < 5; ++i) {
    cudaEventRecord(e0);
    cudaMemsetAsync(psi, 0, amps * 16);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  printf("cudaMemset %6.0f GB/s\n%s\n", GB / best * 1e3, cudaGetErrorString(cudaGetLastError()));
}
