// HBM write / read / copy bandwidth probe for the access shapes the fused tile pass uses
// (16-byte and 32-byte vector accesses, lanes contiguous, 16 amplitudes per thread per tile,
// persistent grids of 1-2 CTAs per SM).  Bounds the expansion passes, which are write-only.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/bw_probe scripts/bw_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int W>  // W = 16 or 32 bytes per access
__device__ __forceinline__ void st(double2* p, double2 v) {
  if constexpr (W == 16) {
    __stcs(p, v);
  } else {
    asm volatile("st.global.cs.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(p), "d"(v.x), "d"(v.y), "d"(v.x), "d"(v.y)
                 : "memory");
  }
}
template <int W>
__device__ __forceinline__ double2 ld(const double2* p) {
  if constexpr (W == 16) {
    return __ldcs(p);
  } else {
    double a, b, c, d;
    asm volatile("ld.global.cs.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
    return make_double2(a + c, b + d);
  }
}

// one "tile" = 4096 amplitudes = 64 KiB; thread t of 256 owns 16 amps: W/16 consecutive amps per
// access, lanes contiguous
template <int W, int MODE>  // MODE 0 write, 1 read, 2 copy (in place: read then write)
__global__ void __launch_bounds__(256) probe(double2* psi, uint64_t ntiles, double2* sink) {
  constexpr int A = W / 16;              // amps per access
  constexpr int NACC = 16 / A;           // accesses per thread per tile
  double2 acc = make_double2(0, 0);
  for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    double2* base = psi + (t << 12);
    double2 v[NACC];
    if (MODE >= 1) {
#pragma unroll
      for (int r = 0; r < NACC; ++r) v[r] = ld<W>(base + (uint64_t(r) * 256 + threadIdx.x) * A);
    }
    if (MODE == 1) {
#pragma unroll
      for (int r = 0; r < NACC; ++r) { acc.x += v[r].x; acc.y += v[r].y; }
    } else {
#pragma unroll
      for (int r = 0; r < NACC; ++r) {
        double2 w = MODE == 2 ? make_double2(v[r].x * 0.5, v[r].y * 0.5) : make_double2(double(r), double(t));
        st<W>(base + (uint64_t(r) * 256 + threadIdx.x) * A, w);
      }
    }
  }
  if (MODE == 1 && acc.x == 12345.678) *sink = acc;
}

template <int W, int MODE>
float run(double2* psi, uint64_t ntiles, double2* sink, int grid) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  probe<W, MODE><<<grid, 256>>>(psi, ntiles, sink);
  float best = 1e30f;
  for (int i = 0; i < 5; ++i) {
    cudaEventRecord(e0);
    probe<W, MODE><<<grid, 256>>>(psi, ntiles, sink);
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
  double2 *psi, *sink;
  cudaMalloc(&psi, amps * 16);
  cudaMalloc(&sink, 16);
  cudaMemset(psi, 0, amps * 16);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const uint64_t ntiles = amps >> 12;
  const double GB = amps * 16.0 / 1e9;
  const int grids[] = {sms, 2 * sms, 4 * sms, 8 * sms};
  for (int g : grids) {
    printf("grid %5d  write16 %6.0f write32 %6.0f  read16 %6.0f read32 %6.0f  copy16 %6.0f copy32 %6.0f GB/s\n", g,
           GB / run<16, 0>(psi, ntiles, sink, g) * 1e3, GB / run<32, 0>(psi, ntiles, sink, g) * 1e3,
           GB / run<16, 1>(psi, ntiles, sink, g) * 1e3, GB / run<32, 1>(psi, ntiles, sink, g) * 1e3,
           2 * GB / run<16, 2>(psi, ntiles, sink, g) * 1e3, 2 * GB / run<32, 2>(psi, ntiles, sink, g) * 1e3);
  }
  float ms;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  cudaMemsetAsync(psi, 0, amps * 16);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  cudaEventElapsedTime(&ms, e0, e1);
  printf("cudaMemset %6.0f GB/s\n", GB / ms * 1e3);
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
