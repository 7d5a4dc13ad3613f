// GFC-style lossless compression of amplitude doubles.
//
// The paper compresses each state chunk on the GPU before it crosses the host link: a chunk is
// cut into segments, one warp per segment; a segment into micro-chunks of 32 doubles, one per
// lane; lane j subtracts double j of the previous micro-chunk and stores the residual as a
// 4-bit prefix (sign + count of leading zero bytes) plus the remaining bytes. The
// byte format (readings G1-G5; oracle/gfc.py is the independent reference):
//   residual = w - prev (64-bit patterns, mod 2^64), prev = 0 for a segment's first micro-chunk;
//   nibble = sign << 3 | min(7, leading zero bytes of |residual|), then 8 - count low bytes;
//   micro-chunk = ceil(cnt/2) nibble bytes (value i in byte i/2, low nibble for even i),
//   then the payloads in value order; a segment stream is zero-padded to 16 bytes.
//
// B200 mapping: persistent grid of 148 x 8 CTAs, 8 warps each, one warp per segment at a time.
// Compression is two passes over the input (sizes, then encode straight into the final,
// 16-byte aligned position after a device scan of the sizes), so no worst-case staging copy is
// needed. Each warp stages its stream in a 1 KB shared-memory ring and writes 512-byte blocks
// (32 lanes x 16 B, coalesced); decompression reads the stream through the same ring and writes
// each micro-chunk as one coalesced 256-byte store. Inputs are read 4 micro-chunks ahead
// (1 KB in flight per warp) to keep enough bytes in flight for HBM.
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"

namespace qgpu {
namespace {

constexpr int kWarps = 8;       // warps per CTA
constexpr int kRing = 1024;     // staging ring per warp (bytes)
constexpr int kBlock = 512;     // ring <-> global transfer unit (32 lanes x 16 B)
constexpr int kAhead = 4;       // micro-chunks loaded ahead
constexpr unsigned kFull = 0xffffffffu;

struct Code {
  uint32_t nib;   // sign << 3 | leading zero bytes (capped at 7)
  int nb;         // payload bytes
  uint64_t mag;   // |residual|
};

__device__ __forceinline__ Code encode_value(uint64_t w, uint64_t prev) {
  const uint64_t r = w - prev;
  const bool neg = static_cast<int64_t>(r) < 0;
  Code c;
  c.mag = neg ? (0ull - r) : r;
  const int lzb = min(__clzll(static_cast<long long>(c.mag)) >> 3, 7);
  c.nb = 8 - lzb;
  c.nib = (neg ? 8u : 0u) | uint32_t(lzb);
  return c;
}

__device__ __forceinline__ int warp_incl_scan(int v, int lane) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int u = __shfl_up_sync(kFull, v, d);
    if (lane >= d) v += u;
  }
  return v;
}

__device__ __forceinline__ uint64_t seg_count(uint64_t n, uint32_t seg, uint64_t s) {
  const uint64_t b = s * seg;
  return (n - b < seg) ? n - b : seg;
}

// Pass 1: padded stream size of every segment -> sizes[s] (offsets[s + 1] before the scan).
__global__ void __launch_bounds__(kWarps * 32) gfc_size_kernel(const uint64_t* __restrict__ in, uint64_t n,
                                                               uint32_t seg, uint64_t nseg,
                                                               uint64_t* __restrict__ sizes) {
  const int lane = threadIdx.x & 31;
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t s = gw; s < nseg; s += nw) {
    const uint64_t cnt = seg_count(n, seg, s);
    const uint64_t* p = in + s * seg;
    uint64_t prev = 0, bytes = 0;
    for (uint64_t k = 0; k < cnt; k += 32 * kAhead) {
      uint64_t w[kAhead];
#pragma unroll
      for (int a = 0; a < kAhead; ++a) {
        const uint64_t i = k + uint64_t(a) * 32 + lane;
        w[a] = i < cnt ? __ldcs(reinterpret_cast<const unsigned long long*>(p + i)) : 0ull;
      }
#pragma unroll
      for (int a = 0; a < kAhead; ++a) {
        const uint64_t k0 = k + uint64_t(a) * 32;
        if (k0 >= cnt) break;
        const int c = int(cnt - k0 < 32 ? cnt - k0 : 32);
        const int nb = lane < c ? encode_value(w[a], prev).nb : 0;
        bytes += uint64_t((c + 1) / 2) + uint64_t(__reduce_add_sync(kFull, unsigned(nb)));
        prev = w[a];
      }
    }
    if (lane == 0) sizes[s] = (bytes + 15) & ~15ull;
  }
}

// Pass 2: encode each segment at its offset (byte stores into the ring: measured faster than
// 64-bit shared atomics, which serialise when many 1-byte payloads share a word).
__global__ void __launch_bounds__(kWarps * 32) gfc_encode_kernel(const uint64_t* __restrict__ in, uint64_t n,
                                                                 uint32_t seg, uint64_t nseg,
                                                                 const uint64_t* __restrict__ offsets,
                                                                 unsigned char* __restrict__ out) {
  __shared__ __align__(16) unsigned char rings[kWarps][kRing];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  unsigned char* ring = rings[wid];
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t s = gw; s < nseg; s += nw) {
    const uint64_t cnt = seg_count(n, seg, s);
    const uint64_t* p = in + s * seg;
    unsigned char* dst = out + offsets[s];
    uint64_t prev = 0, pos = 0, flushed = 0;
    for (uint64_t k = 0; k < cnt; k += 32 * kAhead) {
      uint64_t w[kAhead];
#pragma unroll
      for (int a = 0; a < kAhead; ++a) {
        const uint64_t i = k + uint64_t(a) * 32 + lane;
        w[a] = i < cnt ? __ldcs(reinterpret_cast<const unsigned long long*>(p + i)) : 0ull;
      }
#pragma unroll
      for (int a = 0; a < kAhead; ++a) {
        const uint64_t k0 = k + uint64_t(a) * 32;
        if (k0 >= cnt) break;
        const int c = int(cnt - k0 < 32 ? cnt - k0 : 32);
        const bool valid = lane < c;
        Code cd = encode_value(w[a], prev);
        if (!valid) cd.nb = 0, cd.nib = 0;
        const int npre = (c + 1) / 2;
        const uint32_t hi = __shfl_down_sync(kFull, cd.nib, 1);
        if (!(lane & 1) && valid) ring[(pos + uint64_t(lane >> 1)) % kRing] = uint8_t(cd.nib | (hi << 4));
        const int incl = warp_incl_scan(cd.nb, lane);
        const int total = __shfl_sync(kFull, incl, 31);
        const uint64_t q = pos + uint64_t(npre) + uint64_t(incl - cd.nb);
        for (int b = 0; b < cd.nb; ++b) ring[(q + uint64_t(b)) % kRing] = uint8_t(cd.mag >> (8 * b));
        pos += uint64_t(npre + total);
        prev = w[a];
        __syncwarp();
        while (pos - flushed >= uint64_t(kBlock)) {
          const int4 v = reinterpret_cast<const int4*>(ring + flushed % kRing)[lane];
          __stcs(reinterpret_cast<int4*>(dst + flushed) + lane, v);
          flushed += kBlock;
        }
        __syncwarp();
      }
    }
    const uint64_t padded = (pos + 15) & ~15ull;
    if (uint64_t(lane) < padded - pos) ring[(pos + uint64_t(lane)) % kRing] = 0;
    __syncwarp();
    const uint64_t rem = (padded - flushed) / 16;  // <= 32 + 1 blocks of 16 B
    for (uint64_t j = lane; j < rem; j += 32)
      __stcs(reinterpret_cast<int4*>(dst + flushed) + j,
             reinterpret_cast<const int4*>(ring + (flushed + 16 * j) % kRing)[0]);
    __syncwarp();
  }
}

// Decode: the stream is staged in the ring in 512-byte blocks; a lane reads its nibble and its
// payload as two aligned 64-bit words and a funnel shift.
__global__ void __launch_bounds__(kWarps * 32) gfc_decode_kernel(const unsigned char* __restrict__ in,
                                                                 const uint64_t* __restrict__ offsets, uint64_t n,
                                                                 uint32_t seg, uint64_t nseg,
                                                                 uint64_t* __restrict__ out) {
  constexpr uint32_t kW = kRing / 8;
  __shared__ __align__(16) unsigned long long rings[kWarps][kW];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  unsigned long long* ring = rings[wid];
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  constexpr uint64_t kMaxChunk = 16 + 32 * 8;
  for (uint64_t s = gw; s < nseg; s += nw) {
    const uint64_t cnt = seg_count(n, seg, s);
    uint64_t* dst = out + s * seg;
    const unsigned char* src = in + offsets[s];
    const uint64_t sbytes = offsets[s + 1] - offsets[s];
    uint64_t prev = 0, pos = 0, loaded = 0;
    for (uint64_t k = 0; k < cnt; k += 32) {
      while (loaded < sbytes && loaded - pos < kMaxChunk) {
        const uint64_t off = loaded + 16 * uint64_t(lane);
        if (off < sbytes)
          reinterpret_cast<int4*>(ring)[(off % kRing) / 16] = __ldcs(reinterpret_cast<const int4*>(src + off));
        loaded += kBlock;
        __syncwarp();
      }
      const int c = int(cnt - k < 32 ? cnt - k : 32);
      const bool valid = lane < c;
      const int npre = (c + 1) / 2;
      uint32_t nib = 0;
      if (valid) {
        const uint64_t bp = pos + uint64_t(lane >> 1);
        nib = uint32_t(ring[(bp >> 3) % kW] >> (8 * (bp & 7) + 4 * (lane & 1))) & 15u;
      }
      const int nb = valid ? 8 - int(nib & 7u) : 0;
      const int incl = warp_incl_scan(nb, lane);
      const int total = __shfl_sync(kFull, incl, 31);
      uint64_t mag = 0;
      if (nb) {
        const uint64_t q = pos + uint64_t(npre) + uint64_t(incl - nb);
        const uint32_t wi = uint32_t(q >> 3) % kW, sh = uint32_t(q & 7) * 8;
        uint64_t v = ring[wi] >> sh;
        if (sh) v |= uint64_t(ring[(wi + 1) % kW]) << (64 - sh);
        mag = nb == 8 ? v : (v & ((1ull << (8 * nb)) - 1));
      }
      const uint64_t w = prev + ((nib & 8u) ? (0ull - mag) : mag);
      if (valid) __stcs(reinterpret_cast<unsigned long long*>(dst + k + uint64_t(lane)), (unsigned long long)w);
      prev = w;
      pos += uint64_t(npre + total);
      __syncwarp();
    }
  }
}

// In-place inclusive scan of a[0..n) (uint64), three kernels: block scans, scan of the block
// totals (one CTA, carried across rounds), add-back.
constexpr int kScanT = 1024, kScanE = 4;  // threads, elements per thread

__device__ __forceinline__ uint64_t block_incl_scan(uint64_t v, uint64_t* sh) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint64_t u = __shfl_up_sync(kFull, v, d);
    if (lane >= d) v += u;
  }
  if (lane == 31) sh[w] = v;
  __syncthreads();
  if (w == 0) {
    uint64_t t = lane < int(blockDim.x >> 5) ? sh[lane] : 0;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint64_t u = __shfl_up_sync(kFull, t, d);
      if (lane >= d) t += u;
    }
    sh[lane] = t;
  }
  __syncthreads();
  const uint64_t r = v + (w > 0 ? sh[w - 1] : 0);
  __syncthreads();
  return r;
}

__global__ void __launch_bounds__(kScanT) scan_blocks_kernel(uint64_t* a, uint64_t n, uint64_t* totals) {
  __shared__ uint64_t sh[32];
  const uint64_t base = uint64_t(blockIdx.x) * kScanT * kScanE + uint64_t(threadIdx.x) * kScanE;
  uint64_t v[kScanE], run = 0;
#pragma unroll
  for (int e = 0; e < kScanE; ++e) {
    v[e] = base + e < n ? a[base + e] : 0;
    run += v[e];
    v[e] = run;
  }
  const uint64_t incl = block_incl_scan(run, sh);
  const uint64_t excl = incl - run;
#pragma unroll
  for (int e = 0; e < kScanE; ++e)
    if (base + e < n) a[base + e] = v[e] + excl;
  if (threadIdx.x == kScanT - 1) totals[blockIdx.x] = incl;
}

__global__ void __launch_bounds__(kScanT) scan_totals_kernel(uint64_t* t, uint64_t nb) {
  // exclusive scan of the block totals, in rounds of kScanT carried by `carry`
  __shared__ uint64_t sh[32];
  __shared__ uint64_t round_total;
  uint64_t carry = 0;
  for (uint64_t b0 = 0; b0 < nb; b0 += kScanT) {
    const uint64_t i = b0 + threadIdx.x;
    const uint64_t v = i < nb ? t[i] : 0;
    const uint64_t incl = block_incl_scan(v, sh);
    if (i < nb) t[i] = incl - v + carry;
    if (threadIdx.x == kScanT - 1) round_total = incl;
    __syncthreads();
    carry += round_total;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(kScanT) scan_add_kernel(uint64_t* a, uint64_t n, const uint64_t* totals) {
  const uint64_t add = totals[blockIdx.x];
  const uint64_t base = uint64_t(blockIdx.x) * kScanT * kScanE + uint64_t(threadIdx.x) * kScanE;
#pragma unroll
  for (int e = 0; e < kScanE; ++e)
    if (base + e < n) a[base + e] += add;
}

unsigned gfc_grid(uint64_t nseg) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t want = (nseg + kWarps - 1) / kWarps;
  return unsigned(want < uint64_t(sms) * 8 ? want : uint64_t(sms) * 8);
}

}  // namespace

uint64_t gfc_scan_scratch_elems(uint64_t n) {
  const uint64_t per = uint64_t(kScanT) * kScanE;
  return (n + per - 1) / per;
}

cudaError_t launch_scan_u64(cudaStream_t st, uint64_t* a, uint64_t n, uint64_t* scratch) {
  if (n == 0) return cudaSuccess;
  const uint64_t nb = gfc_scan_scratch_elems(n);
  scan_blocks_kernel<<<unsigned(nb), kScanT, 0, st>>>(a, n, scratch);
  if (nb > 1) {
    scan_totals_kernel<<<1, kScanT, 0, st>>>(scratch, nb);
    scan_add_kernel<<<unsigned(nb), kScanT, 0, st>>>(a, n, scratch);
  }
  return cudaGetLastError();
}

cudaError_t launch_gfc_sizes(cudaStream_t st, const double* in, uint64_t n, uint32_t seg, uint64_t* sizes) {
  const uint64_t nseg = (n + seg - 1) / seg;
  if (nseg == 0) return cudaSuccess;
  gfc_size_kernel<<<gfc_grid(nseg), kWarps * 32, 0, st>>>(reinterpret_cast<const uint64_t*>(in), n, seg, nseg,
                                                          sizes);
  return cudaGetLastError();
}

cudaError_t launch_gfc_encode(cudaStream_t st, const double* in, uint64_t n, uint32_t seg, const uint64_t* offsets,
                              void* out) {
  const uint64_t nseg = (n + seg - 1) / seg;
  if (nseg == 0) return cudaSuccess;
  gfc_encode_kernel<<<gfc_grid(nseg), kWarps * 32, 0, st>>>(reinterpret_cast<const uint64_t*>(in), n, seg, nseg,
                                                            offsets, static_cast<unsigned char*>(out));
  return cudaGetLastError();
}

cudaError_t launch_gfc_decode(cudaStream_t st, const void* in, const uint64_t* offsets, uint64_t n, uint32_t seg,
                              double* out) {
  const uint64_t nseg = (n + seg - 1) / seg;
  if (nseg == 0) return cudaSuccess;
  gfc_decode_kernel<<<gfc_grid(nseg), kWarps * 32, 0, st>>>(static_cast<const unsigned char*>(in), offsets, n, seg,
                                                            nseg, reinterpret_cast<uint64_t*>(out));
  return cudaGetLastError();
}

}  // namespace qgpu
