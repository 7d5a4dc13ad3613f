// sm_100a kernels of the Q-GPU hot path. All state traffic is complex128
// (16 B per amplitude) moved as 128-bit double2 accesses; the live prefix
// [0, 2^k) is the only part of the buffer a pass reads (pruning) and amplitudes in
// [L_in, L_out) are produced from implicit zeros (first-touch expansion, a5).
//
//   pair_kernel   a6  1-qubit U (+controls) on (i, i | 2^t), t >= 5: two coalesced streams
//   pair_shfl     a6  1-qubit U with t < 5: each lane owns one amplitude, partner by shuffle
//   quad_kernel   a7  2-qubit U (+controls) on {i, i|2^t0, i|2^t1, i|2^t0|2^t1}
//   phase_kernel  a8  diagonal gate: touches only amplitudes whose entry differs from 1
//   tile_kernel   a9  fused pass: 2^b amplitudes per tile staged in shared memory, every op
//                     of the pass applied, one HBM read + one HBM write per amplitude
//   gather/probs  a11 readout
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>

#include "kernels.h"

namespace qgpu {

namespace {

__device__ __forceinline__ double2 ld_stream(const double2* p) { return __ldcs(p); }

constexpr int kThreads = 256;

}  // namespace

// ------------------------------------------------------------------------------ a6 pair
template <int PPT>
__global__ void __launch_bounds__(kThreads) pair_kernel(PairArgs a) {
  const uint64_t stride = uint64_t(gridDim.x) * kThreads * PPT;
  const double2 u00 = a.u[0], u01 = a.u[1], u10 = a.u[2], u11 = a.u[3];
  const uint64_t tb = 1ull << a.t;
  for (uint64_t p0 = uint64_t(blockIdx.x) * kThreads * PPT + threadIdx.x; p0 < a.npairs;
       p0 += stride) {
    double2 x0[PPT], x1[PPT];
    uint64_t i0[PPT];
#pragma unroll
    for (int r = 0; r < PPT; ++r) {
      const uint64_t p = p0 + uint64_t(r) * kThreads;
      i0[r] = deposit(p, a.ins, a.nins) | a.cset;
      const bool ok = p < a.npairs;
      x0[r] = (ok && i0[r] < a.L_in) ? ld_stream(a.psi + i0[r]) : make_double2(0, 0);
      x1[r] = (ok && (i0[r] | tb) < a.L_in) ? ld_stream(a.psi + (i0[r] | tb)) : make_double2(0, 0);
    }
#pragma unroll
    for (int r = 0; r < PPT; ++r) {
      const uint64_t p = p0 + uint64_t(r) * kThreads;
      if (p >= a.npairs) break;
      const double2 y0 = cfma(u00, x0[r], cmul(u01, x1[r]));
      const double2 y1 = cfma(u10, x0[r], cmul(u11, x1[r]));
      st_stream(a.psi + i0[r], y0);
      st_stream(a.psi + (i0[r] | tb), y1);
    }
  }
}

// t < 5 and every local control >= 5: 32 consecutive amplitudes per warp, partner in lane ^ 2^t
template <int APT>
__global__ void __launch_bounds__(kThreads) pair_shfl_kernel(PairArgs a) {
  const uint64_t namps = a.npairs * 2;  // amplitudes enumerated (controls fixed to 1)
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (uint64_t(blockIdx.x) * kThreads + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * kThreads) >> 5;
  const int tm = 1 << a.t;
  const bool hi = (lane & tm) != 0;
  // out = c0 * a0 + c1 * a1 with a0/a1 the amplitudes with target bit 0/1, evaluated in the
  // same order as pair_kernel (so both paths round identically)
  const double2 c0 = hi ? a.u[2] : a.u[0];
  const double2 c1 = hi ? a.u[3] : a.u[1];
  for (uint64_t w0 = warp * APT; w0 * 32 < namps; w0 += nwarps * APT) {
    double2 x[APT];
    uint64_t idx[APT];
#pragma unroll
    for (int r = 0; r < APT; ++r) {
      const uint64_t aidx = (w0 + r) * 32 + lane;
      idx[r] = deposit(aidx, a.ins_c, a.nins_c) | a.cset;
      x[r] = (aidx < namps && idx[r] < a.L_in) ? ld_stream(a.psi + idx[r]) : make_double2(0, 0);
    }
#pragma unroll
    for (int r = 0; r < APT; ++r) {
      double2 pv;
      pv.x = __shfl_xor_sync(0xffffffffu, x[r].x, tm);
      pv.y = __shfl_xor_sync(0xffffffffu, x[r].y, tm);
      const uint64_t aidx = (w0 + r) * 32 + lane;
      const double2 a0 = hi ? pv : x[r], a1 = hi ? x[r] : pv;
      if (aidx < namps) st_stream(a.psi + idx[r], cfma(c0, a0, cmul(c1, a1)));
    }
  }
}

// ------------------------------------------------------------------------------ a7 quad
template <int QPT>
__global__ void __launch_bounds__(kThreads) quad_kernel(QuadArgs a) {
  const uint64_t stride = uint64_t(gridDim.x) * kThreads * QPT;
  const uint64_t o1 = 1ull << a.t0, o2 = 1ull << a.t1;
  for (uint64_t q0 = uint64_t(blockIdx.x) * kThreads * QPT + threadIdx.x; q0 < a.nquads;
       q0 += stride) {
    double2 x[QPT][4];
    uint64_t base[QPT];
#pragma unroll
    for (int r = 0; r < QPT; ++r) {
      const uint64_t q = q0 + uint64_t(r) * kThreads;
      base[r] = deposit(q, a.ins, a.nins) | a.cset;
      const bool ok = q < a.nquads;
      const uint64_t off[4] = {0, o1, o2, o1 | o2};
#pragma unroll
      for (int v = 0; v < 4; ++v) {
        const uint64_t i = base[r] | off[v];
        x[r][v] = (ok && i < a.L_in) ? ld_stream(a.psi + i) : make_double2(0, 0);
      }
    }
#pragma unroll
    for (int r = 0; r < QPT; ++r) {
      const uint64_t q = q0 + uint64_t(r) * kThreads;
      if (q >= a.nquads) break;
      const uint64_t off[4] = {0, o1, o2, o1 | o2};
#pragma unroll
      for (int row = 0; row < 4; ++row) {
        double2 y = cmul(a.u[row * 4 + 0], x[r][0]);
        y = cfma(a.u[row * 4 + 1], x[r][1], y);
        y = cfma(a.u[row * 4 + 2], x[r][2], y);
        y = cfma(a.u[row * 4 + 3], x[r][3], y);
        st_stream(a.psi + (base[r] | off[row]), y);
      }
    }
  }
}

// ----------------------------------------------------------------------------- a8 phase
// Single-term form (one diagonal entry != 1): psi[i] *= phase for every i with
// (i & mask) == match -- enumerated directly, so CZ/CP touch 1/4 of the live amplitudes.
// Multi-term form: every amplitude with the controls set, times d[target bits].
template <int APT>
__global__ void __launch_bounds__(kThreads) phase_kernel(PhaseArgs a) {
  const uint64_t stride = uint64_t(gridDim.x) * kThreads * APT;
  for (uint64_t v0 = uint64_t(blockIdx.x) * kThreads * APT + threadIdx.x; v0 < a.count;
       v0 += stride) {
    double2 x[APT];
    uint64_t idx[APT];
#pragma unroll
    for (int r = 0; r < APT; ++r) {
      const uint64_t v = v0 + uint64_t(r) * kThreads;
      idx[r] = deposit(v, a.ins, a.nins) | a.fixed;
      x[r] = (v < a.count) ? ld_stream(a.psi + idx[r]) : make_double2(0, 0);
    }
#pragma unroll
    for (int r = 0; r < APT; ++r) {
      const uint64_t v = v0 + uint64_t(r) * kThreads;
      if (v >= a.count) break;
      int sel = 0;
      if (a.nt >= 1) sel |= int(idx[r] >> a.t0 & 1);
      if (a.nt >= 2) sel |= int(idx[r] >> a.t1 & 1) << 1;
      st_stream(a.psi + idx[r], cmul(x[r], a.d[sel]));
    }
  }
}

// ------------------------------------------------------------------------------ a9 tile
// The generic (interpreted) fused-pass kernel: the pass program is walked op by op. The
// persistent tile loop, loads, constants and store are tile_driver (tile_common.cuh); the JIT
// path (jit.cpp) replaces this body by straight-line code specialised to one pass.
template <int NR>
struct InterpBody {
  static constexpr unsigned kZM0 = 0u;
  static constexpr uint32_t kZW0 = 0u;
  static constexpr bool kStatic = false;  // mappings read from the program at run time
  static constexpr bool kHasScalar = true;
  static constexpr uint32_t kJ0[kRegAmps] = {};
  static constexpr uint64_t kP0[kRegAmps] = {};
  static constexpr uint64_t kPF[kRegAmps] = {};
  int nops;
  __device__ __forceinline__ void operator()(double2 (&v)[kRegAmps], Mapping& mp, const TileCtx& c) const {
    for (int i = 1; i < nops; ++i) {
      const TileOp& op = c.ops[i];
      switch (op.kind) {
        case OP_RUN:
          op_run<NR>(v, op, c, mp, op.a0, op.a1, op.cls, int(op.tmask), int(op.tmatch));
          break;
        case OP_U1R: {
          if (!op_active(op, c.gbase) || (mp.base & op.tmask) != op.tmatch) break;
          const double2* u = c.pool + op.moff;
          switch (op.a0 * 4 + op.cls) {
#define QGPU_U1R(K, CL) \
  case K * 4 + CL: op_u1r<NR, K, CL>(v, u, op.rmask, op.rmatch); break;
            QGPU_U1R(0, 0) QGPU_U1R(0, 1) QGPU_U1R(0, 2) QGPU_U1R(0, 3) QGPU_U1R(1, 0) QGPU_U1R(1, 1)
            QGPU_U1R(1, 2) QGPU_U1R(1, 3) QGPU_U1R(2, 0) QGPU_U1R(2, 1) QGPU_U1R(2, 2) QGPU_U1R(2, 3)
            QGPU_U1R(3, 0) QGPU_U1R(3, 1) QGPU_U1R(3, 2) QGPU_U1R(3, 3)
#undef QGPU_U1R
            default: break;
          }
          break;
        }
        case OP_U1L: {
          if (!op_active(op, c.gbase)) break;
          const bool tc = (mp.base & op.tmask) == op.tmatch;
          const double2* u = c.pool + op.moff;
          if (op.cls == MAT_X) op_u1l<NR, MAT_X>(v, u, op.a0, c.lane, tc, op.rmask, op.rmatch);
          else if (op.cls == MAT_RI) op_u1l<NR, MAT_RI>(v, u, op.a0, c.lane, tc, op.rmask, op.rmatch);
          else if (op.cls == MAT_REAL) op_u1l<NR, MAT_REAL>(v, u, op.a0, c.lane, tc, op.rmask, op.rmatch);
          else op_u1l<NR, MAT_GENERIC>(v, u, op.a0, c.lane, tc, op.rmask, op.rmatch);
          break;
        }
        case OP_U2R: {
          if (!op_active(op, c.gbase) || (mp.base & op.tmask) != op.tmatch) break;
          const double2* u = c.pool + op.moff;
          switch (op.a0 * 4 + op.a1) {
#define QGPU_U2R(A, B) \
  case A * 4 + B: op_u2r<NR, A, B>(v, u, op.rmask, op.rmatch); break;
            QGPU_U2R(0, 1) QGPU_U2R(0, 2) QGPU_U2R(0, 3) QGPU_U2R(1, 0) QGPU_U2R(1, 2) QGPU_U2R(1, 3)
            QGPU_U2R(2, 0) QGPU_U2R(2, 1) QGPU_U2R(2, 3) QGPU_U2R(3, 0) QGPU_U2R(3, 1) QGPU_U2R(3, 2)
#undef QGPU_U2R
            default: break;
          }
          break;
        }
        case OP_REMAP:
          tile_spill<NR>(v, c, mp);
          mp = make_mapping<NR>(op, c.nw, c.lane, c.warp);
          tile_reload<NR>(v, c, mp);
          break;
        default: {  // OP_SMEM1 / OP_SMEM2 (tile-uniform condition is uniform: barriers are safe)
          if (!op_active(op, c.gbase)) break;
          tile_spill<NR>(v, c, mp);
          if (op.kind == OP_SMEM2) op_smem2(c, op);
          else if (op.cls == MAT_X) op_smem1<MAT_X>(c, op);
          else if (op.cls == MAT_RI) op_smem1<MAT_RI>(c, op);
          else if (op.cls == MAT_REAL) op_smem1<MAT_REAL>(c, op);
          else op_smem1<MAT_GENERIC>(c, op);
          tile_reload<NR>(v, c, mp);
          break;
        }
      }
    }
  }
};

template <int NR>
__global__ void __launch_bounds__(NR >= 4 ? 256 : 512, 1) tile_kernel(TileArgs a) {
  InterpBody<NR> body{a.nops};
  tile_driver<NR>(a, body);
}

// ------------------------------------------------------------------------------ a11
__global__ void gather_kernel(GatherArgs a) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t x = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; x < a.count; x += stride) {
    const uint64_t X = a.start + x;
    double2 v = make_double2(0, 0);
    if ((X & a.unassigned) == 0) {
      uint64_t phys = 0;
      for (int q = 0; q < a.n; ++q)
        if (X >> q & 1) phys |= 1ull << a.pos[q];
      if ((phys >> a.m) == a.rank) {
        if ((phys & ((1ull << a.m) - 1)) < a.L) v = a.psi[phys & ((1ull << a.m) - 1)];
      } else if (a.only_owned) {
        continue;
      }
    } else if (a.only_owned) {
      continue;
    }
    a.out[x] = v;
  }
}

// per-CTA buckets in shared memory (2^m <= 4096), partial sums per CTA, then a fixed-order
// second pass (deterministic given the grid).
__global__ void __launch_bounds__(kThreads) probs_block_kernel(ProbArgs a) {
  extern __shared__ double hist[];
  const uint32_t B = 1u << a.m;
  for (uint32_t y = threadIdx.x; y < B; y += blockDim.x) hist[y] = 0.0;
  __syncthreads();
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < a.L; i += stride) {
    const double2 v = a.psi[i];
    uint32_t y = uint32_t(a.yfixed);
    for (int j = 0; j < a.m; ++j) y |= uint32_t((i >> a.ppos[j]) & 1) << j;
    atomicAdd(&hist[y], v.x * v.x + v.y * v.y);
  }
  __syncthreads();
  for (uint32_t y = threadIdx.x; y < B; y += blockDim.x) a.partial[uint64_t(blockIdx.x) * B + y] = hist[y];
}

__global__ void probs_reduce_kernel(const double* partial, int nblk, uint32_t B, double* out) {
  for (uint32_t y = blockIdx.x * blockDim.x + threadIdx.x; y < B; y += gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int k = 0; k < nblk; ++k) s += partial[uint64_t(k) * B + y];
    out[y] = s;
  }
}

__global__ void probs_global_kernel(ProbArgs a) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < a.L; i += stride) {
    const double2 v = a.psi[i];
    uint64_t y = a.yfixed;
    for (int j = 0; j < a.m; ++j) y |= ((i >> a.ppos[j]) & 1) << j;
    atomicAdd(&a.out[y], v.x * v.x + v.y * v.y);
  }
}

__global__ void set_amp_kernel(double2* psi, uint64_t i, double2 v) { psi[i] = v; }

// a10 (virtual ranks): exchange the lp=1 half of shard a with the lp=0 half of shard b
__global__ void swap_halves_kernel(double2* a, double2* b, int lp, uint64_t half) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t t = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < half; t += stride) {
    const uint64_t i0 = insert0(t, lp);
    const uint64_t ia = i0 | (1ull << lp);
    const double2 x = __ldcs(a + ia), y = __ldcs(b + i0);
    __stcs(a + ia, y);
    __stcs(b + i0, x);
  }
}
// a10 (NCCL): gather / scatter slab [t0, t0+count) of the half with local bit lp == bit
__global__ void pack_half_kernel(const double2* psi, double2* buf, int lp, int bit, uint64_t t0, uint64_t count) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t t = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < count; t += stride)
    buf[t] = __ldcs(psi + (insert0(t0 + t, lp) | (uint64_t(bit) << lp)));
}
__global__ void unpack_half_kernel(double2* psi, const double2* buf, int lp, int bit, uint64_t t0, uint64_t count) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t t = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < count; t += stride)
    __stcs(psi + (insert0(t0 + t, lp) | (uint64_t(bit) << lp)), buf[t]);
}
__global__ void add_kernel(double* out, const double* in, uint64_t count) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t t = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < count; t += stride) out[t] += in[t];
}

// --------------------------------------------------------------------------- launchers
namespace {
int g_num_sms = 0;
int num_sms() {
  if (!g_num_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_num_sms <= 0) g_num_sms = 148;
  }
  return g_num_sms;
}
unsigned grid_for(uint64_t work_items, int per_block, int blocks_per_sm) {
  const uint64_t need = (work_items + per_block - 1) / per_block;
  const uint64_t cap = uint64_t(num_sms()) * blocks_per_sm;
  return unsigned(std::max<uint64_t>(1, std::min(need, cap)));
}
}  // namespace

int device_num_sms() { return num_sms(); }

size_t tile_smem_bytes(const TileArgs& a) {
  const size_t nh = size_t(1) << (a.b - a.l);
  const size_t nwarps = size_t(1) << a.nw;
  return size_t(a.nbuf) * (size_t(1) << a.b) * 16 + ((nh + 1) & ~size_t(1)) * 8 + size_t(a.blob_bytes) +
         nwarps * size_t(a.npat) * 16 + 16;
}

cudaError_t launch_pair(cudaStream_t st, const PairArgs& a, bool shfl) {
  if (a.npairs == 0) return cudaSuccess;
  if (shfl) {
    constexpr int APT = 4;
    const unsigned g = grid_for(a.npairs * 2, kThreads * APT, 8);
    pair_shfl_kernel<APT><<<g, kThreads, 0, st>>>(a);
  } else {
    constexpr int PPT = 2;
    const unsigned g = grid_for(a.npairs, kThreads * PPT, 8);
    pair_kernel<PPT><<<g, kThreads, 0, st>>>(a);
  }
  return cudaGetLastError();
}

cudaError_t launch_quad(cudaStream_t st, const QuadArgs& a) {
  if (a.nquads == 0) return cudaSuccess;
  constexpr int QPT = 1;
  const unsigned g = grid_for(a.nquads, kThreads * QPT, 8);
  quad_kernel<QPT><<<g, kThreads, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_phase(cudaStream_t st, const PhaseArgs& a) {
  if (a.count == 0) return cudaSuccess;
  constexpr int APT = 4;
  const unsigned g = grid_for(a.count, kThreads * APT, 8);
  phase_kernel<APT><<<g, kThreads, 0, st>>>(a);
  return cudaGetLastError();
}

template <int NR>
cudaError_t launch_tile_nr(cudaStream_t st, const TileArgs& a, size_t smem) {
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(tile_kernel<NR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         227 * 1024);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  const int threads = 32 << a.nw;
  int bps = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, tile_kernel<NR>, threads, smem);
  if (bps <= 0) bps = 1;
  const unsigned g = unsigned(std::min<uint64_t>(a.ntiles, uint64_t(num_sms()) * bps));
  tile_kernel<NR><<<g, threads, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tile(cudaStream_t st, const TileArgs& a) {
  if (a.ntiles == 0) return cudaSuccess;
  const size_t smem = tile_smem_bytes(a);
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  switch (a.nr) {
    case 0: return launch_tile_nr<0>(st, a, smem);
    case 1: return launch_tile_nr<1>(st, a, smem);
    case 2: return launch_tile_nr<2>(st, a, smem);
    case 3: return launch_tile_nr<3>(st, a, smem);
    default: return launch_tile_nr<4>(st, a, smem);
  }
}

cudaError_t launch_gather(cudaStream_t st, const GatherArgs& a) {
  if (a.count == 0) return cudaSuccess;
  const unsigned g = grid_for(a.count, 256, 8);
  gather_kernel<<<g, 256, 0, st>>>(a);
  return cudaGetLastError();
}

// out: device buffer of 2^m doubles; scratch: >= probs_scratch_bytes(m) bytes
size_t probs_scratch_doubles(int m) {
  if (m > 12) return 0;
  return size_t(num_sms()) * 2 * (size_t(1) << m);
}

cudaError_t launch_probs(cudaStream_t st, ProbArgs a, double* scratch) {
  const uint32_t B = 1u << a.m;
  if (a.m <= 12) {
    const unsigned g = unsigned(num_sms()) * 2;
    a.partial = scratch;
    probs_block_kernel<<<g, kThreads, B * sizeof(double), st>>>(a);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    probs_reduce_kernel<<<(B + 255) / 256, 256, 0, st>>>(scratch, int(g), B, a.out);
    return cudaGetLastError();
  }
  cudaError_t e = cudaMemsetAsync(a.out, 0, sizeof(double) * (size_t(1) << a.m), st);
  if (e != cudaSuccess) return e;
  if (a.L == 0) return cudaSuccess;
  const unsigned g = grid_for(a.L, 256, 8);
  probs_global_kernel<<<g, 256, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_swap_halves(cudaStream_t st, double2* a, double2* b, int lp, uint64_t half) {
  swap_halves_kernel<<<grid_for(half, 256 * 4, 8), 256, 0, st>>>(a, b, lp, half);
  return cudaGetLastError();
}
cudaError_t launch_pack_half(cudaStream_t st, const double2* psi, double2* buf, int lp, int bit, uint64_t t0,
                             uint64_t count) {
  pack_half_kernel<<<grid_for(count, 256 * 4, 8), 256, 0, st>>>(psi, buf, lp, bit, t0, count);
  return cudaGetLastError();
}
cudaError_t launch_unpack_half(cudaStream_t st, double2* psi, const double2* buf, int lp, int bit, uint64_t t0,
                               uint64_t count) {
  unpack_half_kernel<<<grid_for(count, 256 * 4, 8), 256, 0, st>>>(psi, buf, lp, bit, t0, count);
  return cudaGetLastError();
}
cudaError_t launch_add(cudaStream_t st, double* out, const double* in, uint64_t count) {
  if (!count) return cudaSuccess;
  add_kernel<<<grid_for(count, 256 * 4, 8), 256, 0, st>>>(out, in, count);
  return cudaGetLastError();
}

cudaError_t launch_set_amp(cudaStream_t st, double2* psi, uint64_t i, double re, double im) {
  set_amp_kernel<<<1, 1, 0, st>>>(psi, i, make_double2(re, im));
  return cudaGetLastError();
}

}  // namespace qgpu
