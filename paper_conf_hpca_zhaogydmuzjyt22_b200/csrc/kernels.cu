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
#include <cstdlib>
#include <bit>
#include <vector>

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

// Single-term diagonal with position 0 fixed (e.g. CP / CZ / CX-type phases on qubit 0): the
// affected amplitudes are every other 16-byte slot, i.e. half of each 32-byte DRAM sector. Each
// thread reads and writes the whole sector (the affected amplitude and its bit-0 partner,
// unchanged), so no sector is written partially (a partial write costs a fill read).
template <int APT>
__global__ void __launch_bounds__(kThreads) phase_sector_kernel(PhaseArgs a) {
  const uint64_t stride = uint64_t(gridDim.x) * kThreads * APT;
  for (uint64_t v0 = uint64_t(blockIdx.x) * kThreads * APT + threadIdx.x; v0 < a.count;
       v0 += stride) {
    double2 x0[APT], x1[APT];
    uint64_t idx[APT];
#pragma unroll
    for (int r = 0; r < APT; ++r) {
      const uint64_t v = v0 + uint64_t(r) * kThreads;
      idx[r] = (deposit(v, a.ins, a.nins) | a.fixed) & ~1ull;
      const bool ok = v < a.count;
      x0[r] = ok ? ld_stream(a.psi + idx[r]) : make_double2(0, 0);
      x1[r] = ok ? ld_stream(a.psi + idx[r] + 1) : make_double2(0, 0);
    }
    const bool odd = a.fixed & 1;
#pragma unroll
    for (int r = 0; r < APT; ++r) {
      const uint64_t v = v0 + uint64_t(r) * kThreads;
      if (v >= a.count) break;
      const uint64_t i = idx[r] | (odd ? 1 : 0);
      int sel = 0;
      if (a.nt >= 1) sel |= int(i >> a.t0 & 1);
      if (a.nt >= 2) sel |= int(i >> a.t1 & 1) << 1;
      if (odd) x1[r] = cmul(x1[r], a.d[sel]);
      else x0[r] = cmul(x0[r], a.d[sel]);
      st_stream(a.psi + idx[r], x0[r]);
      st_stream(a.psi + idx[r] + 1, x1[r]);
    }
  }
}

// ------------------------------------------------------------------------------ a9 tile
// The generic (interpreted) fused-pass kernel: the pass program is walked op by op. The
// persistent tile loop, loads, constants and store are tile_driver (tile_common.cuh); the JIT
// path (jit.cpp) replaces this body by straight-line code specialised to one pass.
template <int NR, bool H>
struct InterpBody {
  static constexpr unsigned kZM0 = 0u;
  static constexpr uint32_t kZW0 = 0u;
  static constexpr bool kStatic = false;  // mappings read from the program at run time
  static constexpr bool kHist = H;        // H: the instantiation launched for a fused measurement
  static constexpr int kHistMode = -1;    // its epilogue too (a.hacc)
  static constexpr bool kHistRS = false;  // mode 2 with run-time masks (a.hlred, a.hrb)
  static constexpr uint32_t kHlred = 0u, kDead = 0u;
  static constexpr bool kHistGlob = false;  // (a.hglob at run time)
  static constexpr int kNsrun = -1;       // tile positions read from the arguments
  static constexpr int kSrunPos[1] = {0};
  static constexpr int kSrunLen[1] = {0};
  static constexpr bool kHasScalar = true;
  static constexpr bool kGroupRemap = false;  // remaps use CTA barriers
  __device__ static void init_mbar(uint64_t*) {}
  static constexpr uint32_t kJ0[kRegAmps] = {};
  static constexpr uint64_t kP0[kRegAmps] = {};
  static constexpr uint64_t kPF[kRegAmps] = {};
  static constexpr uint32_t kJF[kRegAmps] = {};
  int nops;
  static constexpr bool kEarlyPrefetch = false;  // the driver prefetches after the program
  static constexpr bool kScalarFolded = false;   // the driver applies the tile-uniform scalar
  template <class PF>
  __device__ __forceinline__ void operator()(double2 (&v)[kRegAmps], Mapping& mp, const TileCtx& c,
                                             const TileArgs&, PF&&) const {
    for (int i = 1; i < nops; ++i) {
      const TileOp& op = c.ops[i];
      switch (op.kind) {
        case OP_RUN:
          op_run<NR>(v, op, c, mp, op.a0, op.a1, op.cls, int(op.tmask), int(op.tmatch));
          break;
        case OP_U1R: {
          if (!op_active(op, c.gbase) || (mp.base & op.tmask) != op.tmatch) break;
          const double2* u = c.pool + op.moff;
          switch (op.a0 * 8 + op.cls) {
#define QGPU_U1R(K, CL) \
  case K * 8 + CL: op_u1r<NR, K, CL>(v, u, op.rmask, op.rmatch); break;
            QGPU_U1R(0, 0) QGPU_U1R(0, 1) QGPU_U1R(0, 2) QGPU_U1R(0, 3) QGPU_U1R(1, 0) QGPU_U1R(1, 1)
            QGPU_U1R(1, 2) QGPU_U1R(1, 3) QGPU_U1R(2, 0) QGPU_U1R(2, 1) QGPU_U1R(2, 2) QGPU_U1R(2, 3)
            QGPU_U1R(3, 0) QGPU_U1R(3, 1) QGPU_U1R(3, 2) QGPU_U1R(3, 3)
            QGPU_U1R(0, 4) QGPU_U1R(0, 5) QGPU_U1R(0, 6) QGPU_U1R(0, 7) QGPU_U1R(1, 4) QGPU_U1R(1, 5)
            QGPU_U1R(1, 6) QGPU_U1R(1, 7) QGPU_U1R(2, 4) QGPU_U1R(2, 5) QGPU_U1R(2, 6) QGPU_U1R(2, 7)
            QGPU_U1R(3, 4) QGPU_U1R(3, 5) QGPU_U1R(3, 6) QGPU_U1R(3, 7)
#undef QGPU_U1R
            default: break;
          }
          break;
        }
        case OP_U1L: {
          if (!op_active(op, c.gbase)) break;
          const bool tc = (mp.base & op.tmask) == op.tmatch;
          const double2* u = c.pool + op.moff;
          switch (op.cls) {
#define QGPU_U1L(CL) \
  case CL: op_u1l<NR, CL>(v, u, op.a0, c.lane, tc, op.rmask, op.rmatch); break;
            QGPU_U1L(MAT_X) QGPU_U1L(MAT_RI) QGPU_U1L(MAT_REAL) QGPU_U1L(MAT_RU) QGPU_U1L(MAT_RUN)
            QGPU_U1L(MAT_IU) QGPU_U1L(MAT_IUN)
#undef QGPU_U1L
            default: op_u1l<NR, MAT_GENERIC>(v, u, op.a0, c.lane, tc, op.rmask, op.rmatch); break;
          }
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
          else switch (op.cls) {
#define QGPU_SM1(CL) \
  case CL: op_smem1<CL>(c, op); break;
            QGPU_SM1(MAT_X) QGPU_SM1(MAT_RI) QGPU_SM1(MAT_REAL) QGPU_SM1(MAT_RU) QGPU_SM1(MAT_RUN)
            QGPU_SM1(MAT_IU) QGPU_SM1(MAT_IUN)
#undef QGPU_SM1
            default: op_smem1<MAT_GENERIC>(c, op); break;
          }
          tile_reload<NR>(v, c, mp);
          break;
        }
      }
    }
  }
};

template <int NR, bool H>
__global__ void __launch_bounds__(NR >= 4 ? 256 : 512, 1) tile_kernel(TileArgs a) {
  InterpBody<NR, H> body{a.nops};
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

// a11 sharded readout, point to point: ownership of a logical index (kernels.h)
__device__ __forceinline__ bool owned_local(const GatherArgs& a, uint64_t X, uint64_t* local) {
  if (X & a.unassigned) return false;
  uint64_t phys = 0;
  for (int q = 0; q < a.n; ++q)
    if (X >> q & 1) phys |= 1ull << a.pos[q];
  if ((phys >> a.m) != a.rank) return false;
  *local = phys & ((1ull << a.m) - 1);
  return true;
}
__global__ void owner_flags_kernel(GatherArgs a, uint64_t* flags) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t x = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; x < a.count; x += stride) {
    uint64_t loc;
    flags[x] = owned_local(a, a.start + x, &loc) ? 1u : 0u;
  }
}
__global__ void owned_compact_kernel(GatherArgs a, const uint64_t* pos, double2* compact) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t x = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; x < a.count; x += stride) {
    uint64_t loc;
    if (owned_local(a, a.start + x, &loc)) compact[pos[x] - 1] = loc < a.L ? a.psi[loc] : make_double2(0, 0);
  }
}
__global__ void owned_scatter_kernel(GatherArgs a, const uint64_t* pos, const double2* compact) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t x = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; x < a.count; x += stride) {
    uint64_t loc;
    if (owned_local(a, a.start + x, &loc)) a.out[x] = compact[pos[x] - 1];
  }
}

// a11 probabilities. Each warp owns a contiguous range of the live prefix and walks it 32
// amplitudes at a time (lane bits = index bits 0..4). The bucket index splits into a part
// given by requested positions < 5 (per lane) and a part given by positions >= 5 (uniform over
// the warp, changing only every 2^(p-5) steps): |psi|^2 accumulates in a register while the
// uniform part is unchanged; on a change the lanes are reduced over the non-requested lane bits
// (butterfly) and one lane per lane-pattern adds into the histogram (shared memory for
// 2^m <= 4096 buckets, then one atomic per bucket and CTA into the output; global otherwise).
__device__ __forceinline__ void probs_flush(double acc, int lane, uint32_t lowreq, uint32_t ylow, uint64_t hi,
                                            double* hist, bool private_hist) {
  // sum over the lane bits that are not requested
#pragma unroll
  for (int b = 0; b < 5; ++b)
    if (!((lowreq >> b) & 1)) acc += __shfl_xor_sync(0xffffffffu, acc, 1 << b);
  // representatives (lanes whose non-requested bits are 0) hold distinct buckets
  if ((uint32_t(lane) & ~lowreq & 31u) == 0 && acc != 0.0) {
    const uint64_t y = hi | ylow;
    if (private_hist) hist[y] += acc;  // this warp's own histogram: no other writer
    else atomicAdd(&hist[y], acc);
  }
}

// mode 0: per-warp private histograms in shared memory (2^m <= 1024), mode 1: one shared
// histogram per CTA with atomics (2^m <= 4096), mode 2: global atomics. The bucket of an
// index is assembled from five byte tables (bits 8k..8k+7 of the index -> bucket bits).
__global__ void __launch_bounds__(kThreads) probs_kernel(ProbArgs a, int mode) {
  extern __shared__ double shist[];
  __shared__ uint32_t btab[5][256];
  const uint32_t B = 1u << a.m;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5, nwb = blockDim.x >> 5;
  double* hist = mode == 0 ? shist + size_t(wib) * B : (mode == 1 ? shist : a.out);
  for (int e = threadIdx.x; e < 5 * 256; e += blockDim.x) {
    const int k = e >> 8, byte = e & 255;
    uint32_t y = 0;
    for (int j = 0; j < a.m; ++j) {
      const int p = a.ppos[j] - 8 * k;
      if (p >= 0 && p < 8 && ((byte >> p) & 1)) y |= 1u << j;
    }
    btab[k][byte] = y;
  }
  if (mode < 2) {
    const uint32_t tot = mode == 0 ? B * nwb : B;
    for (uint32_t y = threadIdx.x; y < tot; y += blockDim.x) shist[y] = 0.0;
  }
  __syncthreads();
  uint32_t lowreq = 0;
  for (int j = 0; j < a.m; ++j)
    if (a.ppos[j] < 5) lowreq |= 1u << a.ppos[j];
  const uint32_t ylow = btab[0][lane];  // bucket bits from the lane bits (positions 0..4)
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t steps = (a.L + 31) >> 5;
  const uint64_t per = (steps + nwarps - 1) / nwarps;
  const uint64_t s0 = gw * per, s1 = min(steps, s0 + per);
  // requested positions >= 5 (uniform over the warp at each step)
  uint64_t himask = 0;
  for (int j = 0; j < a.m; ++j)
    if (a.ppos[j] >= 5 && a.ppos[j] < 40) himask |= 1ull << a.ppos[j];
  double acc = 0.0;
  uint64_t cur = ~0ull, curbits = ~0ull;
  constexpr int U = 8;  // loads in flight per lane
  for (uint64_t st = s0; st < s1; st += U) {
    double2 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t i = ((st + u) << 5) | uint64_t(lane);
      v[u] = (st + u < s1 && i < a.L) ? __ldcs(a.psi + i) : make_double2(0.0, 0.0);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t bits = ((st + u) << 5) & himask;
      if (bits != curbits) {
        const uint64_t hi = a.yfixed | btab[0][bits & 255] | btab[1][(bits >> 8) & 255] |
                            btab[2][(bits >> 16) & 255] | btab[3][(bits >> 24) & 255] | btab[4][(bits >> 32) & 255];
        if (cur != ~0ull) probs_flush(acc, lane, lowreq, ylow, cur, hist, mode == 0);
        acc = 0.0;
        cur = hi;
        curbits = bits;
      }
      acc = fma(v[u].x, v[u].x, fma(v[u].y, v[u].y, acc));
    }
  }
  if (cur != ~0ull) probs_flush(acc, lane, lowreq, ylow, cur, hist, mode == 0);
  if (mode < 2) {
    __syncthreads();
    for (uint32_t y = threadIdx.x; y < B; y += blockDim.x) {
      double t = 0.0;
      if (mode == 0)
        for (int w = 0; w < nwb; ++w) t += shist[size_t(w) * B + y];
      else
        t = shist[y];
      if (t != 0.0) atomicAdd(&a.out[y], t);
    }
  }
}

// a11 probabilities, mapped form: the index bits are dealt to the thread so that requested
// positions are lane bits (0..4), warp bits or CTA-id bits wherever possible; then a thread's
// bucket is fixed over its whole loop except for the <= 3 requested positions left in the loop
// (the innermost loop bits, one register accumulator each). No histogram, no atomics in the
// loop: every warp reads 512 contiguous bytes per step; at the end the lanes are reduced over the
// non-requested lane bits and one atomic per bucket and warp adds into the output. Needs the
// live range to be a power of two (it always is) and >= 2^5.
struct ProbMap {
  uint64_t fixed;                 // positions < k not enumerated by the loop (lanes, warps, CTAs, e)
  int wbits, cbits, ebits;
  int wpos[4], cpos[16], epos[3];
  int nfrun;                      // runs of fixed (non-loop) positions, ascending
  int frun_pos[40], frun_len[40];
  int obits;                      // loop bits
};

template <int E>
__global__ void __launch_bounds__(512) probs_mapped_kernel(ProbArgs a, ProbMap mp) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t tb = uint64_t(lane);
  for (int k = 0; k < mp.wbits; ++k)
    if ((warp >> k) & 1) tb |= 1ull << mp.wpos[k];
  for (int k = 0; k < mp.cbits; ++k)
    if ((blockIdx.x >> k) & 1) tb |= 1ull << mp.cpos[k];
  auto bucket = [&](uint64_t idx) {
    uint64_t y = a.yfixed;
    for (int j = 0; j < a.m; ++j)
      if (a.ppos[j] < 63 && ((idx >> a.ppos[j]) & 1)) y |= 1ull << j;
    return y;
  };
  constexpr int NE = 1 << E;
  uint64_t eoff[NE];
#pragma unroll
  for (int e = 0; e < NE; ++e) {
    eoff[e] = 0;
    for (int k = 0; k < E; ++k)
      if ((e >> k) & 1) eoff[e] |= 1ull << mp.epos[k];
  }
  double acc[NE];
#pragma unroll
  for (int e = 0; e < NE; ++e) acc[e] = 0.0;
  constexpr int U = NE >= 8 ? 1 : 8 / NE;  // loads in flight per thread: U * NE = 8
  const uint64_t nouter = 1ull << mp.obits;
  // the loop's index bits, enumerated by a masked increment: with every fixed position set, +1
  // carries straight through them to the next loop bit (t_{o+1} = ((t_o | fixed) + 1) & ~fixed)
  const uint64_t fixed = mp.fixed;
  uint64_t tnext = 0;
  for (uint64_t o = 0; o < nouter; o += U) {
    double2 v[U][NE];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t t = tnext;
      tnext = ((tnext | fixed) + 1) & ~fixed;
      const bool ok = o + u < nouter;
#pragma unroll
      for (int e = 0; e < NE; ++e) v[u][e] = ok ? __ldcs(a.psi + (tb | t | eoff[e])) : make_double2(0.0, 0.0);
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int e = 0; e < NE; ++e) acc[e] = fma(v[u][e].x, v[u][e].x, fma(v[u][e].y, v[u][e].y, acc[e]));
  }
  uint32_t lowreq = 0;
  for (int j = 0; j < a.m; ++j)
    if (a.ppos[j] < 5) lowreq |= 1u << a.ppos[j];
#pragma unroll
  for (int e = 0; e < NE; ++e) {
    double x = acc[e];
#pragma unroll
    for (int b = 0; b < 5; ++b)
      if (!((lowreq >> b) & 1)) x += __shfl_xor_sync(0xffffffffu, x, 1 << b);
    if ((uint32_t(lane) & ~lowreq & 31u) == 0 && x != 0.0) atomicAdd(&a.out[bucket(tb | eoff[e])], x);
  }
}

// Deal the live index bits (k = log2 L) to lanes / warps / CTAs / loop for probs_mapped_kernel;
// false if more than 3 requested positions would be left in the loop.
bool plan_probs_map(const ProbArgs& a, int k, ProbMap* mp) {
  if (k < 5) return false;
  std::vector<int> req;
  uint64_t reqmask = 0;
  for (int j = 0; j < a.m; ++j)
    if (a.ppos[j] >= 5 && a.ppos[j] < k) req.push_back(a.ppos[j]), reqmask |= 1ull << a.ppos[j];
  std::sort(req.begin(), req.end());
  std::vector<int> other;  // non-requested positions >= 5, highest first
  for (int p = k - 1; p >= 5; --p)
    if (!((reqmask >> p) & 1)) other.push_back(p);
  size_t ri = 0, oi = 0;
  uint64_t fixed = 31;
  *mp = ProbMap{};
  mp->wbits = std::min(4, k - 5);
  for (int i = 0; i < mp->wbits; ++i) {
    const int p = ri < req.size() ? req[ri++] : other[oi++];
    mp->wpos[i] = p;
    fixed |= 1ull << p;
  }
  mp->cbits = std::min(10, k - 5 - mp->wbits);
  for (int i = 0; i < mp->cbits; ++i) {
    const int p = ri < req.size() ? req[ri++] : other[oi++];
    mp->cpos[i] = p;
    fixed |= 1ull << p;
  }
  mp->ebits = int(req.size() - ri);
  if (mp->ebits > 3) return false;
  for (int i = 0; i < mp->ebits; ++i) {
    mp->epos[i] = req[ri + i];
    fixed |= 1ull << mp->epos[i];
  }
  mp->obits = k - 5 - mp->wbits - mp->cbits - mp->ebits;
  mp->fixed = fixed;
  mp->nfrun = 0;
  for (int p = 0; p < k;) {
    if (!((fixed >> p) & 1)) {
      ++p;
      continue;
    }
    int q = p;
    while (q + 1 < k && ((fixed >> (q + 1)) & 1)) ++q;
    mp->frun_pos[mp->nfrun] = p;
    mp->frun_len[mp->nfrun] = q - p + 1;
    mp->nfrun++;
    p = q + 1;
  }
  return true;
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
// a10 batched swap: gather / scatter one slab of every exchanged block (kernels.h BlockArgs).
// blockIdx.y = block; x grid-strides over the slab's rest indices, so with swapped positions >= 5
// every warp moves >= 512 contiguous bytes.
__global__ void pack_blocks_kernel(BlockArgs a) {
  const uint64_t pat = a.pat[blockIdx.y];
  double2* out = a.buf + uint64_t(blockIdx.y) * a.cnt;
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t t = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < a.cnt; t += stride)
    out[t] = __ldcs(a.psi + (deposit(a.t0 + t, a.ins, a.nins) | pat));
}
__global__ void unpack_blocks_kernel(BlockArgs a) {
  const uint64_t pat = a.pat[blockIdx.y];
  const double2* in = a.buf + uint64_t(blockIdx.y) * a.cnt;
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t t = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < a.cnt; t += stride)
    __stcs(a.psi + (deposit(a.t0 + t, a.ins, a.nins) | pat), in[t]);
}
__global__ void add_kernel(double* out, const double* in, uint64_t count) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t t = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < count; t += stride) out[t] += in[t];
}

// --------------------------------------------------------------------------- launchers
namespace {
constexpr int kMaxDevices = 64;
int cur_device() {
  int dev = 0;
  cudaGetDevice(&dev);
  return (dev >= 0 && dev < kMaxDevices) ? dev : 0;
}
int g_num_sms[kMaxDevices] = {};
int num_sms() {
  const int dev = cur_device();
  if (!g_num_sms[dev]) {
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    g_num_sms[dev] = v > 0 ? v : 148;
  }
  return g_num_sms[dev];
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
         2 * nwarps * size_t(a.npat) * 16 + size_t(a.nmbar) * 8 + 16 + (a.hist ? (size_t(8) << a.hm) * (a.hacc == 2 ? (a.hglob ? 0 : nwarps) : 1) : 0);
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
  // two quads (8 loads of 16 B) in flight per thread (QGPU_QPT=1: one, A/B)
  const char* qe = std::getenv("QGPU_QPT");
  if (qe && qe[0] == '1') {
    const unsigned g1 = grid_for(a.nquads, kThreads, 8);
    quad_kernel<1><<<g1, kThreads, 0, st>>>(a);
    return cudaGetLastError();
  }
  constexpr int QPT = 2;
  const unsigned g = grid_for(a.nquads, kThreads * QPT, 8);
  quad_kernel<QPT><<<g, kThreads, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_phase(cudaStream_t st, const PhaseArgs& a) {
  if (a.count == 0) return cudaSuccess;
  constexpr int APT = 4;
  const unsigned g = grid_for(a.count, kThreads * APT, 8);
  // position 0 among the fixed (enumerated) positions: whole 32-byte sectors
  bool sector = false;
  for (int i = 0; i < a.nins; ++i) sector = sector || a.ins[i] == 0;
  if (sector) phase_sector_kernel<APT><<<g, kThreads, 0, st>>>(a);
  else phase_kernel<APT><<<g, kThreads, 0, st>>>(a);
  return cudaGetLastError();
}

template <int NR, bool H>
cudaError_t launch_tile_nr(cudaStream_t st, const TileArgs& a, size_t smem) {
  static bool configured[kMaxDevices] = {};  // function attributes are per device
  const int dev = cur_device();
  if (!configured[dev]) {
    cudaError_t e = cudaFuncSetAttribute(tile_kernel<NR, H>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         227 * 1024);
    if (e != cudaSuccess) return e;
    configured[dev] = true;
  }
  const int threads = 32 << a.nw;
  int bps = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, tile_kernel<NR, H>, threads, smem);
  if (bps <= 0) bps = 1;
  const unsigned g = unsigned(std::min<uint64_t>(a.ntiles, uint64_t(num_sms()) * bps));
  tile_kernel<NR, H><<<g, threads, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tile(cudaStream_t st, const TileArgs& a) {
  if (a.ntiles == 0) return cudaSuccess;
  const size_t smem = tile_smem_bytes(a);
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  // the fused-measurement epilogues live only in the H instantiation: they cost registers
  if (a.hist) {
    switch (a.nr) {
      case 0: return launch_tile_nr<0, true>(st, a, smem);
      case 1: return launch_tile_nr<1, true>(st, a, smem);
      case 2: return launch_tile_nr<2, true>(st, a, smem);
      case 3: return launch_tile_nr<3, true>(st, a, smem);
      default: return launch_tile_nr<4, true>(st, a, smem);
    }
  }
  switch (a.nr) {
    case 0: return launch_tile_nr<0, false>(st, a, smem);
    case 1: return launch_tile_nr<1, false>(st, a, smem);
    case 2: return launch_tile_nr<2, false>(st, a, smem);
    case 3: return launch_tile_nr<3, false>(st, a, smem);
    default: return launch_tile_nr<4, false>(st, a, smem);
  }
}

cudaError_t launch_owner_flags(cudaStream_t st, const GatherArgs& a, uint64_t* flags) {
  if (a.count == 0) return cudaSuccess;
  owner_flags_kernel<<<grid_for(a.count, 256, 8), 256, 0, st>>>(a, flags);
  return cudaGetLastError();
}
cudaError_t launch_owned_compact(cudaStream_t st, const GatherArgs& a, const uint64_t* pos, double2* compact) {
  if (a.count == 0) return cudaSuccess;
  owned_compact_kernel<<<grid_for(a.count, 256, 8), 256, 0, st>>>(a, pos, compact);
  return cudaGetLastError();
}
cudaError_t launch_owned_scatter(cudaStream_t st, const GatherArgs& a, const uint64_t* pos, const double2* compact) {
  if (a.count == 0) return cudaSuccess;
  owned_scatter_kernel<<<grid_for(a.count, 256, 8), 256, 0, st>>>(a, pos, compact);
  return cudaGetLastError();
}

cudaError_t launch_gather(cudaStream_t st, const GatherArgs& a) {
  if (a.count == 0) return cudaSuccess;
  const unsigned g = grid_for(a.count, 256, 8);
  gather_kernel<<<g, 256, 0, st>>>(a);
  return cudaGetLastError();
}

// out: device buffer of 2^m doubles; scratch: >= probs_scratch_bytes(m) bytes
size_t probs_scratch_doubles(int) { return 0; }

cudaError_t launch_probs(cudaStream_t st, ProbArgs a, double*) {
  const size_t B = size_t(1) << a.m;
  cudaError_t e = cudaMemsetAsync(a.out, 0, sizeof(double) * B, st);
  if (e != cudaSuccess || a.L == 0) return e;
  const int k = std::countr_zero(a.L);
  ProbMap mp;
  if ((a.L & (a.L - 1)) == 0 && std::getenv("QGPU_PROBS_HIST") == nullptr && plan_probs_map(a, k, &mp)) {
    const unsigned grid = 1u << mp.cbits, threads = 32u << mp.wbits;
    switch (mp.ebits) {
      case 0: probs_mapped_kernel<0><<<grid, threads, 0, st>>>(a, mp); break;
      case 1: probs_mapped_kernel<1><<<grid, threads, 0, st>>>(a, mp); break;
      case 2: probs_mapped_kernel<2><<<grid, threads, 0, st>>>(a, mp); break;
      default: probs_mapped_kernel<3><<<grid, threads, 0, st>>>(a, mp); break;
    }
    return cudaGetLastError();
  }
  const int mode = a.m <= 10 ? 0 : (a.m <= 12 ? 1 : 2);
  const size_t smem = mode == 0 ? B * sizeof(double) * (kThreads / 32) : (mode == 1 ? B * sizeof(double) : 0);
  static bool configured[kMaxDevices] = {};
  const int dev = cur_device();
  if (!configured[dev]) {
    cudaFuncSetAttribute(probs_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024);
    configured[dev] = true;
  }
  const unsigned g = unsigned(num_sms()) * 2;
  probs_kernel<<<g, kThreads, smem, st>>>(a, mode);
  return cudaGetLastError();
}

cudaError_t launch_swap_halves(cudaStream_t st, double2* a, double2* b, int lp, uint64_t half) {
  swap_halves_kernel<<<grid_for(half, 256 * 4, 8), 256, 0, st>>>(a, b, lp, half);
  return cudaGetLastError();
}
cudaError_t launch_pack_blocks(cudaStream_t st, const BlockArgs& a) {
  if (!a.cnt || !a.nb) return cudaSuccess;
  const unsigned gx = std::max(1u, grid_for(a.cnt * a.nb, 256 * 4, 8) / unsigned(a.nb));
  pack_blocks_kernel<<<dim3(gx, unsigned(a.nb)), 256, 0, st>>>(a);
  return cudaGetLastError();
}
cudaError_t launch_unpack_blocks(cudaStream_t st, const BlockArgs& a) {
  if (!a.cnt || !a.nb) return cudaSuccess;
  const unsigned gx = std::max(1u, grid_for(a.cnt * a.nb, 256 * 4, 8) / unsigned(a.nb));
  unpack_blocks_kernel<<<dim3(gx, unsigned(a.nb)), 256, 0, st>>>(a);
  return cudaGetLastError();
}
cudaError_t launch_add(cudaStream_t st, double* out, const double* in, uint64_t count) {
  if (!count) return cudaSuccess;
  add_kernel<<<grid_for(count, 256 * 4, 8), 256, 0, st>>>(out, in, count);
  return cudaGetLastError();
}

// zero-position skipping: materialise the zero halves, psi[i] = 0 for i < L with (i & mask) != 0
__global__ void zero_where_kernel(double2* psi, uint64_t L, uint64_t mask) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < L; i += stride)
    if (i & mask) __stcs(psi + i, make_double2(0.0, 0.0));
}
cudaError_t launch_zero_where(cudaStream_t st, double2* psi, uint64_t L, uint64_t mask) {
  if (!L || !mask) return cudaSuccess;
  zero_where_kernel<<<grid_for(L, 256 * 4, 8), 256, 0, st>>>(psi, L, mask);
  return cudaGetLastError();
}

// FP64 roofline peak: independent DFMA chains (8 per thread, so the pipe, not the latency,
// bounds the issue rate) on every SM; the result is stored so nothing is eliminated.
__global__ void __launch_bounds__(256) fp64_probe_kernel(double* out, int iters, double a, double b) {
  double x[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) x[k] = double(threadIdx.x + k);
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = fma(x[k], a, b);
  }
  double s = 0.0;
#pragma unroll
  for (int k = 0; k < 8; ++k) s += x[k];
  if (s == 12345.678) out[threadIdx.x] = s;  // practically never; keeps the chains live
}

cudaError_t probe_fp64(double* fma_per_s) {
  double* out = nullptr;
  cudaError_t e = cudaMalloc(&out, 256 * sizeof(double));
  if (e != cudaSuccess) return e;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 1 << 14;
  const unsigned grid = unsigned(num_sms()) * 8;
  double best = 0.0;
  fp64_probe_kernel<<<grid, 256>>>(out, iters, 0.999999, 1e-7);  // warm-up
  for (int r = 0; r < 3 && e == cudaSuccess; ++r) {
    cudaEventRecord(a);
    fp64_probe_kernel<<<grid, 256>>>(out, iters, 0.999999, 1e-7);
    cudaEventRecord(b);
    e = cudaEventSynchronize(b);
    float ms = 0;
    if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, a, b);
    if (e == cudaSuccess && ms > 0) best = std::max(best, double(grid) * 256.0 * 8.0 * iters / (ms * 1e-3));
  }
  if (e == cudaSuccess) e = cudaGetLastError();
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(out);
  *fma_per_s = best;
  return e;
}

cudaError_t launch_set_amp(cudaStream_t st, double2* psi, uint64_t i, double re, double im) {
  set_amp_kernel<<<1, 1, 0, st>>>(psi, i, make_double2(re, im));
  return cudaGetLastError();
}

}  // namespace qgpu
