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

__device__ __forceinline__ double2 cmul(double2 a, double2 b) {
  return make_double2(fma(a.x, b.x, -a.y * b.y), fma(a.x, b.y, a.y * b.x));
}
// a*b + c
__device__ __forceinline__ double2 cfma(double2 a, double2 b, double2 c) {
  return make_double2(fma(a.x, b.x, fma(-a.y, b.y, c.x)), fma(a.x, b.y, fma(a.y, b.x, c.y)));
}
__device__ __forceinline__ uint64_t insert0(uint64_t v, int b) {
  const uint64_t lo = v & ((1ull << b) - 1);
  return ((v >> b) << (b + 1)) | lo;
}
// insert zero bits at the (ascending) positions ins[0..nins)
__device__ __forceinline__ uint64_t deposit(uint64_t v, const int* ins, int nins) {
  for (int i = 0; i < nins; ++i) v = insert0(v, ins[i]);
  return v;
}
__device__ __forceinline__ double2 ld_stream(const double2* p) { return __ldcs(p); }
__device__ __forceinline__ void st_stream(double2* p, double2 v) { __stcs(p, v); }

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
// One CTA processes tiles of T = 2^b amplitudes: tile-local bit i <-> physical position
// spos[i]; spos[0..l) = 0..l-1, so a warp moves 32 consecutive amplitudes (512 B). The
// non-tile bits of the live range index the tiles (grid-stride, persistent CTAs).
//  * load: cp.async (LDGSTS) global -> shared, 16 B per request, every request of the tile in
//    flight at once with no register staging; requests at index >= L_in use src-size 0, i.e.
//    the hardware zero-fills them (first-touch expansion, a5).
//  * op conditions on bits outside the tile are tile-uniform: evaluated once per tile into
//    `active`. PHASE ops whose condition lies entirely outside the tile multiply the whole
//    tile by one scalar; they commute with every op of the pass (which act on tile bits only),
//    so their product is applied once, at the store.
//  * U1/U2 ops: pairs/quads read-modify-write in shared memory, one barrier per op.
//  * runs of PHASE ops: each thread keeps its 16 amplitudes in registers across the run; the
//    condition on the thread's fixed tile bits is tested once per op and thread.
constexpr int kTileMaxPer = 16;  // amplitudes per thread (T <= 16 * kThreads = 4096)

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, int src_bytes) {
  const unsigned sa = static_cast<unsigned>(__cvta_generic_to_shared(smem));
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(sa), "l"(gmem), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.wait_all;\n" ::: "memory");
}

__global__ void __launch_bounds__(kThreads, 2) tile_kernel(TileArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int b = a.b, l = a.l;
  const uint32_t T = 1u << b;
  const int nh = 1 << (b - l);
  double2* s = reinterpret_cast<double2*>(smem_raw);
  uint64_t* hiOff = reinterpret_cast<uint64_t*>(s + T);
  unsigned char* blob = reinterpret_cast<unsigned char*>(hiOff + ((nh + 1) & ~1));
  const TileOp* ops = reinterpret_cast<const TileOp*>(blob);
  const double2* pool = reinterpret_cast<const double2*>(blob + a.ops_bytes);
  unsigned char* active = blob + a.ops_bytes + size_t(a.npool) * 16;
  double2* scal_s = reinterpret_cast<double2*>(active + ((a.nops + 15) & ~15));

  {  // stage the pass's ops and matrices in shared memory (once per CTA)
    const int4* src = reinterpret_cast<const int4*>(a.blob);
    int4* dst = reinterpret_cast<int4*>(blob);
    const int n16 = (a.ops_bytes + a.npool * 16) / 16;
    for (int i = threadIdx.x; i < n16; i += kThreads) dst[i] = src[i];
  }
  for (int h = threadIdx.x; h < nh; h += kThreads) {
    uint64_t off = 0;
    for (int i = l; i < b; ++i)
      if (h >> (i - l) & 1) off |= 1ull << a.spos[i];
    hiOff[h] = off;
  }
  __syncthreads();
  const uint32_t lowmask = (1u << l) - 1;
  const int per = (T + kThreads - 1) / kThreads;
  const uint32_t tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31;

  for (uint64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x) {
    const uint64_t base = deposit(tile, a.spos, b);
    const uint64_t gbase = a.rank_base | base;
    // ---- issue every load of the tile
#pragma unroll
    for (int r = 0; r < kTileMaxPer; ++r) {
      const uint32_t j = tid + r * kThreads;
      if (r < per && j < T) {
        const uint64_t idx = base | (j & lowmask) | hiOff[j >> l];
        const bool live = idx < a.L_in;
        cp_async16(s + j, a.psi + (live ? idx : 0), live ? 16 : 0);
      }
    }
    asm volatile("cp.async.commit_group;\n" ::: "memory");
    // ---- tile-uniform op conditions (overlaps the loads)
    for (int k = tid; k < a.nops; k += kThreads)
      active[k] = (gbase & ops[k].omask) == ops[k].omatch;
    __syncthreads();
    if (warp == 0) {  // product of outside-only phases: lane-strided, then butterfly
      double2 sc = make_double2(1.0, 0.0);
      for (int k = lane; k < a.nscalar; k += 32)
        if (active[k]) sc = cmul(sc, pool[ops[k].moff]);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        double2 t;
        t.x = __shfl_xor_sync(0xffffffffu, sc.x, o);
        t.y = __shfl_xor_sync(0xffffffffu, sc.y, o);
        sc = cmul(sc, t);
      }
      if (lane == 0) *scal_s = sc;
    }
    cp_async_wait_all();
    __syncthreads();
    // ---- apply the pass's ops in order
    int i = a.nscalar;
    while (i < a.nops) {
      const int kind = ops[i].kind;
      if (kind == OP_PHASE) {
        // a run of commuting phase terms, grouped by their condition on the owned index r:
        // accumulate each group's product per thread, then multiply the matching amplitudes
        double2 v[kTileMaxPer];
#pragma unroll
        for (int r = 0; r < kTileMaxPer; ++r) {
          const uint32_t jj = tid + r * kThreads;
          if (r < per && jj < T) v[r] = s[jj];
        }
        double2 acc = make_double2(1.0, 0.0);
        bool any = false;
        for (;; ++i) {
          const TileOp& o = ops[i];
          if (active[i] && (tid & o.lmask & (kThreads - 1)) == (o.lmatch & (kThreads - 1))) {
            acc = cmul(acc, pool[o.moff]);
            any = true;
          }
          if (o.t0) {  // end of group: apply to the owned amplitudes whose r matches
            if (any) {
              const uint32_t mh = o.lmask >> 8, th = o.lmatch >> 8;
#pragma unroll
              for (int r = 0; r < kTileMaxPer; ++r)
                if (r < per && (uint32_t(r) & mh) == th) v[r] = cmul(v[r], acc);
            }
            acc = make_double2(1.0, 0.0);
            any = false;
          }
          if (o.t1) break;
        }
        ++i;
#pragma unroll
        for (int r = 0; r < kTileMaxPer; ++r) {
          const uint32_t jj = tid + r * kThreads;
          if (r < per && jj < T) s[jj] = v[r];
        }
        __syncthreads();
      } else if (kind == OP_U1) {
        if (active[i]) {
          const int t = ops[i].t0;
          const uint32_t lm = ops[i].lmask;
          const double2* u = pool + ops[i].moff;
          const double2 u00 = u[0], u01 = u[1], u10 = u[2], u11 = u[3];
          for (uint32_t p = tid; p < T / 2; p += kThreads) {
            const uint32_t i0 = uint32_t(insert0(p, t));
            if ((i0 & lm) != lm) continue;
            const uint32_t i1 = i0 | (1u << t);
            const double2 x0 = s[i0], x1 = s[i1];
            s[i0] = cfma(u00, x0, cmul(u01, x1));
            s[i1] = cfma(u10, x0, cmul(u11, x1));
          }
          __syncthreads();
        }
        ++i;
      } else {  // OP_U2
        if (active[i]) {
          const int t0 = ops[i].t0, t1 = ops[i].t1;
          const int lo = min(t0, t1), hi = max(t0, t1);
          const uint32_t lm = ops[i].lmask;
          const double2* u = pool + ops[i].moff;
          const uint32_t o1 = 1u << t0, o2 = 1u << t1;
          for (uint32_t p = tid; p < T / 4; p += kThreads) {
            const uint32_t i0 = uint32_t(insert0(insert0(p, lo), hi));
            if ((i0 & lm) != lm) continue;
            const double2 x0 = s[i0], x1 = s[i0 | o1], x2 = s[i0 | o2], x3 = s[i0 | o1 | o2];
#pragma unroll
            for (int row = 0; row < 4; ++row) {
              double2 y = cmul(u[row * 4], x0);
              y = cfma(u[row * 4 + 1], x1, y);
              y = cfma(u[row * 4 + 2], x2, y);
              y = cfma(u[row * 4 + 3], x3, y);
              const uint32_t o = (row & 1 ? o1 : 0u) | (row & 2 ? o2 : 0u);
              s[i0 | o] = y;
            }
          }
          __syncthreads();
        }
        ++i;
      }
    }
    // ---- store every amplitude of the tile (including the expanded zero region)
    const double2 sc = *scal_s;
    const bool has_sc = !(sc.x == 1.0 && sc.y == 0.0);
#pragma unroll
    for (int r = 0; r < kTileMaxPer; ++r) {
      const uint32_t j = tid + r * kThreads;
      if (r < per && j < T) {
        const double2 x = has_sc ? cmul(s[j], sc) : s[j];
        st_stream(a.psi + (base | (j & lowmask) | hiOff[j >> l]), x);
      }
    }
    __syncthreads();
  }
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
      if ((phys >> a.m) == a.rank && (phys & ((1ull << a.m) - 1)) < a.L)
        v = a.psi[phys & ((1ull << a.m) - 1)];
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
    uint32_t y = 0;
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
    uint64_t y = 0;
    for (int j = 0; j < a.m; ++j) y |= ((i >> a.ppos[j]) & 1) << j;
    atomicAdd(&a.out[y], v.x * v.x + v.y * v.y);
  }
}

__global__ void set_amp_kernel(double2* psi, uint64_t i, double2 v) { psi[i] = v; }

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

size_t tile_smem_bytes(int b, int l, int nops, int ops_bytes, int npool) {
  const size_t nh = size_t(1) << (b - l);
  return (size_t(1) << b) * 16 + ((nh + 1) & ~size_t(1)) * 8 + size_t(ops_bytes) +
         size_t(npool) * 16 + size_t((nops + 15) & ~15) + 16;
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

cudaError_t launch_tile(cudaStream_t st, const TileArgs& a) {
  if (a.ntiles == 0) return cudaSuccess;
  const size_t smem = tile_smem_bytes(a.b, a.l, a.nops, a.ops_bytes, a.npool);
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(tile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         227 * 1024);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  int bps = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, tile_kernel, kThreads, smem);
  if (bps <= 0) bps = 1;
  const unsigned g = unsigned(std::min<uint64_t>(a.ntiles, uint64_t(num_sms()) * bps));
  tile_kernel<<<g, kThreads, smem, st>>>(a);
  return cudaGetLastError();
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

cudaError_t launch_set_amp(cudaStream_t st, double2* psi, uint64_t i, double re, double im) {
  set_amp_kernel<<<1, 1, 0, st>>>(psi, i, make_double2(re, im));
  return cudaGetLastError();
}

}  // namespace qgpu
