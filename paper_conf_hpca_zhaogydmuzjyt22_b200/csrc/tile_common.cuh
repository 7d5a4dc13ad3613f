// Device code of the fused tile pass (a9), self-contained so that it is compiled both into
// libqgpu.so (the generic, interpreted tile kernel in kernels.cu) and, as source text, by NVRTC
// into per-pass specialised kernels (jit.cpp). No host headers.
//
// Thread/amplitude mapping: a tile holds T = 2^b amplitudes (tile-local index j); tile bits
// 0..4 are the lane bits (physical positions 0..4, so a warp moves 512 contiguous bytes), the
// other b-5 tile bits are split into NR <= 4 REGISTER bits (each thread owns the 2^NR
// amplitudes that differ in them) and nw = b-5-NR WARP bits. OP_REMAP re-distributes the tile
// through shared memory so that other tile bits become register bits; gates on register bits
// run in registers, gates on lane bits use warp shuffles, everything else is a shared-memory op.
#pragma once

#ifdef __CUDACC_RTC__
typedef unsigned int uint32_t;
typedef unsigned short uint16_t;
typedef unsigned long long uint64_t;
#else
#include <cstdint>
#endif

namespace qgpu {

constexpr int kMaxTileBits = 13;
constexpr int kRegAmps = 16;
constexpr int kUmatParam = 512;  // complex entries of the U-matrix pool passed as a kernel parameter

enum OpKind : int {
  OP_REMAP = 0,  // a0: packed register bits (4 bits each), a1: packed warp bits
  OP_U1R = 1,    // 1-qubit U on register bit index a0
  OP_U1L = 2,    // 1-qubit U on lane bit a0
  OP_U2R = 3,    // 2-qubit U on register bit indices a0 (U bit 0), a1 (U bit 1)
  OP_SMEM1 = 4,  // 1-qubit U on tile bit a0 via shared memory (tmask/tmatch: full condition)
  OP_SMEM2 = 5,  // 2-qubit U on tile bits a0, a1 via shared memory
  OP_RUN = 6     // run of diagonal phase patterns: entries [moff, moff + cnt)
};
enum MatClass : int {
  MAT_GENERIC = 0,  // complex 2x2: 16 FP64 per pair
  MAT_REAL = 1,     // real entries (H, RY): 8 per pair
  MAT_X = 2,        // exactly X: a swap, no arithmetic
  MAT_RI = 3,       // real diagonal, imaginary off-diagonal (RX, SX up to phase...): 8 per pair
  // Unit-diagonal forms of REAL / RI: an unconditional op's matrix divided by its U00 (|U00| =
  // |U11| >= the off-diagonal magnitudes, U11 / U00 = +1 or -1), the factor U00 deferred into the
  // pass's tile-uniform scalar. 4 FP64 per pair (one DFMA per output component): H, RX, RY, SX,
  // SY and the real rotation of a split generic gate.
  MAT_RU = 4,       // [[1, b], [c, 1]] real b, c
  MAT_RUN = 5,      // [[1, b], [c, -1]]
  MAT_IU = 6,       // [[1, i b], [i c, 1]] real b, c
  MAT_IUN = 7       // [[1, i b], [i c, -1]]
};
#if defined(__CUDACC__)
#define QGPU_HD __host__ __device__
#else
#define QGPU_HD
#endif
QGPU_HD constexpr bool mat_unit(int c) { return c >= MAT_RU; }
QGPU_HD constexpr bool mat_unit_neg(int c) { return c == MAT_RUN || c == MAT_IUN; }
QGPU_HD constexpr bool mat_unit_imag(int c) { return c == MAT_IU || c == MAT_IUN; }

struct TileOp {
  int kind;
  int a0, a1;
  int cls;                 // matrix class (U ops); RUN: entries of slot 2
  uint32_t tmask, tmatch;  // condition on the thread's fixed tile bits (lane + warp bits)
  uint32_t rmask, rmatch;  // condition on the owned register index r
  uint32_t moff, cnt;      // matrix offset in the pool (complex units) / run entries
  uint64_t omask, omatch;  // tile-uniform condition on (rank << m | index) bits outside the tile
  uint64_t pad;
};
static_assert(sizeof(TileOp) == 64, "TileOp layout");

// One distinct diagonal pattern of a run: the product of its active terms is computed once per
// tile, then applied to the amplitudes matching (tmask,tmatch) x (rmask,rmatch).
struct RunEntry {
  uint32_t tmask, tmatch;
  uint16_t rmask, rmatch, pat, gend;  // gend: last entry of a group with equal (rmask, rmatch)
};
static_assert(sizeof(RunEntry) == 16, "RunEntry layout");
struct PhaseTerm {
  uint64_t omask, omatch;  // tile-uniform condition
  double re, im;           // phase factor
};
// Per-tile pattern constant = Chi(tile >> lb) * Tlo[pattern][tile & (2^lb - 1)] * loose terms:
// terms[first, first + nhi) depend only on tile-index bits >= lb (recomputed once per chunk of
// 2^lb consecutive tiles), terms[first + nhi, first + count) straddle both (evaluated per tile),
// and the terms on the low lb tile-index bits are folded into the host-built table Tlo.
struct Pattern {
  uint32_t first, count, nhi, pad;
};

#if defined(__CUDACC__)

struct TileArgs {
  double2* psi;
  const void* blob;        // TileProgram blob (ops | entries | patterns | terms | scalar | pool)
  int blob_bytes;
  int nops, npat, nscalar;
  int spat;                // pattern holding the tile-uniform (scalar) terms, -1: none
  int lb;                  // low tile-index bits covered by the Tlo tables
  int off_entries, off_patterns, off_terms, off_scalar, off_pool, off_tlo;
  int nr, nw;              // register / warp bits of the thread mapping
  int b, l;
  int spos[kMaxTileBits];
  int nsrun;                      // maximal runs of consecutive tile positions (for deposit)
  int srun_pos[kMaxTileBits], srun_len[kMaxTileBits];
  uint64_t ntiles;          // tiles the kernel visits (tiles selecting a zout half excluded)
  int nzs;                  // tile-index bits of the zout positions: visited tile j is the real
  int zs_pos[32];            // tile deposit(j, zs_pos) -- the skipped halves are never dealt out,
                            // so every CTA receives an equal share of the tiles that do work
  uint64_t L_in;
  uint64_t zin, zout;      // zero-position skipping (Pass::zin / zout): amplitudes with a zin bit
                           // read as zero; tiles with a zout bit are neither loaded nor stored
  uint64_t rank_base;      // rank << m (global bits for tile-uniform conditions)
  const double2* zero;     // >= 2^kMaxTileBits zero amplitudes (source of the expanded region)
  int nbuf;                // tile buffers in shared memory (1, 2 or 3)
  int bstore;              // 1: results staged in the tile buffer and written by bulk async
                           // copies (needs nbuf == 3), 0: per-thread stores from registers
  int remaps;              // the program contains REMAP / shared-memory ops
  int nmbar;               // mbarriers for warp-group remaps (JIT programs), 8 B each in smem
  // measurement fused into the pass (qgpu_apply_circuit_probabilities): hist != nullptr adds
  // |psi_i|^2 of every stored amplitude to hist[bucket(i)], bucket bit j = bit hpos[j] of i
  double* hist;
  int hm;
  int hpos[30];
  // 1: every requested qubit sits on a tile bit of the final mapping (or is never involved), so
  // an owned slot's bucket is the same in every tile: each thread sums |psi|^2 per slot in
  // registers across its tiles and adds to the histogram once at the end of the kernel.
  // 2: requested qubits on lane / register bits mixed with tile-index bits: one private
  // histogram per warp in shared memory (2^hm doubles each); per slot the lanes first sum over
  // the unrequested lane bits (hlred) with shuffles, then the remaining lanes -- whose buckets
  // differ -- add without atomics. 0: requested bits uniform across a warp's slots.
  int hacc;
  uint32_t hlred;
  // mode 2 without private histograms: the lanes add straight to hist (global f64 reductions,
  // no shared memory), used when per-warp histograms would cost the pass CTAs per SM
  int hglob;
  // the pass's U matrices as a kernel parameter (constant bank), when they fit: the NVRTC bodies
  // read them at compile-time offsets (no shared-memory loads, no registers held across tiles)
  int umat_n;
  double2 umat[kUmatParam];
};

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
// tile stores: streaming (evict-first) by default; QGPU_JIT_OPTS="-DQGPU_STORE_WB" / "-DQGPU_STORE_CG"
// compile the NVRTC bodies with write-back / L2-only stores instead (A/B of write-heavy passes)
#if defined(QGPU_STORE_WB)
__device__ __forceinline__ void st_stream(double2* p, double2 v) { *p = v; }
#elif defined(QGPU_STORE_CG)
__device__ __forceinline__ void st_stream(double2* p, double2 v) { __stcg(p, v); }
#else
__device__ __forceinline__ void st_stream(double2* p, double2 v) { __stcs(p, v); }
#endif

// tile index -> base amplitude index: insert the tile positions (as runs of consecutive bits)
__device__ __forceinline__ uint64_t tile_base(uint64_t t, const TileArgs& a) {
  for (int i = 0; i < a.nsrun; ++i) {
    const int p = a.srun_pos[i];
    t = ((t >> p) << (p + a.srun_len[i])) | (t & ((1ull << p) - 1));
  }
  return t;
}

// same with the runs fixed at compile time (NVRTC-specialised passes: Body::kNsrun >= 0)
template <class Body>
__device__ __forceinline__ uint64_t tile_base_t(uint64_t t, const TileArgs& a) {
  if constexpr (Body::kNsrun >= 0) {
#pragma unroll
    for (int i = 0; i < Body::kNsrun; ++i) {
      const int p = Body::kSrunPos[i];
      t = ((t >> p) << (p + Body::kSrunLen[i])) | (t & ((1ull << p) - 1));
    }
    return t;
  } else {
    return tile_base(t, a);
  }
}

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, int src_bytes) {
  const unsigned sa = static_cast<unsigned>(__cvta_generic_to_shared(smem));
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(sa), "l"(gmem), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// ---- bulk asynchronous copies (TMA bulk path, SASS UBLKCP) with an mbarrier per buffer
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("{\n.reg .b64 st;\nmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}\n"
               ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  do {
    asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}\n"
                 : "=r"(done) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  } while (!done);
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("{\n.reg .b64 st;\nmbarrier.arrive.shared::cta.b64 st, [%0];\n}\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;\n"
               ::"l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;\n" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;\n" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }

// (x0, x1) <- U (x0, x1), U = [[u0 u1] [u2 u3]], with the matrix-class shortcut
template <int CLS>
__device__ __forceinline__ void apply2(double2& x0, double2& x1, const double2 (&u)[4]) {
  if (CLS == MAT_X) {
    const double2 t = x0;
    x0 = x1;
    x1 = t;
  } else if (CLS == MAT_REAL) {
    const double a = u[0].x, bq = u[1].x, c = u[2].x, d = u[3].x;
    const double2 y0 = make_double2(fma(a, x0.x, bq * x1.x), fma(a, x0.y, bq * x1.y));
    const double2 y1 = make_double2(fma(c, x0.x, d * x1.x), fma(c, x0.y, d * x1.y));
    x0 = y0;
    x1 = y1;
  } else if (CLS == MAT_RI) {  // u = [[a, i b], [i c, d]] with a, b, c, d real
    const double a = u[0].x, bq = u[1].y, c = u[2].y, d = u[3].x;
    const double2 y0 = make_double2(fma(a, x0.x, -bq * x1.y), fma(a, x0.y, bq * x1.x));
    const double2 y1 = make_double2(fma(d, x1.x, -c * x0.y), fma(d, x1.y, c * x0.x));
    x0 = y0;
    x1 = y1;
  } else if (CLS == MAT_RU || CLS == MAT_RUN) {  // [[1, b], [c, +-1]]
    const double bq = u[1].x, c = u[2].x;
    const double2 x1s = CLS == MAT_RUN ? make_double2(-x1.x, -x1.y) : x1;
    const double2 y0 = make_double2(fma(bq, x1.x, x0.x), fma(bq, x1.y, x0.y));
    const double2 y1 = make_double2(fma(c, x0.x, x1s.x), fma(c, x0.y, x1s.y));
    x0 = y0;
    x1 = y1;
  } else if (CLS == MAT_IU || CLS == MAT_IUN) {  // [[1, i b], [i c, +-1]]
    const double bq = u[1].y, c = u[2].y;
    const double2 x1s = CLS == MAT_IUN ? make_double2(-x1.x, -x1.y) : x1;
    const double2 y0 = make_double2(fma(-bq, x1.y, x0.x), fma(bq, x1.x, x0.y));
    const double2 y1 = make_double2(fma(-c, x0.y, x1s.x), fma(c, x0.x, x1s.y));
    x0 = y0;
    x1 = y1;
  } else {
    const double2 y0 = cfma(u[0], x0, cmul(u[1], x1));
    const double2 y1 = cfma(u[2], x0, cmul(u[3], x1));
    x0 = y0;
    x1 = y1;
  }
}

struct Mapping {
  uint32_t base;   // tile index of the thread's r = 0 amplitude (lane + warp bits)
  uint32_t rb[4];  // tile-index bit of each register bit
  __device__ __forceinline__ uint32_t j(int r) const {
    return base | ((r & 1) ? rb[0] : 0u) | ((r & 2) ? rb[1] : 0u) | ((r & 4) ? rb[2] : 0u) |
           ((r & 8) ? rb[3] : 0u);
  }
};

template <int NR>
__device__ __forceinline__ Mapping make_mapping(const TileOp& op, int nw, int lane, int warp) {
  Mapping mp;
  mp.base = uint32_t(lane);
  for (int k = 0; k < nw; ++k)
    if (warp >> k & 1) mp.base |= 1u << ((op.a1 >> (4 * k)) & 15);
#pragma unroll
  for (int k = 0; k < 4; ++k) mp.rb[k] = (k < NR) ? (1u << ((op.a0 >> (4 * k)) & 15)) : 0u;
  return mp;
}

// Per-tile context handed to the program body.
struct TileCtx {
  double2* s;            // current tile buffer (natural order)
  const TileOp* ops;
  const RunEntry* ents;
  const double2* pool;
  const double2* C;      // per-tile pattern constants
  uint64_t gbase;        // rank << m | tile base index
  uint32_t T;
  int nthr, tid, lane, warp, nw;
  bool own;              // this lane owns amplitudes (b >= 5 always)
  uint64_t* mbar;        // warp-group remap barriers (JIT), one per (remap, group)
  uint32_t mpar;         // their phase parity for this tile
};

template <int NR>
__device__ __forceinline__ void tile_spill(const double2 (&v)[kRegAmps], const TileCtx& c, const Mapping& mp) {
  __syncthreads();
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r)
    if (c.own) c.s[mp.j(r)] = v[r];
  __syncthreads();
}
template <int NR>
__device__ __forceinline__ void tile_reload(double2 (&v)[kRegAmps], const TileCtx& c, const Mapping& mp) {
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) v[r] = c.own ? c.s[mp.j(r)] : make_double2(0, 0);
}

// Static-mapping variants (JIT): slot r of the thread sits at tile index base + J[r], J a
// compile-time table, so every shared-memory access uses an immediate offset.
template <int NR>
__device__ __forceinline__ void tile_spill_j(const double2 (&v)[kRegAmps], const TileCtx& c, uint32_t base,
                                             const uint32_t (&J)[kRegAmps]) {
  __syncthreads();
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r)
    if (c.own) c.s[base + J[r]] = v[r];
  __syncthreads();
}
template <int NR>
__device__ __forceinline__ void tile_reload_j(double2 (&v)[kRegAmps], const TileCtx& c, uint32_t base,
                                              const uint32_t (&J)[kRegAmps]) {
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) v[r] = c.own ? c.s[base + J[r]] : make_double2(0, 0);
}

// Warp-group remap (JIT): a remap that turns register bits into warp bits and back only moves
// amplitudes between the warps that differ in the warp-bit indices it changes (the warp-bit
// indices of unchanged positions are kept), so instead of two CTA-wide barriers the group
// (2, 4 or 8 warps) meets at an mbarrier: every thread stores its slots under the old mapping,
// arrives, waits for the group's phase, then reloads under the new mapping. No WAR hazard: a
// thread's old slots are disjoint from every other thread's old slots, and the tile loop keeps
// one CTA barrier per tile, so the warps of a CTA are never a tile apart.
template <int NR>
__device__ __forceinline__ void tile_store_j(const double2 (&v)[kRegAmps], const TileCtx& c, uint32_t base,
                                             const uint32_t (&J)[kRegAmps]) {
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r)
    if (c.own) c.s[base + J[r]] = v[r];
}
__device__ __forceinline__ void group_sync(const TileCtx& c, int idx) {
  mbar_arrive(c.mbar + idx);
  mbar_wait(c.mbar + idx, c.mpar);
}

__device__ __forceinline__ bool op_active(const TileOp& op, uint64_t gbase) {
  return (gbase & op.omask) == op.omatch;
}

// 1-qubit U on register bit K for every owned pair whose r satisfies (r & rm) == rt
template <int NR, int K, int CLS>
__device__ __forceinline__ void op_u1r(double2 (&v)[kRegAmps], const double2* up, uint32_t rm, uint32_t rt) {
  const double2 u[4] = {up[0], up[1], up[2], up[3]};
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) {
    if (r >> K & 1) continue;
    if ((uint32_t(r) & rm) == rt) apply2<CLS>(v[r], v[r | (1 << K)], u);
  }
}

// 1-qubit U on lane bit t: partner amplitude by warp shuffle
template <int NR, int CLS>
__device__ __forceinline__ void op_u1l(double2 (&v)[kRegAmps], const double2* up, int t, int lane, bool tc,
                                       uint32_t rm, uint32_t rt) {
  const bool hi = (lane >> t) & 1;
  const double2 c0 = hi ? up[2] : up[0], c1 = hi ? up[3] : up[1];
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) {
    if ((uint32_t(r) & rm) != rt) continue;
    double2 pv;
    pv.x = __shfl_xor_sync(0xffffffffu, v[r].x, 1 << t);
    pv.y = __shfl_xor_sync(0xffffffffu, v[r].y, 1 << t);
    const double2 a0 = hi ? pv : v[r], a1 = hi ? v[r] : pv;
    double2 y;
    if (CLS == MAT_X) {
      y = pv;
    } else if (CLS == MAT_REAL) {
      y = make_double2(fma(c0.x, a0.x, c1.x * a1.x), fma(c0.x, a0.y, c1.x * a1.y));
    } else if (CLS == MAT_RI) {  // lo lane: a x0 + i b x1; hi lane: i c x0 + d x1
      const double2 own = hi ? a1 : a0, oth = hi ? a0 : a1;
      const double dg = hi ? up[3].x : up[0].x, od = hi ? up[2].y : up[1].y;
      y = make_double2(fma(dg, own.x, -od * oth.y), fma(dg, own.y, od * oth.x));
    } else if (mat_unit(CLS)) {  // own coefficient +-1: one DFMA per component
      const double2 own = v[r];
      const double2 owns = (mat_unit_neg(CLS) && hi) ? make_double2(-own.x, -own.y) : own;
      if (mat_unit_imag(CLS)) {
        const double od = hi ? up[2].y : up[1].y;
        y = make_double2(fma(-od, pv.y, owns.x), fma(od, pv.x, owns.y));
      } else {
        const double od = hi ? up[2].x : up[1].x;
        y = make_double2(fma(od, pv.x, owns.x), fma(od, pv.y, owns.y));
      }
    } else {
      y = cfma(c0, a0, cmul(c1, a1));
    }
    if (tc) v[r] = y;
  }
}

// 2-qubit U on register bits K0 (U index bit 0) and K1 (bit 1)
template <int NR, int K0, int K1>
__device__ __forceinline__ void op_u2r(double2 (&v)[kRegAmps], const double2* u, uint32_t rm, uint32_t rt) {
  constexpr int m0 = 1 << K0, m1 = 1 << K1;
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) {
    if (r & (m0 | m1)) continue;
    if ((uint32_t(r) & rm) != rt) continue;
    const double2 x0 = v[r], x1 = v[r | m0], x2 = v[r | m1], x3 = v[r | m0 | m1];
#pragma unroll
    for (int row = 0; row < 4; ++row) {
      double2 y = cmul(u[row * 4], x0);
      y = cfma(u[row * 4 + 1], x1, y);
      y = cfma(u[row * 4 + 2], x2, y);
      y = cfma(u[row * 4 + 3], x3, y);
      v[r | (row & 1 ? m0 : 0) | (row & 2 ? m1 : 0)] = y;
    }
  }
}

// Run of diagonal patterns. Slot 0 (no condition on r): one factor for all owned amplitudes;
// slots 1..4 ("r bit k set"): one factor per bit, the 2^NR table is built by doubling; the
// remaining entries have a general condition on r and are applied group by group.
template <int NR>
__device__ __forceinline__ void op_run(double2 (&v)[kRegAmps], const TileOp& op, const TileCtx& c,
                                       const Mapping& mp, int n0, int n1, int n2, int n3, int n4) {
  uint32_t e = op.moff;
  double2 t0 = make_double2(1.0, 0.0);
  for (const uint32_t end = e + uint32_t(n0); e < end; ++e) {
    const RunEntry en = c.ents[e];
    if ((mp.base & en.tmask) == en.tmatch) t0 = cmul(t0, c.C[en.pat]);
  }
  double2 ek[4];
  const int ne[4] = {n1, n2, n3, n4};
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    ek[k] = make_double2(1.0, 0.0);
    for (const uint32_t end = e + uint32_t(ne[k]); e < end; ++e) {
      const RunEntry en = c.ents[e];
      if ((mp.base & en.tmask) == en.tmatch) ek[k] = cmul(ek[k], c.C[en.pat]);
    }
  }
  if (n0 + n1 + n2 + n3 + n4 > 0) {
    double2 P[kRegAmps];
    P[0] = t0;
#pragma unroll
    for (int k = 0; k < NR; ++k)
#pragma unroll
      for (int r = 0; r < (1 << k); ++r) P[r | (1 << k)] = cmul(P[r], ek[k]);
#pragma unroll
    for (int r = 0; r < (1 << NR); ++r) v[r] = cmul(v[r], P[r]);
  }
  double2 acc = make_double2(1.0, 0.0);
  for (const uint32_t end = op.moff + op.cnt; e < end; ++e) {
    const RunEntry en = c.ents[e];
    if ((mp.base & en.tmask) == en.tmatch) acc = cmul(acc, c.C[en.pat]);
    if (en.gend) {
#pragma unroll
      for (int r = 0; r < (1 << NR); ++r) {
        const bool mt = (uint32_t(r) & en.rmask) == en.rmatch;
        v[r] = cmul(v[r], mt ? acc : make_double2(1.0, 0.0));
      }
      acc = make_double2(1.0, 0.0);
    }
  }
}

// ---- JIT variants aware of compile-time zero slots (first-touch expansion, a5): slot r is
// known to be exactly zero when one of its register bits is a tile position >= L_in that no
// non-diagonal op has targeted yet. ZM is the 16-bit mask of such slots.
template <int CLS>
__device__ __forceinline__ void apply2_x1zero(double2& x0, double2& x1, const double2 (&u)[4]) {
  // (x0, 0) -> (u00 x0, u10 x0)
  if (CLS == MAT_X) {
    x1 = x0;
    x0 = make_double2(0.0, 0.0);
  } else if (CLS == MAT_REAL) {
    x1 = make_double2(u[2].x * x0.x, u[2].x * x0.y);
    x0 = make_double2(u[0].x * x0.x, u[0].x * x0.y);
  } else if (CLS == MAT_RU || CLS == MAT_RUN) {  // (x0, 0) -> (x0, c x0)
    x1 = make_double2(u[2].x * x0.x, u[2].x * x0.y);
  } else if (CLS == MAT_IU || CLS == MAT_IUN) {  // (x0, 0) -> (x0, i c x0)
    x1 = make_double2(-u[2].y * x0.y, u[2].y * x0.x);
  } else {
    x1 = cmul(u[2], x0);
    x0 = cmul(u[0], x0);
  }
}
template <int CLS>
__device__ __forceinline__ void apply2_x0zero(double2& x0, double2& x1, const double2 (&u)[4]) {
  // (0, x1) -> (u01 x1, u11 x1)
  if (CLS == MAT_X) {
    x0 = x1;
    x1 = make_double2(0.0, 0.0);
  } else if (CLS == MAT_REAL) {
    x0 = make_double2(u[1].x * x1.x, u[1].x * x1.y);
    x1 = make_double2(u[3].x * x1.x, u[3].x * x1.y);
  } else if (CLS == MAT_RU || CLS == MAT_RUN) {  // (0, x1) -> (b x1, +-x1)
    x0 = make_double2(u[1].x * x1.x, u[1].x * x1.y);
    if (CLS == MAT_RUN) x1 = make_double2(-x1.x, -x1.y);
  } else if (CLS == MAT_IU || CLS == MAT_IUN) {  // (0, x1) -> (i b x1, +-x1)
    x0 = make_double2(-u[1].y * x1.y, u[1].y * x1.x);
    if (CLS == MAT_IUN) x1 = make_double2(-x1.x, -x1.y);
  } else {
    x0 = cmul(u[1], x1);
    x1 = cmul(u[3], x1);
  }
}
template <int NR, int K, int CLS, unsigned ZM>
__device__ __forceinline__ void op_u1r_z(double2 (&v)[kRegAmps], const double2* up, uint32_t rm, uint32_t rt) {
  const double2 u[4] = {up[0], up[1], up[2], up[3]};
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) {
    if (r >> K & 1) continue;
    if ((uint32_t(r) & rm) != rt) continue;
    const int r1 = r | (1 << K);
    const bool z0 = (ZM >> r) & 1, z1 = (ZM >> r1) & 1;
    if (z0 && z1) continue;
    if (z1) apply2_x1zero<CLS>(v[r], v[r1], u);
    else if (z0) apply2_x0zero<CLS>(v[r], v[r1], u);
    else apply2<CLS>(v[r], v[r1], u);
  }
}
template <int NR, int CLS, unsigned ZM>
__device__ __forceinline__ void op_u1l_z(double2 (&v)[kRegAmps], const double2* up, int t, int lane, bool tc,
                                         uint32_t rm, uint32_t rt) {
  const bool hi = (lane >> t) & 1;
  const double2 c0 = hi ? up[2] : up[0], c1 = hi ? up[3] : up[1];
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) {
    if ((uint32_t(r) & rm) != rt) continue;
    if ((ZM >> r) & 1) continue;  // the partner slot (same r, other lane) is zero as well
    double2 pv;
    pv.x = __shfl_xor_sync(0xffffffffu, v[r].x, 1 << t);
    pv.y = __shfl_xor_sync(0xffffffffu, v[r].y, 1 << t);
    const double2 a0 = hi ? pv : v[r], a1 = hi ? v[r] : pv;
    double2 y;
    if (CLS == MAT_X) {
      y = pv;
    } else if (CLS == MAT_REAL) {
      y = make_double2(fma(c0.x, a0.x, c1.x * a1.x), fma(c0.x, a0.y, c1.x * a1.y));
    } else if (CLS == MAT_RI) {
      const double2 own = hi ? a1 : a0, oth = hi ? a0 : a1;
      const double dg = hi ? up[3].x : up[0].x, od = hi ? up[2].y : up[1].y;
      y = make_double2(fma(dg, own.x, -od * oth.y), fma(dg, own.y, od * oth.x));
    } else if (mat_unit(CLS)) {  // own coefficient +-1: one DFMA per component
      const double2 own = v[r];
      const double2 owns = (mat_unit_neg(CLS) && hi) ? make_double2(-own.x, -own.y) : own;
      if (mat_unit_imag(CLS)) {
        const double od = hi ? up[2].y : up[1].y;
        y = make_double2(fma(-od, pv.y, owns.x), fma(od, pv.x, owns.y));
      } else {
        const double od = hi ? up[2].x : up[1].x;
        y = make_double2(fma(od, pv.x, owns.x), fma(od, pv.y, owns.y));
      }
    } else {
      y = cfma(c0, a0, cmul(c1, a1));
    }
    if (tc) v[r] = y;
  }
}
template <int NR, int K0, int K1, unsigned ZM>
__device__ __forceinline__ void op_u2r_z(double2 (&v)[kRegAmps], const double2* u, uint32_t rm, uint32_t rt) {
  constexpr int m0 = 1 << K0, m1 = 1 << K1;
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) {
    if (r & (m0 | m1)) continue;
    if ((uint32_t(r) & rm) != rt) continue;
    if (((ZM >> r) & 1) && ((ZM >> (r | m0)) & 1) && ((ZM >> (r | m1)) & 1) && ((ZM >> (r | m0 | m1)) & 1))
      continue;
    const double2 x0 = v[r], x1 = v[r | m0], x2 = v[r | m1], x3 = v[r | m0 | m1];
#pragma unroll
    for (int row = 0; row < 4; ++row) {
      double2 y = cmul(u[row * 4], x0);
      y = cfma(u[row * 4 + 1], x1, y);
      y = cfma(u[row * 4 + 2], x2, y);
      y = cfma(u[row * 4 + 3], x3, y);
      v[r | (row & 1 ? m0 : 0) | (row & 2 ? m1 : 0)] = y;
    }
  }
}
template <int NR, bool E0, bool E1, bool E2, bool E3, unsigned ZM>
__device__ __forceinline__ void run_apply_table_z(double2 (&v)[kRegAmps], double2 t0, double2 e0, double2 e1,
                                                  double2 e2, double2 e3) {
  double2 P[kRegAmps];
  P[0] = t0;
  const double2 ek[4] = {e0, e1, e2, e3};
  const bool has[4] = {E0, E1, E2, E3};
#pragma unroll
  for (int k = 0; k < NR; ++k)
#pragma unroll
    for (int r = 0; r < (1 << k); ++r) P[r | (1 << k)] = has[k] ? cmul(P[r], ek[k]) : P[r];
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r)
    if (!((ZM >> r) & 1)) v[r] = cmul(v[r], P[r]);
}
// As run_apply_table_z with compile-time identity tracking: T0 = false means t0 == 1, so the
// table entries that are products of identities are neither formed nor applied.
template <int NR, bool T0, bool E0, bool E1, bool E2, bool E3, unsigned ZM>
__device__ __forceinline__ void run_apply_ptab_z(double2 (&v)[kRegAmps], double2 t0, double2 e0, double2 e1,
                                                 double2 e2, double2 e3) {
  double2 P[kRegAmps];
  bool id[kRegAmps];
  P[0] = t0;
  id[0] = !T0;
  const double2 ek[4] = {e0, e1, e2, e3};
  const bool has[4] = {E0, E1, E2, E3};
#pragma unroll
  for (int k = 0; k < NR; ++k)
#pragma unroll
    for (int r = 0; r < (1 << k); ++r) {
      const int q = r | (1 << k);
      if (!has[k]) {
        P[q] = P[r];
        id[q] = id[r];
      } else if (id[r]) {
        P[q] = ek[k];
        id[q] = false;
      } else {
        P[q] = cmul(P[r], ek[k]);
        id[q] = false;
      }
    }
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r)
    if (!((ZM >> r) & 1) && !id[r]) v[r] = cmul(v[r], P[r]);
}
// Same product as run_apply_ptab_z with two 4-entry tables instead of one 16-entry table: A over
// register bits 0-1 (t0, e0, e1), B over bits 2-3 (e2, e3), v[r] *= A[r & 3] * B[r >> 2] applied
// as two multiplies. About the same FP64 count (16 + 12 multiplies + 4 for the tables vs 16 + 15)
// but 8 complex table registers instead of 16 at the program's register peak.
template <int NR, bool T0, bool E0, bool E1, bool E2, bool E3, unsigned ZM>
__device__ __forceinline__ void run_apply_split_z(double2 (&v)[kRegAmps], double2 t0, double2 e0, double2 e1,
                                                  double2 e2, double2 e3) {
  double2 A[4], B[4];
  bool ia[4], ib[4];
  A[0] = t0;
  ia[0] = !T0;
  A[1] = ia[0] ? e0 : cmul(A[0], e0);
  ia[1] = ia[0] && !E0;
  if (!E0) A[1] = A[0];
  A[2] = ia[0] ? e1 : cmul(A[0], e1);
  ia[2] = ia[0] && !E1;
  if (!E1) A[2] = A[0];
  A[3] = ia[1] ? e1 : cmul(A[1], e1);
  ia[3] = ia[1] && !E1;
  if (!E1) A[3] = A[1];
  B[0] = make_double2(1.0, 0.0);
  ib[0] = true;
  B[1] = e2;
  ib[1] = !E2;
  B[2] = e3;
  ib[2] = !E3;
  B[3] = E2 ? (E3 ? cmul(e2, e3) : e2) : e3;
  ib[3] = !E2 && !E3;
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) {
    if ((ZM >> r) & 1) continue;
    const int ra = r & 3, rb = r >> 2;
    const bool use_a = !ia[ra] && (NR >= 1) && (ra < (1 << (NR < 2 ? NR : 2)));
    const bool use_b = NR > 2 && !ib[rb];
    if (use_a) v[r] = cmul(v[r], A[ra]);
    if (use_b) v[r] = cmul(v[r], B[rb]);
  }
}
template <int NR, unsigned RM, unsigned RT, unsigned ZM>
__device__ __forceinline__ void run_apply_group_z(double2 (&v)[kRegAmps], double2 acc) {
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r)
    if ((unsigned(r) & RM) == RT && !((ZM >> r) & 1)) v[r] = cmul(v[r], acc);
}

// JIT helpers for a run whose entries are compile-time: multiply the owned amplitudes by the
// table P[r] = t0 * prod_{k: r_k = 1} e_k (built by doubling; bits without entries skipped).
template <int NR, bool E0, bool E1, bool E2, bool E3>
__device__ __forceinline__ void run_apply_table(double2 (&v)[kRegAmps], double2 t0, double2 e0, double2 e1,
                                                double2 e2, double2 e3) {
  double2 P[kRegAmps];
  P[0] = t0;
  const double2 ek[4] = {e0, e1, e2, e3};
  const bool has[4] = {E0, E1, E2, E3};
#pragma unroll
  for (int k = 0; k < NR; ++k)
#pragma unroll
    for (int r = 0; r < (1 << k); ++r) P[r | (1 << k)] = has[k] ? cmul(P[r], ek[k]) : P[r];
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r) v[r] = cmul(v[r], P[r]);
}
template <int NR, unsigned RM, unsigned RT>
__device__ __forceinline__ void run_apply_group(double2 (&v)[kRegAmps], double2 acc) {
#pragma unroll
  for (int r = 0; r < (1 << NR); ++r)
    if ((unsigned(r) & RM) == RT) v[r] = cmul(v[r], acc);
}

// Shared-memory fallback ops (tile in natural order in c.s; caller spills/reloads)
template <int CLS>
__device__ __forceinline__ void op_smem1(const TileCtx& c, const TileOp& op) {
  const int t = op.a0;
  const double2* up = c.pool + op.moff;
  const double2 u[4] = {up[0], up[1], up[2], up[3]};
  for (uint32_t pp = c.tid; pp < c.T / 2; pp += c.nthr) {
    const uint32_t i0 = uint32_t(insert0(pp, t));
    if ((i0 & op.tmask) != op.tmatch) continue;
    const uint32_t i1 = i0 | (1u << t);
    double2 x0 = c.s[i0], x1 = c.s[i1];
    apply2<CLS>(x0, x1, u);
    c.s[i0] = x0;
    c.s[i1] = x1;
  }
  __syncthreads();
}

__device__ __forceinline__ void op_smem2(const TileCtx& c, const TileOp& op) {
  const int t0 = op.a0, t1 = op.a1;
  const int lo = min(t0, t1), hi = max(t0, t1);
  const double2* u = c.pool + op.moff;
  const uint32_t o1 = 1u << t0, o2 = 1u << t1;
  for (uint32_t pp = c.tid; pp < c.T / 4; pp += c.nthr) {
    const uint32_t i0 = uint32_t(insert0(insert0(pp, lo), hi));
    if ((i0 & op.tmask) != op.tmatch) continue;
    const double2 x0 = c.s[i0], x1 = c.s[i0 | o1], x2 = c.s[i0 | o2], x3 = c.s[i0 | o1 | o2];
#pragma unroll
    for (int row = 0; row < 4; ++row) {
      double2 y = cmul(u[row * 4], x0);
      y = cfma(u[row * 4 + 1], x1, y);
      y = cfma(u[row * 4 + 2], x2, y);
      y = cfma(u[row * 4 + 3], x3, y);
      c.s[i0 | (row & 1 ? o1 : 0u) | (row & 2 ? o2 : 0u)] = y;
    }
  }
  __syncthreads();
}

// Physical offset (within the tile) of an owned slot r under mapping mp: phys is linear in the
// tile bits, phys(j(r)) = phys(base_j) | OR_k r_k phys(rb_k).
struct SlotAddr {
  uint64_t pb;
  uint64_t prb[4];
  __device__ __forceinline__ uint64_t at(int r) const {
    return pb | ((r & 1) ? prb[0] : 0ull) | ((r & 2) ? prb[1] : 0ull) | ((r & 4) ? prb[2] : 0ull) |
           ((r & 8) ? prb[3] : 0ull);
  }
};
template <int NR>
__device__ __forceinline__ SlotAddr slot_addr(const Mapping& mp, const uint64_t* hiOff, uint32_t lowmask, int l) {
  SlotAddr sa;
  sa.pb = (mp.base & lowmask) | hiOff[mp.base >> l];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint32_t bit = mp.rb[q];
    sa.prb[q] = (q < NR) ? ((bit & lowmask) | hiOff[bit >> l]) : 0ull;
  }
  return sa;
}

// Each thread prefetches exactly the slots it owns under the initial mapping (cp.async, 16 B,
// src-size 0 = hardware zero-fill beyond L_in): no thread reads another thread's load, so a
// tile needs no CTA barrier unless its program remaps. ZM: slots known to be zero (skipped).
template <int NR, class Body>
__device__ __forceinline__ void issue_own_loads(double2* buf, const TileArgs& a, const Mapping& mp0,
                                                const SlotAddr& sa0, uint64_t base, unsigned zm, bool own) {
  if (own && base < a.L_in && !(base & a.zin)) {
#pragma unroll
    for (int r = 0; r < (1 << NR); ++r) {
      if ((zm >> r) & 1) continue;
      uint64_t idx;
      uint32_t j;
      if constexpr (Body::kStatic) {
        idx = (base | sa0.pb) + Body::kP0[r];  // the register bits are disjoint from base_j's
        j = mp0.base + Body::kJ0[r];
      } else {
        idx = base | sa0.at(r);
        j = mp0.j(r);
      }
      const bool live = idx < a.L_in && !(idx & a.zin);
      cp_async16(buf + j, a.psi + (live ? idx : 0), live ? 16 : 0);
    }
  }
  asm volatile("cp.async.commit_group;\n" ::: "memory");
}

// Bulk store of a staged tile: the tile buffer holds the results at their tile index; runs of
// 2^l consecutive tile indices are contiguous in HBM. The lanes of warp 0 first wait until the
// previous tile's bulk reads of shared memory are done (that buffer is the next prefetch target),
// then the barrier publishes both facts to the CTA, then they issue one copy per run.
__device__ __forceinline__ void bulk_store_tile(double2* s, const TileArgs& a, uint64_t base, const uint64_t* hiOff,
                                                int warp, int lane) {
  fence_proxy_async();
  if (warp == 0) asm volatile("cp.async.bulk.wait_group.read 0;\n" ::: "memory");
  __syncthreads();
  if (warp == 0) {
    const int nh = 1 << (a.b - a.l);
    const uint32_t run = 16u << a.l;
    for (int h = lane; h < nh; h += 32) bulk_s2g(a.psi + (base | hiOff[h]), s + (size_t(h) << a.l), run);
    bulk_commit();
  }
}

// The persistent tile loop shared by the interpreted and the JIT kernels: one CTA per SM, nbuf
// tile buffers (3; 2 when the program blob is large). Tile i+1 is prefetched into the slots its
// threads will own while tile i is computed in registers; stores go straight from registers
// (lane bits = physical positions 0..4: each warp store writes 512 contiguous bytes). Pattern
// constants are computed per warp and the tile-uniform phase per lane, so a tile without
// remaps runs with no CTA-wide barrier.
// Body: void operator()(double2 (&v)[16], Mapping& mp, const TileCtx& c, const TileArgs& a); Body::kZM0 = slots
// known zero at the start of the pass, Body::kZW0 = warp bits whose warps hold only zeros.
template <int NR, class Body>
__device__ __forceinline__ void tile_driver(const TileArgs& a, Body& body) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  const int b = a.b, l = a.l, nw = a.nw, nbuf = a.nbuf;
  const uint32_t T = 1u << b;
  const int nh = 1 << (b - l);
  const int nthr = blockDim.x, nwarps = nthr >> 5;
  double2* bufs = reinterpret_cast<double2*>(smem_raw);  // nbuf x T
  uint64_t* hiOff = reinterpret_cast<uint64_t*>(bufs + nbuf * T);
  unsigned char* blob = reinterpret_cast<unsigned char*>(hiOff + ((nh + 1) & ~1));
  const TileOp* ops = reinterpret_cast<const TileOp*>(blob);
  const RunEntry* ents = reinterpret_cast<const RunEntry*>(blob + a.off_entries);
  const Pattern* pats = reinterpret_cast<const Pattern*>(blob + a.off_patterns);
  const PhaseTerm* terms = reinterpret_cast<const PhaseTerm*>(blob + a.off_terms);
  const double2* pool = reinterpret_cast<const double2*>(blob + a.off_pool);
  const double2* tlo = reinterpret_cast<const double2*>(blob + a.off_tlo);
  double2* Cw = reinterpret_cast<double2*>(blob + a.blob_bytes);  // per-warp pattern constants
  double2* Chw = Cw + (size_t(nthr) >> 5) * a.npat;               // per-warp high-bit parts
  uint64_t* mbar = reinterpret_cast<uint64_t*>(Chw + (size_t(nthr) >> 5) * a.npat);
  if (threadIdx.x == 0) Body::init_mbar(mbar);
  double* hsm = reinterpret_cast<double*>(mbar + a.nmbar);  // fused-measurement histogram
  // the fused-measurement epilogue: compile-time in NVRTC variants, else TileArgs::hacc
  const int hmode = Body::kHistMode >= 0 ? Body::kHistMode : a.hacc;
  if constexpr (Body::kHist)
    if (a.hist) {
      const int hn = (hmode == 2 ? (a.hglob ? 0 : (blockDim.x >> 5)) : 1) << a.hm;
      for (int i = threadIdx.x; i < hn; i += blockDim.x) hsm[i] = 0.0;
    }

  {
    const int4* src = reinterpret_cast<const int4*>(a.blob);
    int4* dst = reinterpret_cast<int4*>(blob);
    for (int i = threadIdx.x; i < a.blob_bytes / 16; i += nthr) dst[i] = src[i];
  }
  for (int h = threadIdx.x; h < nh; h += nthr) {
    uint64_t off = 0;
    for (int i = l; i < b; ++i)
      if (h >> (i - l) & 1) off |= 1ull << a.spos[i];
    hiOff[h] = off;
  }
  __syncthreads();
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lowmask = (1u << l) - 1;
  TileCtx c;
  c.ops = ops;
  c.ents = ents;
  c.pool = pool;
  c.C = Cw + size_t(warp) * a.npat;
  c.T = T;
  c.nthr = nthr;
  c.tid = tid;
  c.lane = lane;
  c.warp = warp;
  c.nw = nw;
  c.own = lane < int(T);
  c.mbar = mbar;
  c.mpar = 0;
  uint32_t nexec = 0;  // tiles whose program ran (the remap barriers' phase)
  const Mapping mp0 = make_mapping<NR>(ops[0], nw, lane, warp);  // ops[0] is always OP_REMAP
  const SlotAddr sa0 = slot_addr<NR>(mp0, hiOff, lowmask, l);
  const bool wzero = (mp0.base & Body::kZW0) != 0u;  // this warp's slots start in the zero region
  const unsigned zm0 = wzero ? 0xffffu : Body::kZM0;
  (void)nwarps;

  // Tile order: rounds of G CTAs x 2^lb consecutive tiles (CTA i takes chunk i of each round),
  // so a CTA walks runs of 2^lb tiles that share the high tile-index bits; the tiles left over
  // after the full rounds are dealt out one at a time.
  const uint64_t G = gridDim.x, CH = 1ull << a.lb;
  const uint64_t nfull = (a.ntiles / (G * CH)) * CH;  // tiles per CTA in full rounds
  const uint64_t rem0 = nfull * G;
  auto tile_at = [&](uint64_t it) -> uint64_t {
    if (it < nfull) return ((it >> a.lb) * G + blockIdx.x) * CH + (it & (CH - 1));
    return rem0 + blockIdx.x + (it - nfull) * G;
  };
  auto real = [&](uint64_t j) -> uint64_t { return a.nzs ? deposit(j, a.zs_pos, a.nzs) : j; };
  uint64_t tile = tile_at(0);
  uint64_t base_next = tile_base_t<Body>(real(tile), a);  // base of `tile`, carried across iterations
  if (tile < a.ntiles) issue_own_loads<NR, Body>(bufs, a, mp0, sa0, base_next, zm0, c.own);
  int k = 0;
  uint64_t cur_hi = ~0ull;
  double hacc[1 << NR];   // fused measurement with a.hacc: per-slot sums over this thread's tiles
  Mapping mpf = mp0;      // the final mapping (the same after every tile)
  uint32_t hb0 = 0, hrb[4] = {0u, 0u, 0u, 0u};  // hmode == 2: bucket parts (thread, register bits)
  bool hbk_set = false;
  if constexpr (Body::kHist) {
#pragma unroll
    for (int r = 0; r < (1 << NR); ++r) hacc[r] = 0.0;
  }
  for (uint64_t it = 0; tile < a.ntiles; ++it) {
    double2* s = bufs + k * T;
    const int kn = (k + 1 == nbuf) ? 0 : k + 1;
    const uint64_t base = base_next;
    const uint64_t gbase = a.rank_base | base;
    const uint64_t next = tile_at(it + 1);
    const bool more = next < a.ntiles;
    base_next = tile_base_t<Body>(real(next), a);
    // nbuf >= 2: prefetch into the next buffer now; nbuf == 1 (programs without remaps, every
    // thread reads only its own slots): prefetch into the same buffer right after the reload
    if (more && nbuf > 1) issue_own_loads<NR, Body>(bufs + kn * T, a, mp0, sa0, base_next, zm0, c.own);
    if (base & a.zout) {
      // zero-position skipping: a non-tile bit of this tile selects a half that is zero and is
      // not materialised in memory -> nothing to load, compute or store
      if (more && nbuf == 1) {
        cp_async_wait_all();
        issue_own_loads<NR, Body>(s, a, mp0, sa0, base_next, zm0, c.own);
      }
      k = kn;
      tile = next;
      continue;
    }
    if (base >= a.L_in || (base & a.zin)) {
      // the whole tile lies in the zero region of a first-touch expansion and no op of the pass
      // targets its non-tile bits: it stays zero -> store zeros, skip the program
      if (a.bstore) {
        if (c.own) {
#pragma unroll
          for (int r = 0; r < (1 << NR); ++r) s[mp0.j(r)] = make_double2(0.0, 0.0);
        }
        bulk_store_tile(s, a, base, hiOff, warp, lane);
        k = kn;
        tile = next;
        continue;
      }
      if (c.own) {
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r) st_stream(a.psi + (base | sa0.at(r)), make_double2(0.0, 0.0));
      }
      if (more && nbuf == 1) {
        cp_async_wait_all();
        issue_own_loads<NR, Body>(s, a, mp0, sa0, base_next, zm0, c.own);
      }
      k = kn;
      tile = next;
      // no barrier: a zero tile neither reads nor fills its buffer (its loads were skipped), so
      // running ahead through zero tiles cannot overwrite a buffer another warp still reads --
      // the barrier after each live tile (every program with remaps ends a live tile with one)
      // already orders every reuse of a buffer
      continue;
    }
    // pattern constants of this tile, per warp (lane-strided; each lane owns the same patterns
    // in Chw and Cw): high-bit part once per run of 2^lb tiles, then table x loose terms
    {
      const uint64_t treal = real(tile);
      const uint64_t hi = treal >> a.lb;
      const uint32_t lo = uint32_t(treal) & uint32_t(CH - 1);
      double2* cw = Cw + size_t(warp) * a.npat;
      double2* chw = Chw + size_t(warp) * a.npat;
      if (hi != cur_hi) {
        cur_hi = hi;
        for (int pi = lane; pi < a.npat; pi += 32) {
          double2 cc = make_double2(1.0, 0.0);
          const Pattern pt = pats[pi];
          for (uint32_t q = pt.first; q < pt.first + pt.nhi; ++q)
            if ((gbase & terms[q].omask) == terms[q].omatch) cc = cmul(cc, make_double2(terms[q].re, terms[q].im));
          chw[pi] = cc;
        }
      }
      for (int pi = lane; pi < a.npat; pi += 32) {
        double2 cc = cmul(chw[pi], tlo[(size_t(pi) << a.lb) + lo]);
        const Pattern pt = pats[pi];
        for (uint32_t q = pt.first + pt.nhi; q < pt.first + pt.count; ++q)
          if ((gbase & terms[q].omask) == terms[q].omatch) cc = cmul(cc, make_double2(terms[q].re, terms[q].im));
        cw[pi] = cc;
      }
    }
    if (more && nbuf > 1) asm volatile("cp.async.wait_group 1;\n" ::: "memory");
    else cp_async_wait_all();
    __syncwarp();
    // tile-uniform phase (the scalar pattern)
    const double2 sc = (Body::kHasScalar && a.spat >= 0) ? Cw[size_t(warp) * a.npat + a.spat] : make_double2(1.0, 0.0);
    c.s = s;
    c.gbase = gbase;
    double2 v[kRegAmps];
    Mapping mp = mp0;
#pragma unroll
    for (int r = 0; r < (1 << NR); ++r) {
      uint32_t j;
      if constexpr (Body::kStatic) j = mp0.base + Body::kJ0[r];
      else j = mp0.j(r);
      v[r] = (c.own && !((zm0 >> r) & 1)) ? s[j] : make_double2(0.0, 0.0);
    }
    // nbuf == 1 without remaps: each thread reads only its own slots, so the next tile's loads
    // can go into the buffer right after this reload; with remaps (two CTAs per SM, each single-
    // buffered: the other CTA's compute covers this one's load latency) the buffer is free only
    // once every thread of the CTA has finished the program's remaps
    if (more && nbuf == 1 && !a.remaps) issue_own_loads<NR, Body>(s, a, mp0, sa0, base_next, zm0, c.own);
    c.mpar = nexec & 1u;
    ++nexec;
    // nbuf == 1 with remaps: the next tile's loads go into the buffer once every thread is past
    // the program's last remap / shared-memory op -- at that op when the body marks it
    // (Body::kEarlyPrefetch, NVRTC bodies: the rest of the program overlaps the load latency),
    // else after the program. Bulk stores read the buffer at the end: no early prefetch then.
    const bool early = Body::kEarlyPrefetch && more && nbuf == 1 && a.remaps && !a.bstore;
    body(v, mp, c, a, [&]() {
      if (early) {
        __syncthreads();
        issue_own_loads<NR, Body>(s, a, mp0, sa0, base_next, zm0, c.own);
      }
    });
    if (more && nbuf == 1 && a.remaps && !early) {
      __syncthreads();
      issue_own_loads<NR, Body>(s, a, mp0, sa0, base_next, zm0, c.own);
    }
    if (Body::kHasScalar && !Body::kScalarFolded && !(sc.x == 1.0 && sc.y == 0.0)) {
#pragma unroll
      for (int r = 0; r < (1 << NR); ++r) v[r] = cmul(v[r], sc);
    }
    if constexpr (Body::kHist) if (a.hist && c.own && hmode == 1) {  // buckets fixed per slot
#pragma unroll
      for (int r = 0; r < (1 << NR); ++r) hacc[r] += fma(v[r].x, v[r].x, v[r].y * v[r].y);
      mpf = mp;
    }
    if constexpr (Body::kHist) if (a.hist && hmode == 2) {
      // per-warp private histogram. Bucket extraction is linear in the index bits, so a slot's
      // bucket = hb0 (thread part at tile base 0) | hrb[k] for each set register bit k of r |
      // bt (the tile base's bits, uniform); the final mapping is the same in every tile
      if (!hbk_set) {
        hbk_set = true;
        uint64_t pbh = 0;
        SlotAddr sah{};
        if constexpr (Body::kStatic) pbh = (mp.base & lowmask) | hiOff[mp.base >> l];
        else sah = slot_addr<NR>(mp, hiOff, lowmask, l);
        auto bkt = [&](uint64_t idx) {
          uint32_t bk = 0;
          for (int j = 0; j < a.hm; ++j) bk |= uint32_t(idx >> a.hpos[j] & 1) << j;
          return bk;
        };
        if constexpr (Body::kStatic) hb0 = bkt(pbh);
        else hb0 = bkt(sah.pb);
#pragma unroll
        for (int k = 0; k < NR; ++k) {
          if constexpr (Body::kStatic) hrb[k] = bkt(Body::kPF[1 << k]);
          else hrb[k] = bkt(sah.prb[k]);
        }
      }
      uint32_t bt = hb0;
      for (int j = 0; j < a.hm; ++j) bt |= uint32_t(gbase >> a.hpos[j] & 1) << j;
      double* hw = hsm + (size_t(warp) << a.hm);
      if constexpr (Body::kHistRS) {
        // compile-time epilogue (NVRTC variants, masks Body::kHlred / kDead): slots that differ
        // only in unrequested register bits are summed first; then, per unrequested lane bit,
        // a reduce-scatter step (recursive halving): the two lanes exchange half of their live
        // slot sums and each keeps the half selected by its lane bit, so s steps cost
        // 2^NL (1 - 2^-s) shuffled doubles instead of a butterfly on every slot, and afterwards
        // every lane adds its own 2^(NL - s) buckets (all distinct across the warp)
        constexpr uint32_t kLB = ((1u << NR) - 1u) & ~Body::kDead;
        constexpr int kNL = int(kLB & 1u) + int(kLB >> 1 & 1u) + int(kLB >> 2 & 1u) + int(kLB >> 3 & 1u);
        double x[1 << NR];
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r) x[r] = fma(v[r].x, v[r].x, v[r].y * v[r].y);
#pragma unroll
        for (int k = 0; k < NR; ++k)
          if (Body::kDead >> k & 1u) {
#pragma unroll
            for (int r = 0; r < (1 << NR); ++r)
              if (r >> k & 1) x[r & ~(1 << k)] += x[r];
          }
        // y[i]: the live slot whose live register bits are the bits of i (compile-time deposit)
        double y[1 << NR];
        uint32_t lbk[4] = {0u, 0u, 0u, 0u};  // bucket part of index bit t of y
        {
          int t = 0;
#pragma unroll
          for (int k = 0; k < NR; ++k)
            if (kLB >> k & 1u) lbk[t++] = hrb[k];
        }
#pragma unroll
        for (int i = 0; i < (1 << kNL); ++i) {
          int r = 0, t = 0;
#pragma unroll
          for (int k = 0; k < NR; ++k)
            if (kLB >> k & 1u) r |= ((i >> t++) & 1) << k;
          y[i] = x[r];
        }
        uint32_t bb = bt;
        uint32_t tail = 0u;  // unrequested lane bits left after the halving steps (butterfly)
        int size_log = kNL;
#pragma unroll
        for (int k = 0; k < 5; ++k) {
          if (!(Body::kHlred >> k & 1u)) continue;
          if (size_log == 0) {
            tail |= 1u << k;
            y[0] += __shfl_xor_sync(0xffffffffu, y[0], 1 << k);
            continue;
          }
          const bool h = (lane >> k) & 1;
          const int half = 1 << (size_log - 1);
#pragma unroll
          for (int i = 0; i < (1 << kNL) / 2; ++i) {
            if (i >= half) continue;
            const double lo = y[i], hi = y[i + half];
            const double send = h ? lo : hi;
            const double keep = h ? hi : lo;
            y[i] = keep + __shfl_xor_sync(0xffffffffu, send, 1 << k);
          }
          if (h) bb |= lbk[size_log - 1];
          --size_log;
        }
        if ((uint32_t(lane) & tail) == 0u) {
          double old[1 << NR];
          uint32_t bk[1 << NR];
#pragma unroll
          for (int i = 0; i < (1 << kNL); ++i) {
            if (i >= (1 << size_log)) continue;
            bk[i] = bb;
#pragma unroll
            for (int t = 0; t < 4; ++t)
              if (t < size_log && (i >> t & 1)) bk[i] |= lbk[t];
            if constexpr (!Body::kHistGlob) old[i] = hw[bk[i]];
          }
#pragma unroll
          for (int i = 0; i < (1 << kNL); ++i)
            if (i < (1 << size_log)) {
              if constexpr (Body::kHistGlob) atomicAdd(a.hist + bk[i], y[i]);  // RED.ADD.F64, no return
              else hw[bk[i]] = old[i] + y[i];
            }
        }
      } else {
      const bool writer = (uint32_t(lane) & a.hlred) == 0u;
      double x[1 << NR];
#pragma unroll
      for (int r = 0; r < (1 << NR); ++r) {
        x[r] = fma(v[r].x, v[r].x, v[r].y * v[r].y);
#pragma unroll
        for (int k = 0; k < 5; ++k)
          if (a.hlred >> k & 1) x[r] += __shfl_xor_sync(0xffffffffu, x[r], 1 << k);
      }
      // slots that differ only in unrequested register bits share a bucket: sum them first, so
      // the remaining ("live") slots have distinct buckets and all their loads can be issued
      // before any store (one shared-memory latency per tile instead of one per slot)
      uint32_t dead = 0;
#pragma unroll
      for (int k = 0; k < NR; ++k)
        if (hrb[k] == 0u) {
          dead |= 1u << k;
#pragma unroll
          for (int r = 0; r < (1 << NR); ++r)
            if (r >> k & 1) x[r & ~(1 << k)] += x[r];
        }
      if (writer) {
        uint32_t bk[1 << NR];
        double old[1 << NR];
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r) {
          bk[r] = bt;
#pragma unroll
          for (int k = 0; k < NR; ++k)
            if (r >> k & 1) bk[r] |= hrb[k];
          old[r] = ((uint32_t(r) & dead) == 0u && !a.hglob) ? hw[bk[r]] : 0.0;
        }
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r)
          if ((uint32_t(r) & dead) == 0u) {
            if (a.hglob) atomicAdd(a.hist + bk[r], x[r]);
            else hw[bk[r]] = old[r] + x[r];
          }
      }
      }
    }
    if constexpr (Body::kHist) if (a.hist && c.own && hmode == 0) {  // fused measurement: final amplitudes in registers
      uint64_t pbh = 0;
      SlotAddr sah{};
      if constexpr (Body::kStatic) pbh = base | (mp.base & lowmask) | hiOff[mp.base >> l];
      else sah = slot_addr<NR>(mp, hiOff, lowmask, l);
      auto bucket = [&](int r) {
        uint64_t idx;
        if constexpr (Body::kStatic) idx = pbh + Body::kPF[r];
        else idx = base | sah.at(r);
        idx |= a.rank_base;
        uint32_t bk = 0;
        for (int j = 0; j < a.hm; ++j) bk |= uint32_t(idx >> a.hpos[j] & 1) << j;
        return bk;
      };
      // Requested qubits on tile-index / warp bits only (the usual case) give one bucket per
      // warp: sum in registers, reduce across the warp, one shared atomic. Otherwise group per
      // slot: warp-uniform buckets reduce, mixed ones add lane by lane.
      const uint32_t b0 = bucket(0);
      bool same = true;
      double acc = 0.0;
#pragma unroll
      for (int r = 0; r < (1 << NR); ++r) {
        same = same && bucket(r) == b0;
        acc += fma(v[r].x, v[r].x, v[r].y * v[r].y);
      }
      const uint32_t full = 0xffffffffu;
      if (__all_sync(full, same) && __all_sync(full, b0 == __shfl_sync(full, b0, 0))) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(full, acc, o);
        if (c.lane == 0) atomicAdd(hsm + b0, acc);
      } else {
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r) {
          const uint32_t bk = bucket(r);
          double x = fma(v[r].x, v[r].x, v[r].y * v[r].y);
          if (__all_sync(full, bk == __shfl_sync(full, bk, 0))) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(full, x, o);
            if (c.lane == 0) atomicAdd(hsm + bk, x);
          } else {
            atomicAdd(hsm + bk, x);
          }
        }
      }
    }
    if (a.bstore) {
      if (c.own) {
        if constexpr (Body::kStatic) {
#pragma unroll
          for (int r = 0; r < (1 << NR); ++r) s[mp.base + Body::kJF[r]] = v[r];
        } else {
#pragma unroll
          for (int r = 0; r < (1 << NR); ++r) s[mp.j(r)] = v[r];
        }
      }
      bulk_store_tile(s, a, base, hiOff, warp, lane);
    } else if (c.own) {
      if constexpr (Body::kStatic) {
        const uint64_t pb = base | (mp.base & lowmask) | hiOff[mp.base >> l];
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r) st_stream(a.psi + (pb + Body::kPF[r]), v[r]);
      } else {
        const SlotAddr sa = slot_addr<NR>(mp, hiOff, lowmask, l);
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r) st_stream(a.psi + (base | sa.at(r)), v[r]);
      }
    }
    k = kn;
    tile = next;
    // the lanes of this warp are done reading this tile's pattern constants before the next
    // tile's constants are written
    __syncwarp();
    // programs with remaps read other threads' slots of this tile's buffer: no warp may run
    // ahead and prefetch into it (two buffers: the next tile's; three: the tile after a skipped
    // zero / zout tile, which has no barrier of its own) until every warp has finished reading
    // it. With warp-group remaps this is also the one CTA barrier per tile bounding warp drift.
    if (a.remaps) __syncthreads();
  }
  if (a.bstore && warp == 0) bulk_wait_all();  // shared memory must outlive the bulk reads
  if constexpr (Body::kHist) {
    if (a.hist) {
      if (hmode == 1 && c.own) {
        // bucket of slot r: its tile-local index under the final mapping (tile base bits are not
        // requested, so base = 0); one shared-memory add per slot and thread
        uint64_t pbh = 0;
        SlotAddr sah{};
        if constexpr (Body::kStatic) pbh = (mpf.base & lowmask) | hiOff[mpf.base >> l];
        else sah = slot_addr<NR>(mpf, hiOff, lowmask, l);
#pragma unroll
        for (int r = 0; r < (1 << NR); ++r) {
          uint64_t idx;
          if constexpr (Body::kStatic) idx = pbh + Body::kPF[r];
          else idx = sah.at(r);
          uint32_t bk = 0;
          for (int j = 0; j < a.hm; ++j) bk |= uint32_t(idx >> a.hpos[j] & 1) << j;
          if (hacc[r] != 0.0) atomicAdd(hsm + bk, hacc[r]);
        }
      }
      __syncthreads();
      const int hw = hmode == 2 ? (a.hglob ? 0 : int(blockDim.x >> 5)) : 1;
      for (int i = threadIdx.x; i < (hw ? (1 << a.hm) : 0); i += blockDim.x) {
        double t = 0.0;
        for (int w = 0; w < hw; ++w) t += hsm[(size_t(w) << a.hm) + i];
        if (t != 0.0) atomicAdd(a.hist + i, t);
      }
    }
  }
}

#endif  // __CUDACC__

}  // namespace qgpu
