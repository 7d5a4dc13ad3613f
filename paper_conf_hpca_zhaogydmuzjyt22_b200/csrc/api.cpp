// C ABI of libqgpu (include/qgpu.h): state management, execution of the planned passes,
// readout, statistics. No exception crosses the ABI; every CUDA error is mapped to a status.
#include <cuda_runtime.h>

#include <algorithm>
#include <bit>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <exception>
#include <string>
#include <vector>

#include "comm.h"
#include "jit.h"
#include "kernels.h"
#include "qgpu_internal.h"

using namespace qgpu;

struct qgpu_circuit {
  Circuit c;
};

namespace {
// A planned circuit for a given starting qubit map: passes (with their resolved JIT kernels)
// and their packed programs (pinned host blob + device copy). Reused when the same circuit is
// applied again from the same map (e.g. after qgpu_state_reset): no host planning; the packed
// gate data (matrices, phases, conditions) is re-sent host->device on every apply, an async
// copy of a few KB that keeps each apply's inputs flowing like an uncached run.
struct CachedPlan {
  uint64_t key = 0;
  std::vector<int> order;
  std::vector<uint64_t> inv;
  std::vector<Pass> passes;
  std::vector<size_t> off;
  unsigned char* d_blob = nullptr;
  unsigned char* h_blob = nullptr;  // pinned, immutable once packed
  size_t blob_bytes = 0;
  qgpu::QubitMap map_after;
  uint64_t relabels = 0;
  uint64_t last_use = 0;
};
}  // namespace

namespace {

// QGPU_BSTORE: 0 (default) per-thread stores from registers, 1 bulk stores for programs with
// remaps, 2 bulk stores for every tile pass. Measured on B200 (profiles/r01/README.md): bulk
// stores of 1-8 KiB runs are 1.5-1.8x slower than the per-thread stores, so they stay off.
int bstore_mode() {
  static const int v = [] {
    const char* ev = std::getenv("QGPU_BSTORE");
    return ev ? std::atoi(ev) : 0;
  }();
  return v;
}

// host_compress loads: by default the host waits for the slice's store, copies the exact
// compressed size and decodes from device memory; QGPU_HOST_ZC_DECODE=1 (measured slower: the
// decoder reading host memory occupies SMs the concurrent tile passes need) decodes straight
// from pinned host memory without a host wait
bool host_zc_decode() {
  static const bool v = [] {
    const char* ev = std::getenv("QGPU_HOST_ZC_DECODE");
    return ev && std::atoi(ev) != 0;
  }();
  return v;
}

// QGPU_HOST_SWEEP_PER_PASS=1 (ablation): the host tier streams the slices once per pass, as the
// paper traverses every chunk once per gate, instead of once per run of passes
bool host_sweep_per_pass() {
  const char* ev = std::getenv("QGPU_HOST_SWEEP_PER_PASS");  // read per call: ablations flip it
  return ev && std::atoi(ev) != 0;
}

// jit=1: specialise fused passes whose live range is >= 2^jit_min_bits amplitudes
int jit_min_bits() {
  static const int v = [] {
    const char* ev = std::getenv("QGPU_JIT_MIN_BITS");
    return ev ? std::atoi(ev) : 12;
  }();
  return v;
}

thread_local std::string g_err;

qgpu_status fail(qgpu_status s, const char* fmt, ...) {
  static thread_local char buf[1 << 16];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

constexpr int kHostSweep = 100;  // TimedLaunch kind of a host-tier streaming sweep

struct TimedLaunch {
  cudaEvent_t a, b;
  int kind;
  uint64_t bytes;
  int count = 1;  // launches between a and b (a run of consecutive fused passes: one interval)
};

}  // namespace

struct Shard {
  int rank = 0;
  double2* psi = nullptr;
  bool own = false;
};

struct qgpu_state {
  qgpu_config cfg;
  int n = 0, g = 0, m = 0;
  std::vector<Shard> shards;  // 1 per process (NCCL) or world_size (virtual ranks, one GPU)
  bool virt = false;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  double2* psi = nullptr;
  bool own_buf = false;
  uint64_t cap_amps = 0;
  QubitMap map;
  std::vector<uint64_t> trace_order, trace_inv;
  uint64_t gate_counter = 0;
  qgpu_stats stats;
  bool poisoned = false;
  // device op arena (fused tile passes read their ops from here)
  unsigned char* d_ops = nullptr;
  unsigned char* h_ops = nullptr;
  size_t ops_cap = 0;
  cudaEvent_t ops_evt = nullptr;
  // readout scratch
  double* d_scratch = nullptr;
  size_t scratch_cap = 0;  // doubles
  double2* d_zero = nullptr;  // zero amplitudes: source of the expanded region in tile loads
  // timing
  std::vector<TimedLaunch> pending;
  std::vector<cudaEvent_t> event_pool;
  Comm* comm = nullptr;
  std::vector<CachedPlan> plans;  // small LRU (kMaxPlans)
  uint64_t plan_clock = 0;
  // host-memory tier (cfg.host_slice_bits = h > 0, NEXT-2): 2^h slices of 2^m amplitudes in
  // pinned, device-mapped host memory (shards[r].psi = slice r), streamed through device slots
  bool host = false;
  double2* h_state = nullptr;
  std::vector<uint64_t> hlive;       // slice r: amplitudes [0, hlive[r]) valid, the rest zero
  std::vector<double2*> slots;       // device slot buffers, 2^m amplitudes each
  int unit_cap = 0;                  // slices per slot group (slots.size() / groups)
  cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
  cudaEvent_t ev_loaded[2] = {}, ev_computed[2] = {}, ev_stored[2] = {}, ev_join = nullptr;
  bool group_used[2] = {false, false};
  // host_compress: slice r is stored GFC-compressed (hraw[r] = 0) in its own buffer of hcap
  // bytes (raw slices use the same buffer); hoff[r] = its segment offsets (pinned host)
  bool hcomp = false;
  uint32_t hseg = 4096;
  uint64_t hcap = 0, hnseg = 0;
  std::vector<char> hraw;
  std::vector<char> hpoor;              // slice r compressed poorly last time: store it raw
  std::vector<uint64_t*> hoff;
  uint64_t* hoff_base = nullptr;
  // link statistics of compressed transfers: each store also copies its total size into a pinned
  // ring entry; stores and zero-copy loads are counted from the ring at synchronisation points
  uint64_t* hsz = nullptr;
  size_t hsz_n = 0;
  static constexpr size_t kSzRing = 1 << 16;
  std::vector<size_t> store_k;          // slice r: ring entry of its last compressed store
  std::vector<std::pair<size_t, uint64_t>> cnt_d2h, cnt_h2d;  // (ring entry, segments)
  std::vector<uint64_t*> doff, dscan;   // per device slot: offsets, scan scratch
  std::vector<unsigned char*> dstage;   // per device slot: compressed input of a load
  std::vector<cudaEvent_t> ev_slice;   // slice r: its last D2H (host copy valid after it)
  std::vector<uint64_t> slice_seq;     // order of the slices' last D2H (0 = never stored)
  uint64_t store_seq = 0, unit_seq = 0;
  int last_unit = 0;                   // slices per slot group in the previous sweep
  // measurement fused into the last pass (qgpu_apply_circuit_probabilities)
  const Pass* meas_pass = nullptr;     // the pass that accumulates the histogram
  int meas_m = 0;
  int meas_pos[30] = {};
  double* d_meas = nullptr;            // 2^kMeasMax doubles
  bool meas_done = false;
};

namespace {

#define CK(expr)                                                                        \
  do {                                                                                  \
    cudaError_t _e = (expr);                                                            \
    if (_e != cudaSuccess) {                                                            \
      st->poisoned = true;                                                              \
      return fail(QGPU_ERR_CUDA, "%s: %s (%s:%d)", #expr, cudaGetErrorString(_e), __FILE__, \
                  __LINE__);                                                            \
    }                                                                                   \
  } while (0)

#define CK0(expr)                                                                        \
  do {                                                                                   \
    cudaError_t _e = (expr);                                                             \
    if (_e != cudaSuccess)                                                               \
      return fail(QGPU_ERR_CUDA, "%s: %s", #expr, cudaGetErrorString(_e));               \
  } while (0)

cudaEvent_t get_event(qgpu_state* st) {
  if (!st->event_pool.empty()) {
    cudaEvent_t e = st->event_pool.back();
    st->event_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

qgpu_status drain_timing(qgpu_state* st) {
  for (auto& t : st->pending) {
    CK(cudaEventSynchronize(t.b));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, t.a, t.b));
    if (t.kind == PK_SWAP) {
      st->stats.swap_ms += ms;
    } else if (t.kind == kHostSweep) {
      st->stats.host_ms += ms;
    } else {
      st->stats.kernel_ms += ms;
      if (t.kind == PK_TILE) {
        st->stats.tile_kernel_ms += ms;
        st->stats.tile_kernel_launches += uint64_t(t.count);
        st->stats.tile_algo_bytes += t.bytes;
      }
    }
    st->event_pool.push_back(t.a);
    st->event_pool.push_back(t.b);
  }
  st->pending.clear();
  return QGPU_OK;
}

inline uint64_t live(const qgpu_state* st, int k) {
  return st->cfg.prune ? (1ull << k) : (1ull << st->m);
}

void account(qgpu_state* st, uint64_t L_out, uint64_t bytes) {
  qgpu_stats& s = st->stats;
  s.passes++;
  s.amps_processed += L_out;
  s.amps_full += 1ull << st->m;
  const int c = std::min(std::max(st->cfg.chunk_bits, 0), st->m);
  const uint64_t chunk = 1ull << c;
  const uint64_t proc = (L_out + chunk - 1) / chunk;
  s.chunks_processed += proc;
  s.chunks_skipped += (1ull << (st->m - c)) - proc;
  s.algo_bytes += bytes;
}

void sorted_positions(uint64_t mask, int* out, int* n) {
  *n = 0;
  for (; mask; mask &= mask - 1) out[(*n)++] = std::countr_zero(mask);
}

qgpu_status zero_fill(qgpu_state* st, double2* psi, uint64_t from, uint64_t to) {
  if (to > from) CK(cudaMemsetAsync(psi + from, 0, (to - from) * sizeof(double2), st->stream));
  return QGPU_OK;
}

// Global-local swap (a10): exchange rank bit (swap_global - m) with local position swap_local,
// one pair at a time. Virtual ranks: in-device swap of the two halves; NCCL: pack, send/recv with
// the partner rank in slabs through bounded staging, unpack (in place: the received half lands
// in the slots of the half that was sent).
qgpu_status exec_swap(qgpu_state* st, const Pass& p, uint64_t* bytes) {
  const int m = st->m;
  const uint64_t half = 1ull << (m - 1);
  const uint64_t active = 1ull << p.kg;
  for (int i = 0; i < p.nswap; ++i) {
    const int j = p.swap_global[i] - m, lp = p.swap_local[i];
    if (st->virt) {
      for (Shard& sh : st->shards) {
        const uint64_t r = uint64_t(sh.rank);
        if (r >= active || (r >> j & 1)) continue;
        const uint64_t partner = r | (1ull << j);
        CK(launch_swap_halves(st->stream, sh.psi, st->shards[partner].psi, lp, half));
        st->stats.kernels_launched++;
      }
    } else {
      for (Shard& sh : st->shards) {
        if (uint64_t(sh.rank) >= active) continue;
        qgpu_status s = comm_swap_bit(st->comm, sh.psi, m, sh.rank, j, lp, st->stream, &g_err);
        if (s) {
          st->poisoned = true;
          return s;
        }
      }
    }
    *bytes += 16 * half;
    st->stats.swaps++;
    st->stats.swap_bytes += 16 * half;
  }
  return QGPU_OK;
}

// Execute one compute pass (tile / pair / quad / diag) on one rank's local buffer.
qgpu_status exec_compute(qgpu_state* st, const Pass& p, const unsigned char* d_ops, double2* psi,
                         uint64_t rank, uint64_t* bytes_out) {
  const int m = st->m;
  const uint64_t lmask = (m >= 64) ? ~0ull : ((1ull << m) - 1);
  const int kin = st->cfg.prune ? p.k_in : m, kout = st->cfg.prune ? p.k_out : m;
  const uint64_t L_in = 1ull << kin, L_out = 1ull << kout;
  uint64_t bytes = 0;
  if (p.kind == PK_TILE) {
    TileArgs a{};
    a.psi = psi;
    const TileProgram& P = p.prog;
    a.blob = d_ops;
    a.blob_bytes = int(P.bytes);
    a.nops = int(P.ops.size());
    a.npat = int(P.patterns.size());
    a.nscalar = int(P.scalar.size());
    a.spat = P.spat;
    a.lb = P.lb;
    a.off_tlo = int(P.off_tlo);
    a.off_entries = int(P.off_entries);
    a.off_patterns = int(P.off_patterns);
    a.off_terms = int(P.off_terms);
    a.off_scalar = int(P.off_scalar);
    a.off_pool = int(P.off_pool);
    a.nr = P.nr;
    a.nw = P.nw;
    a.b = p.b;
    a.l = p.l;
    for (int i = 0; i < p.b; ++i) a.spos[i] = p.spos[i];
    a.nsrun = 0;
    for (int i = 0; i < p.b;) {
      int j = i;
      while (j + 1 < p.b && p.spos[j + 1] == p.spos[j] + 1) ++j;
      a.srun_pos[a.nsrun] = p.spos[i];
      a.srun_len[a.nsrun] = j - i + 1;
      a.nsrun++;
      i = j + 1;
    }
    a.ntiles = 1ull << (kout - p.b);
    a.L_in = L_in;
    a.zin = st->cfg.prune ? p.zin : 0;
    a.zout = st->cfg.prune ? p.zout : 0;
    a.rank_base = rank << m;
    a.zero = st->d_zero;
    a.remaps = 0;
    a.nmbar = 0;
    for (size_t i = 1; i < P.ops.size(); ++i) {
      if (P.ops[i].kind == OP_REMAP || P.ops[i].kind == OP_SMEM1 || P.ops[i].kind == OP_SMEM2) a.remaps = 1;
      if (P.ops[i].kind == OP_REMAP) a.nmbar += 1 << P.nw;  // one per warp group of each remap
    }
    // programs without remaps need one tile buffer (each thread only reads its own slots),
    // which lets two CTAs share an SM; otherwise triple (or double) buffering
    a.nbuf = a.remaps ? 3 : 1;
    // optional bulk stores (staged tile, async copies per run; QGPU_BSTORE)
    const int bs = bstore_mode();
    if (bs == 2 || (bs == 1 && a.remaps)) a.nbuf = 3;
    if (tile_smem_bytes(a) > 227 * 1024) a.nbuf = 2;
    a.bstore = (a.nbuf == 3 && (bs == 2 || (bs == 1 && a.remaps))) ? 1 : 0;
    if (st->meas_pass == &p && !a.bstore) {  // fused measurement, if its histogram fits in smem
      TileArgs h = a;
      h.hist = st->d_meas;
      h.hm = st->meas_m;
      for (int j = 0; j < st->meas_m; ++j) h.hpos[j] = st->meas_pos[j];
      if (tile_smem_bytes(h) > 227 * 1024 && h.nbuf == 3) h.nbuf = 2;  // make room: double buffering
      if (tile_smem_bytes(h) <= 227 * 1024) {
        a = h;
        st->meas_done = true;
      }
    }
    const int jit = st->cfg.jit;
    cudaError_t e = cudaErrorNotSupported;
    if (jit == 2 || (jit == 1 && p.k_out >= jit_min_bits())) {
      double ms = 0;
      e = launch_tile_jit(st->stream, p, a, tile_smem_bytes(a), device_num_sms(), &ms);
      if (e == cudaSuccess) st->stats.jit_launches++;
      st->stats.jit_ms += ms;
    }
    if (e == cudaErrorNotSupported) e = launch_tile(st->stream, a);
    CK(e);
    st->stats.kernels_launched++;
    // live input / output amplitudes: a skipped zero position halves the part that moves
    bytes = 16 * ((L_in >> std::popcount(a.zin & (L_in - 1))) + (L_out >> std::popcount(a.zout & (L_out - 1))));
  } else if (p.kind == PK_ZERO) {
    CK(launch_zero_where(st->stream, psi, L_out, p.zmask));
    st->stats.kernels_launched++;
    bytes = 16 * (L_out - (L_out >> std::popcount(p.zmask & (L_out - 1))));
  } else {
    PhysGate g = p.gates[0];
    int kind = p.kind;
    const uint64_t gpc = g.pc & ~lmask;                  // controls on rank bits
    const bool rank_ok = ((rank << m) & gpc) == gpc;
    uint64_t lc = g.pc & lmask;
    // Sector-dense form: a control on position 0 makes the pair kernel touch every other 16-byte
    // amplitude, i.e. half of every 32-byte sector, so DRAM moves the whole sector anyway. Folded
    // into the targets (a 2-qubit gate, identity where the control is 0), whole sectors are read
    // and written by one coalesced stream: CX(control 0) 2.1 -> 2.75 TB/s algorithmic. (Controls
    // or diagonal bits on positions 1..2 keep the enumerating kernels: they skip whole sectors,
    // and folding them was measured slower.)
    const int kfull = st->cfg.prune ? kin : m;
    if (kind == PK_PAIR && (lc & 1) && kfull >= 2 && g.p[0] < kfull) {
      cplx U4[16];
      for (int r = 0; r < 4; ++r)
        for (int col = 0; col < 4; ++col) {
          const int r0 = r & 1, r1 = r >> 1, c0 = col & 1, c1 = col >> 1;
          U4[r * 4 + col] = (r1 != c1) ? cplx{0, 0} : (r1 == 0 ? cplx{r0 == c0 ? 1.0 : 0.0, 0} : g.U[r0 * 2 + c0]);
        }
      std::memcpy(g.U, U4, sizeof(U4));
      g.nt = 2;
      g.p[1] = 0;
      lc &= ~1ull;
      kind = PK_QUAD;
    }
    if (!rank_ok) {
      // identity on this rank; the expanded region still has to read as zero
      qgpu_status s = zero_fill(st, psi, L_in, L_out);
      if (s) return s;
      bytes = 16 * (L_out - L_in);
    } else if (kind == PK_PAIR || kind == PK_QUAD) {
      const bool full = g.expands_target || !st->cfg.prune;
      const int krun = full ? kout : kin;
      // the kernel writes only the pairs whose controls are satisfied: the rest of an expanded
      // region [L_in, L_out) must be written as zeros here (the buffer may hold stale data
      // from before a reset, or another slice's in a host-tier slot)
      const bool zero_new = !full || (lc != 0 && L_out > L_in);
      if (zero_new) {
        qgpu_status s = zero_fill(st, psi, L_in, L_out);
        if (s) return s;
      }
      const int nlc = std::popcount(lc);
      const bool ctl_in_range = (lc >> krun) == 0;
      if (kind == PK_PAIR) {
        PairArgs a{};
        a.psi = psi;
        for (int i = 0; i < 4; ++i) a.u[i] = make_double2(g.U[i].re, g.U[i].im);
        a.t = g.p[0];
        sorted_positions(lc | (1ull << g.p[0]), a.ins, &a.nins);
        sorted_positions(lc, a.ins_c, &a.nins_c);
        a.cset = lc;
        a.npairs = ctl_in_range ? (1ull << (krun - 1 - nlc)) : 0;
        a.L_in = L_in;
        const bool shfl = g.p[0] < 5 && krun >= 5 && (lc & 31) == 0;
        CK(launch_pair(st->stream, a, shfl));
        bytes = 32 * a.npairs + (zero_new ? 16 * (L_out - L_in) : 0);
      } else {
        QuadArgs a{};
        a.psi = psi;
        for (int i = 0; i < 16; ++i) a.u[i] = make_double2(g.U[i].re, g.U[i].im);
        a.t0 = g.p[0];
        a.t1 = g.p[1];
        sorted_positions(lc | (1ull << g.p[0]) | (1ull << g.p[1]), a.ins, &a.nins);
        a.cset = lc;
        a.nquads = ctl_in_range ? (1ull << (krun - 2 - nlc)) : 0;
        a.L_in = L_in;
        CK(launch_quad(st->stream, a));
        bytes = 64 * a.nquads + (zero_new ? 16 * (L_out - L_in) : 0);
      }
      st->stats.kernels_launched++;
    } else {  // PK_DIAG: the expanded region stays zero under a diagonal gate
      qgpu_status s = zero_fill(st, psi, L_in, L_out);
      if (s) return s;
      PhaseArgs a{};
      a.psi = psi;
      // targets on rank bits are fixed by this rank: keep the entries that match them
      int lt[2], nlt = 0, gfix = 0, gsel = 0;
      for (int j = 0; j < g.nt; ++j) {
        if (g.p[j] >= m) {
          gsel |= 1 << j;
          if ((rank >> (g.p[j] - m)) & 1) gfix |= 1 << j;
        } else {
          lt[nlt++] = j;
        }
      }
      a.nt = nlt;
      a.t0 = nlt > 0 ? g.p[lt[0]] : 0;
      a.t1 = nlt > 1 ? g.p[lt[1]] : 0;
      const int dim = 1 << g.nt;
      int n_not1 = 0, which = 0;
      for (int w = 0; w < (1 << nlt); ++w) {
        int v = gfix;
        for (int q = 0; q < nlt; ++q)
          if (w >> q & 1) v |= 1 << lt[q];
        const cplx d = g.U[v * (dim + 1)];
        a.d[w] = make_double2(d.re, d.im);
        if (!(d.re == 1.0 && d.im == 0.0)) { ++n_not1; which = w; }
      }
      (void)gsel;
      uint64_t fixed = lc, insmask = lc;
      if (n_not1 == 1) {
        for (int q = 0; q < nlt; ++q) {
          insmask |= 1ull << g.p[lt[q]];
          if (which >> q & 1) fixed |= 1ull << g.p[lt[q]];
        }
      }
      a.fixed = fixed;
      sorted_positions(insmask, a.ins, &a.nins);
      const bool in_range = (insmask >> kin) == 0;
      a.count = (n_not1 == 0 || !in_range) ? 0 : (1ull << (kin - a.nins));
      CK(launch_phase(st->stream, a));
      st->stats.kernels_launched++;
      bytes = 32 * a.count + 16 * (L_out - L_in);
    }
  }
  *bytes_out = bytes;
  return QGPU_OK;
}

// Execute one planned pass: compute passes on every active local shard (ranks >= 2^kg hold
// only zeros and skip the work), swaps through the communicator, activations as memsets.
qgpu_status exec_pass(qgpu_state* st, const Pass& p, const unsigned char* d_ops, bool own_timing = true,
                      uint64_t* bytes_out = nullptr) {
  const int m = st->m;
  const int kin = st->cfg.prune ? p.k_in : m, kout = st->cfg.prune ? p.k_out : m;
  const uint64_t L_in = 1ull << kin, L_out = 1ull << kout;
  const uint64_t active = 1ull << p.kg;
  if (p.kind == PK_RELABEL) {
    if (kout > kin) {
      for (Shard& sh : st->shards)
        if (uint64_t(sh.rank) < active) {
          qgpu_status s = zero_fill(st, sh.psi, L_in, L_out);
          if (s) return s;
        }
      st->stats.kernels_launched++;
      account(st, L_out, 16 * (L_out - L_in));
    }
    return QGPU_OK;
  }
  if (p.kind == PK_ACTIVATE) {
    for (Shard& sh : st->shards)
      if (uint64_t(sh.rank) >= (1ull << p.kg_from) && uint64_t(sh.rank) < active) {
        qgpu_status s = zero_fill(st, sh.psi, 0, 1ull << m);
        if (s) return s;
      }
    return QGPU_OK;
  }
  const bool timing = st->cfg.timing != 0 && own_timing;
  TimedLaunch tl{};
  if (timing) {
    tl.a = get_event(st);
    tl.b = get_event(st);
    tl.kind = p.kind;
    CK(cudaEventRecord(tl.a, st->stream));
  }
  uint64_t bytes = 0;
  if (p.kind == PK_SWAP) {
    qgpu_status s = exec_swap(st, p, &bytes);
    if (s) return s;
  } else {
    bool first = true;
    for (Shard& sh : st->shards) {
      if (uint64_t(sh.rank) >= active) continue;
      uint64_t b = 0;
      qgpu_status s = exec_compute(st, p, d_ops, sh.psi, uint64_t(sh.rank), &b);
      if (s) return s;
      if (first) bytes = b;
      first = false;
    }
  }
  if (timing) {
    CK(cudaEventRecord(tl.b, st->stream));
    tl.bytes = bytes;
    st->pending.push_back(tl);
  }
  if (p.kind != PK_SWAP) {
    account(st, L_out, bytes);
    st->stats.unfused_bytes += p.unfused_bytes;
  }
  if (bytes_out) *bytes_out = bytes;
  return QGPU_OK;
}

// ------------------------------------------------------------ host-memory tier (NEXT-2)
// The paper keeps the state in host memory and moves chunks to the GPU and back for every
// gate, overlapping the transfers on two streams and skipping all-zero chunks
// (Alg.1). B200 form: the circuit is planned for 2^h virtual ranks (slice index = the
// top h physical bits), so between two global-local swaps every pass works on one slice at a
// time. Such a run of passes becomes ONE streaming sweep over the active slices: per unit of
// slices, H2D of their live prefixes (s_h2d), every pass of the run (the state's stream), D2H
// (s_d2h); two slot groups let the copies of one unit overlap the compute of the other. A swap
// is folded into the next sweep: a unit is the set of slices that differ in the swapped rank
// bits, exchanged on the device right after loading. Never-active slices (all zero) are
// skipped, and only the live prefix [0, 2^kl) of a slice crosses the link.

struct HostSwap {
  int j, lp;  // rank bit j <-> local position lp
};

// Ensure two groups of `unit` device slots (one group if memory runs out).
qgpu_status ensure_slots(qgpu_state* st, int unit, int* ngroups) {
  const size_t bytes = (size_t(1) << st->m) * sizeof(double2);
  while (st->slots.size() < size_t(2 * unit)) {
    double2* p = nullptr;
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      if (st->slots.size() >= size_t(unit)) break;
      return fail(QGPU_ERR_OUT_OF_MEMORY, "host tier: cudaMalloc of a %llu-byte slot: %s",
                  (unsigned long long)bytes, cudaGetErrorString(e));
    }
    st->slots.push_back(p);
    if (st->hcomp) {
      uint64_t* o = nullptr;
      uint64_t* sc = nullptr;
      unsigned char* stg = nullptr;
      cudaError_t e2 = cudaMalloc(&o, (st->hnseg + 1) * sizeof(uint64_t));
      if (e2 == cudaSuccess) e2 = cudaMalloc(&sc, std::max<uint64_t>(1, gfc_scan_scratch_elems(st->hnseg)) * sizeof(uint64_t));
      if (e2 == cudaSuccess) e2 = cudaMalloc(&stg, st->hcap);
      if (e2 != cudaSuccess) {
        cudaGetLastError();
        return fail(QGPU_ERR_OUT_OF_MEMORY, "host tier: compression scratch: %s", cudaGetErrorString(e2));
      }
      st->doff.push_back(o);
      st->dscan.push_back(sc);
      st->dstage.push_back(stg);
    }
  }
  *ngroups = st->slots.size() >= size_t(2 * unit) ? 2 : 1;
  return QGPU_OK;
}

// Load slice r (its valid prefix hlive[r]; raw or GFC-compressed) into device buffer `dst` on
// stream `s`, zero-filling [hlive, need). Compressed: the host waits for the slice's last store
// (its size is data dependent), copies the compressed bytes and offsets, decodes on the device.
qgpu_status host_load_slice(qgpu_state* st, uint64_t r, double2* dst, size_t slot, uint64_t need, cudaStream_t s) {
  const uint64_t have = st->hlive[r];
  const uint64_t copy = std::max(std::min(have, need), st->hcomp && !st->hraw[r] ? have : 0);
  if (copy && (!st->hcomp || st->hraw[r])) {
    CK(cudaMemcpyAsync(dst, st->shards[r].psi, copy * sizeof(double2), cudaMemcpyHostToDevice, s));
    st->stats.host_h2d_bytes += copy * sizeof(double2);
    st->stats.h2d_bytes += copy * sizeof(double2);
  } else if (copy) {
    const uint64_t nd = 2 * copy, ns = (nd + st->hseg - 1) / st->hseg;
    if (host_zc_decode()) {
      // zero-copy: the decoder reads the compressed stream and its offsets straight from pinned
      // host memory; only a stream dependency on the slice's last store, no host wait
      CK(cudaStreamWaitEvent(s, st->ev_slice[r], 0));
      CK(launch_gfc_decode(s, st->shards[r].psi, st->hoff[r], nd, st->hseg, reinterpret_cast<double*>(dst)));
      st->stats.kernels_launched++;
      st->cnt_h2d.push_back({st->store_k[r], ns});  // bytes counted at the next sync point
    } else {
      CK(cudaEventSynchronize(st->ev_slice[r]));
      const uint64_t total = st->hoff[r][ns];
      // adaptive: a slice that did not shrink by a quarter is stored raw from now on (dense
      // amplitudes have incompressible bit patterns; compression would only add passes)
      if (4 * total > 3 * nd * sizeof(double)) st->hpoor[r] = 1;
      CK(cudaMemcpyAsync(st->dstage[slot], st->shards[r].psi, total, cudaMemcpyHostToDevice, s));
      CK(cudaMemcpyAsync(st->doff[slot], st->hoff[r], (ns + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice, s));
      CK(launch_gfc_decode(s, st->dstage[slot], st->doff[slot], nd, st->hseg, reinterpret_cast<double*>(dst)));
      st->stats.kernels_launched++;
      st->stats.host_h2d_bytes += total + (ns + 1) * sizeof(uint64_t);
      st->stats.h2d_bytes += total + (ns + 1) * sizeof(uint64_t);
    }
  }
  if (need > copy) CK(cudaMemsetAsync(dst + copy, 0, (need - copy) * sizeof(double2), s));
  return QGPU_OK;
}

void host_account_stores(qgpu_state* st);

// Store the prefix [0, L) of device buffer `src` as slice r on stream `s` (after its compute).
// Compressed: size pass, scan, then the encoder writes the stream straight into the slice's
// pinned host buffer (zero-copy, so no host round trip for the data-dependent size); the
// offsets follow with one D2H copy.
qgpu_status host_store_slice(qgpu_state* st, uint64_t r, const double2* src, size_t slot, uint64_t L, cudaStream_t s) {
  if (!st->hcomp || st->hpoor[r]) {
    if (st->hcomp) st->hraw[r] = 1;
    CK(cudaMemcpyAsync(st->shards[r].psi, src, L * sizeof(double2), cudaMemcpyDeviceToHost, s));
    st->stats.host_d2h_bytes += L * sizeof(double2);
    st->stats.d2h_bytes += L * sizeof(double2);
  } else if (L) {
    const uint64_t nd = 2 * L, ns = (nd + st->hseg - 1) / st->hseg;
    if (st->hsz_n == qgpu_state::kSzRing) {  // ring full: count what it holds first
      CK(cudaStreamSynchronize(s));
      host_account_stores(st);
    }
    const double* in = reinterpret_cast<const double*>(src);
    CK(cudaMemsetAsync(st->doff[slot], 0, sizeof(uint64_t), s));
    CK(launch_gfc_sizes(s, in, nd, st->hseg, st->doff[slot] + 1));
    CK(launch_scan_u64(s, st->doff[slot] + 1, ns, st->dscan[slot]));
    CK(launch_gfc_encode(s, in, nd, st->hseg, st->doff[slot], st->shards[r].psi));
    CK(cudaMemcpyAsync(st->hoff[r], st->doff[slot], (ns + 1) * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    const size_t k = st->hsz_n++;
    CK(cudaMemcpyAsync(st->hsz + k, st->doff[slot] + ns, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    st->store_k[r] = k;
    st->cnt_d2h.push_back({k, ns});
    st->stats.kernels_launched += 3;
    st->hraw[r] = 0;
  }
  st->hlive[r] = L;
  return QGPU_OK;
}

// Readout of slice r: raw slices are read in place (zero-copy); a compressed one is decoded into
// device slot 0 first (on the state's stream, so the next slice waits for this readout)
qgpu_status host_readable(qgpu_state* st, size_t r, const double2** psi) {
  if (!st->host || !st->hcomp || st->hraw[r] || !st->hlive[r]) return QGPU_OK;
  int ng = 1;
  if (qgpu_status s = ensure_slots(st, 1, &ng)) return s;
  if (qgpu_status s = host_load_slice(st, r, st->slots[0], 0, st->hlive[r], st->stream)) return s;
  *psi = st->slots[0];
  return QGPU_OK;
}

// host_compress: add the compressed bytes of stores and zero-copy loads to the link statistics
// (the ring entries are final once s_d2h has drained: callers synchronise it first)
void host_account_stores(qgpu_state* st) {
  if (!st->hcomp) return;
  for (auto [k, ns] : st->cnt_d2h) {
    const uint64_t b = st->hsz[k] + (ns + 1) * sizeof(uint64_t);
    st->stats.host_d2h_bytes += b;
    st->stats.d2h_bytes += b;
  }
  for (auto [k, ns] : st->cnt_h2d) {
    const uint64_t b = st->hsz[k] + (ns + 1) * sizeof(uint64_t);
    st->stats.host_h2d_bytes += b;
    st->stats.h2d_bytes += b;
  }
  st->cnt_d2h.clear();
  st->cnt_h2d.clear();
  // ring entries still referenced by slices are kept: compact them to the front
  std::vector<std::pair<size_t, size_t>> keep;  // (old k, slice)
  for (size_t r = 0; r < st->store_k.size(); ++r)
    if (!st->hraw[r]) keep.push_back({st->store_k[r], r});
  std::sort(keep.begin(), keep.end());
  size_t nk = 0, last = ~size_t(0);
  for (auto [k, r] : keep) {
    if (k != last) {
      st->hsz[nk++] = st->hsz[k];
      last = k;
    }
    st->store_k[r] = nk - 1;
  }
  st->hsz_n = nk;
}

// One streaming sweep: swaps `sw` (made while 2^kg_sw ranks were active), then the passes `run`.
qgpu_status host_sweep(qgpu_state* st, const std::vector<const Pass*>& run,
                       const std::vector<const unsigned char*>& ops, const std::vector<HostSwap>& sw,
                       int kg_sw) {
  const int m = st->m;
  const uint64_t full = 1ull << m;
  int kg = sw.empty() ? 0 : kg_sw;
  for (const Pass* p : run) kg = std::max(kg, p->kg);
  const uint64_t nact = 1ull << kg;
  int ubit[8], nub = 0;
  uint64_t ubits = 0;
  for (const HostSwap& x : sw)
    if (!(ubits >> x.j & 1)) {
      ubits |= 1ull << x.j;
      ubit[nub++] = x.j;
    }
  const int unit = 1 << nub;
  int ngroups = 1;
  if (qgpu_status s = ensure_slots(st, unit, &ngroups)) return s;
  // earlier work on the state's stream (reset, readout, the previous sweep's compute); the
  // previous sweep's stores are waited for per slice and per slot group below, so this sweep's
  // first loads overlap the previous sweep's last stores
  CK(cudaEventRecord(st->ev_join, st->stream));
  CK(cudaStreamWaitEvent(st->s_h2d, st->ev_join, 0));
  if (unit != st->last_unit) {  // the slot groups are re-cut: drain every earlier store
    for (int gi = 0; gi < 2; ++gi)
      if (st->group_used[gi]) CK(cudaStreamWaitEvent(st->s_h2d, st->ev_stored[gi], 0));
    st->last_unit = unit;
  }
  const bool timing = st->cfg.timing != 0;
  const uint64_t L_end = run.empty() ? full : live(st, run.back()->k_out);
  std::vector<char> accounted(run.size(), 0);
  auto unit_slice = [&](uint64_t base, int x) {
    uint64_t r = base;
    for (int i = 0; i < nub; ++i)
      if (x >> i & 1) r |= 1ull << ubit[i];
    return r;
  };
  // units in the order their slices were last stored (earliest first): the first loads of this
  // sweep need only the previous sweep's first stores
  std::vector<std::pair<uint64_t, uint64_t>> units;  // (latest store among the unit's slices, base)
  for (uint64_t base = 0; base < nact; ++base) {
    if (base & ubits) continue;
    uint64_t last = 0;
    for (int x = 0; x < unit; ++x) last = std::max(last, st->slice_seq[unit_slice(base, x)]);
    units.emplace_back(last, base);
  }
  std::stable_sort(units.begin(), units.end(),
                   [](const auto& a, const auto& b) { return a.first < b.first; });
  for (const auto& ub : units) {
    const uint64_t base = ub.second;
    const int gi = (ngroups == 2) ? int(st->unit_seq & 1) : 0;
    ++st->unit_seq;
    double2** slot = &st->slots[size_t(gi) * size_t(unit)];
    uint64_t rs[1 << 8];
    for (int x = 0; x < unit; ++x) rs[x] = unit_slice(base, x);
    const bool swap_here = !sw.empty() && base < (1ull << kg_sw);
    // load: the live prefix from host memory, zeros up to what the first pass reads; the slot
    // group must be drained and each slice's previous store complete
    if (st->group_used[gi]) CK(cudaStreamWaitEvent(st->s_h2d, st->ev_stored[gi], 0));
    for (int x = 0; x < unit; ++x)
      if (st->slice_seq[rs[x]]) CK(cudaStreamWaitEvent(st->s_h2d, st->ev_slice[rs[x]], 0));
    for (int x = 0; x < unit; ++x) {
      const uint64_t r = rs[x];
      uint64_t need = 0;
      if (swap_here) {
        need = full;
      } else {
        for (const Pass* p : run)
          if (r < (1ull << p->kg)) {
            need = live(st, p->k_in);
            break;
          }
      }
      if (qgpu_status s = host_load_slice(st, r, slot[x], size_t(gi) * size_t(unit) + size_t(x), need, st->s_h2d))
        return s;
      st->stats.host_slice_loads++;
    }
    CK(cudaEventRecord(st->ev_loaded[gi], st->s_h2d));
    // compute: swaps, then every pass of the run on every slice active at that pass
    CK(cudaStreamWaitEvent(st->stream, st->ev_loaded[gi], 0));
    if (swap_here) {
      for (const HostSwap& x : sw) {
        int bi = 0;
        while (ubit[bi] != x.j) ++bi;
        for (int xi = 0; xi < unit; ++xi) {
          if (xi >> bi & 1) continue;
          CK(launch_swap_halves(st->stream, slot[xi], slot[xi | (1 << bi)], x.lp, full / 2));
          st->stats.kernels_launched++;
        }
      }
    }
    for (size_t i = 0; i < run.size(); ++i) {
      const Pass& p = *run[i];
      const uint64_t L_in = live(st, p.k_in), L_out = live(st, p.k_out);
      for (int x = 0; x < unit; ++x) {
        const uint64_t r = rs[x];
        if (r >= (1ull << p.kg)) continue;
        uint64_t b = 0;
        if (p.kind == PK_RELABEL) {
          if (L_out <= L_in) continue;
          if (qgpu_status s = zero_fill(st, slot[x], L_in, L_out)) return s;
          st->stats.kernels_launched++;
          b = 16 * (L_out - L_in);
        } else {
          TimedLaunch tl{};
          if (timing) {
            tl.a = get_event(st);
            tl.b = get_event(st);
            tl.kind = p.kind;
            CK(cudaEventRecord(tl.a, st->stream));
          }
          if (qgpu_status s = exec_compute(st, p, ops[i], slot[x], r, &b)) return s;
          if (timing) {
            CK(cudaEventRecord(tl.b, st->stream));
            tl.bytes = b;
            st->pending.push_back(tl);
          }
        }
        if (!accounted[i]) {
          accounted[i] = 1;
          account(st, L_out, b);
          st->stats.unfused_bytes += p.unfused_bytes;
        }
      }
    }
    CK(cudaEventRecord(st->ev_computed[gi], st->stream));
    // store the live prefix back
    CK(cudaStreamWaitEvent(st->s_d2h, st->ev_computed[gi], 0));
    for (int x = 0; x < unit; ++x) {
      const uint64_t r = rs[x];
      if (qgpu_status s = host_store_slice(st, r, slot[x], size_t(gi) * size_t(unit) + size_t(x), L_end, st->s_d2h))
        return s;
      CK(cudaEventRecord(st->ev_slice[r], st->s_d2h));
      st->slice_seq[r] = ++st->store_seq;
    }
    CK(cudaEventRecord(st->ev_stored[gi], st->s_d2h));
    st->group_used[gi] = true;
  }
  st->stats.host_slice_skips += (1ull << st->g) - nact;
  for (const HostSwap& x : sw) {
    (void)x;
    st->stats.swaps++;
    st->stats.swap_bytes += 16 * (full / 2) * (nact >> 1);
  }
  st->stats.host_runs++;
  return QGPU_OK;
}

// Later work on the state's stream (readout, host writes after a sync) sees the stored slices.
qgpu_status host_join(qgpu_state* st) {
  CK(cudaEventRecord(st->ev_join, st->s_d2h));
  CK(cudaStreamWaitEvent(st->stream, st->ev_join, 0));
  return QGPU_OK;
}

// Execute planned passes: resident state pass by pass; host tier as streaming sweeps, one per
// run of passes between global-local swaps (consecutive swaps join one sweep, <= 2 rank bits).
qgpu_status exec_passes(qgpu_state* st, const std::vector<Pass>& passes,
                        const std::vector<const unsigned char*>& ops) {
  if (!st->host) {
    // timing=1: a run of consecutive fused passes on one shard is timed as ONE event interval
    // (events between back-to-back kernels cost a launch gap each); the interval's launches and
    // algorithmic bytes are recorded with it
    const bool group = st->cfg.timing != 0 && st->shards.size() == 1;
    TimedLaunch grp{};
    bool open = false;
    auto close_group = [&]() -> qgpu_status {
      if (!open) return QGPU_OK;
      CK(cudaEventRecord(grp.b, st->stream));
      st->pending.push_back(grp);
      open = false;
      return QGPU_OK;
    };
    for (size_t i = 0; i < passes.size(); ++i) {
      const Pass& p = passes[i];
      if (group && p.kind == PK_TILE) {
        if (!open) {
          grp = TimedLaunch{};
          grp.a = get_event(st);
          grp.b = get_event(st);
          grp.kind = PK_TILE;
          grp.count = 0;
          CK(cudaEventRecord(grp.a, st->stream));
          open = true;
        }
        uint64_t b = 0;
        if (qgpu_status s = exec_pass(st, p, ops[i], false, &b)) return s;
        grp.bytes += b;
        grp.count++;
        continue;
      }
      if (qgpu_status s = close_group()) return s;
      if (qgpu_status s = exec_pass(st, p, ops[i])) return s;
    }
    return close_group();
  }
  std::vector<const Pass*> run;
  std::vector<const unsigned char*> run_ops;
  std::vector<HostSwap> sw;
  int kg_sw = 0;
  // timing=1: one interval from the first load to the last store (sweeps overlap)
  TimedLaunch span{};
  if (st->cfg.timing) {
    span.a = get_event(st);
    span.b = get_event(st);
    span.kind = kHostSweep;
    CK(cudaEventRecord(span.a, st->stream));
  }
  auto flush = [&]() -> qgpu_status {
    if (run.empty() && sw.empty()) return QGPU_OK;
    qgpu_status s = host_sweep(st, run, run_ops, sw, kg_sw);
    run.clear();
    run_ops.clear();
    sw.clear();
    return s;
  };
  for (size_t i = 0; i < passes.size(); ++i) {
    const Pass& p = passes[i];
    if (p.kind == PK_ACTIVATE) continue;  // newly active slices are all zero (hlive = 0)
    if (p.kind == PK_SWAP) {
      if (!run.empty())
        if (qgpu_status s = flush()) return s;
      uint64_t bits = 0;
      for (const HostSwap& x : sw) bits |= 1ull << x.j;
      for (int k = 0; k < p.nswap; ++k) bits |= 1ull << (p.swap_global[k] - st->m);
      if (std::popcount(bits) > 2)
        if (qgpu_status s = flush()) return s;
      for (int k = 0; k < p.nswap; ++k) sw.push_back(HostSwap{p.swap_global[k] - st->m, p.swap_local[k]});
      kg_sw = p.kg;
      continue;
    }
    run.push_back(&p);
    run_ops.push_back(ops[i]);
    if (host_sweep_per_pass())
      if (qgpu_status s = flush()) return s;
  }
  if (qgpu_status s = flush()) return s;
  if (qgpu_status s = host_join(st)) return s;
  if (st->cfg.timing) {
    CK(cudaEventRecord(span.b, st->stream));
    st->pending.push_back(span);
  }
  return QGPU_OK;
}

qgpu_status ensure_ops(qgpu_state* st, size_t n) {
  if (n <= st->ops_cap) return QGPU_OK;
  size_t cap = std::max<size_t>(n, 2 * st->ops_cap);
  cap = std::max<size_t>(cap, 1 << 16);
  CK(cudaStreamSynchronize(st->stream));
  if (st->d_ops) CK(cudaFree(st->d_ops));
  if (st->h_ops) CK(cudaFreeHost(st->h_ops));
  st->d_ops = nullptr;
  st->h_ops = nullptr;
  CK(cudaMalloc(&st->d_ops, cap));
  CK(cudaMallocHost(&st->h_ops, cap));
  st->ops_cap = cap;
  return QGPU_OK;
}

void prepare_jit(qgpu_state* st, const std::vector<Pass>& passes);

qgpu_status run_plan(qgpu_state* st, const std::vector<Pass>& passes) {
  size_t nbytes = 0;
  std::vector<size_t> off(passes.size(), 0);
  for (size_t i = 0; i < passes.size(); ++i) {
    off[i] = nbytes;
    if (passes[i].kind == PK_TILE) nbytes += (passes[i].prog.bytes + 15) / 16 * 16;
  }
  if (nbytes) {
    qgpu_status s = ensure_ops(st, nbytes);
    if (s) return s;
    // the pinned staging buffer may still be read by the previous upload
    CK(cudaEventSynchronize(st->ops_evt));
    for (size_t i = 0; i < passes.size(); ++i)
      if (passes[i].kind == PK_TILE) passes[i].prog.pack(st->h_ops + off[i]);
    CK(cudaMemcpyAsync(st->d_ops, st->h_ops, nbytes, cudaMemcpyHostToDevice, st->stream));
    st->stats.h2d_bytes += nbytes;
    CK(cudaEventRecord(st->ops_evt, st->stream));
  }
  prepare_jit(st, passes);
  std::vector<const unsigned char*> ops(passes.size());
  for (size_t i = 0; i < passes.size(); ++i) ops[i] = st->d_ops + off[i];
  return exec_passes(st, passes, ops);
}

void record_trace(qgpu_state* st, const std::vector<int>& order, const std::vector<uint64_t>& inv,
                  uint64_t base) {
  const uint64_t full = (st->n >= 64) ? ~0ull : ((1ull << st->n) - 1);
  for (size_t k = 0; k < order.size(); ++k) {
    if (st->stats.ops_before_full_involvement < 0 && inv[k] == full)
      st->stats.ops_before_full_involvement = int64_t(st->trace_order.size());
    st->trace_order.push_back(base + uint64_t(order[k]));
    st->trace_inv.push_back(inv[k]);
  }
  st->stats.gates_applied += order.size();
}

qgpu_status check_state(qgpu_state* st) {
  if (!st) return fail(QGPU_ERR_INVALID_ARG, "state is NULL");
  if (st->poisoned) return fail(QGPU_ERR_STATE, "state poisoned by an earlier CUDA/NCCL failure");
  return QGPU_OK;
}

qgpu_status init_amplitudes(qgpu_state* st) {
  if (st->host) {
    // host tier: |0...0> = slice 0 holds psi[0] = 1, every other amplitude reads as zero
    // through hlive (the host pages beyond hlive are never read)
    CK(cudaStreamSynchronize(st->stream));
    CK(cudaStreamSynchronize(st->s_d2h));
    host_account_stores(st);
    st->shards[0].psi[0] = make_double2(1.0, 0.0);
    std::fill(st->hlive.begin(), st->hlive.end(), 0);
    std::fill(st->hraw.begin(), st->hraw.end(), 1);
    std::fill(st->hpoor.begin(), st->hpoor.end(), 0);
    st->hlive[0] = 1;
    return QGPU_OK;
  }
  for (Shard& sh : st->shards) {
    if (!st->cfg.prune) CK(cudaMemsetAsync(sh.psi, 0, (1ull << st->m) * sizeof(double2), st->stream));
    if (sh.rank == 0) {
      CK(launch_set_amp(st->stream, sh.psi, 0, 1.0, 0.0));
      st->stats.kernels_launched++;
    }
  }
  return QGPU_OK;
}

constexpr size_t kMaxPlans = 8;

uint64_t plan_key(const qgpu_state* st, const qgpu_circuit* c) {
  uint64_t h = c->c.hash ? c->c.hash : circuit_hash(c->c);
  auto mix = [&](uint64_t v) {
    h ^= v + 0x9e3779b97f4a7c15ull + (h << 6) + (h >> 2);
  };
  mix(uint64_t(st->cfg.reorder) | uint64_t(st->cfg.involve_rule) << 4);
  mix(uint64_t(st->cfg.fuse_bits));
  mix(uint64_t(st->m));
  mix(st->map.involvement);
  mix(uint64_t(st->map.kl) | uint64_t(st->map.kg) << 8);
  for (int q = 0; q < st->n; ++q) mix(uint64_t(uint32_t(st->map.pos[q])));
  if (const char* ev = std::getenv("QGPU_REGBITS")) mix(uint64_t(std::atoi(ev)) << 32);
  if (const char* ev = std::getenv("QGPU_MAX_UOPS")) mix(uint64_t(std::atoi(ev)) << 40);
  if (const char* ev = std::getenv("QGPU_LOOKAHEAD")) mix(uint64_t(std::atoi(ev)) << 48);
  if (const char* ev = std::getenv("QGPU_ZSKIP")) mix(uint64_t(std::atoi(ev) + 1) << 56);
  if (const char* ev = std::getenv("QGPU_LMIN")) mix(uint64_t(std::atoi(ev) + 1) << 60);
  if (const char* ev = std::getenv("QGPU_LRELAX")) mix(uint64_t(std::atoi(ev) + 1) << 52);
  return h;
}

PlanOptions plan_options(const qgpu_config& cfg, bool fuse);

// Copy the programs of a plan's fused passes to a device buffer owned by the plan.
qgpu_status upload_plan(qgpu_state* st, CachedPlan* cp) {
  size_t nbytes = 0;
  cp->off.assign(cp->passes.size(), 0);
  for (size_t i = 0; i < cp->passes.size(); ++i) {
    cp->off[i] = nbytes;
    if (cp->passes[i].kind == PK_TILE) nbytes += (cp->passes[i].prog.bytes + 15) / 16 * 16;
  }
  cp->blob_bytes = nbytes;
  if (!nbytes) return QGPU_OK;
  CK(cudaMallocHost(&cp->h_blob, nbytes));
  for (size_t i = 0; i < cp->passes.size(); ++i)
    if (cp->passes[i].kind == PK_TILE) cp->passes[i].prog.pack(cp->h_blob + cp->off[i]);
  CK(cudaMalloc(&cp->d_blob, nbytes));
  return QGPU_OK;
}

// Send a plan's packed programs to its device blob, ordered on the state's stream after every
// earlier pass that read the blob.
qgpu_status send_plan(qgpu_state* st, CachedPlan* cp) {
  if (!cp->blob_bytes) return QGPU_OK;
  CK(cudaMemcpyAsync(cp->d_blob, cp->h_blob, cp->blob_bytes, cudaMemcpyHostToDevice, st->stream));
  st->stats.h2d_bytes += cp->blob_bytes;
  return QGPU_OK;
}

void prepare_jit(qgpu_state* st, const std::vector<Pass>& passes) {
  if (!st->cfg.jit) return;
  std::vector<const Pass*> want;
  for (const Pass& p : passes)
    if (p.kind == PK_TILE && (st->cfg.jit == 2 || p.k_out >= jit_min_bits())) want.push_back(&p);
  double ms = 0;
  const int k = jit_prepare(want, &ms);
  st->stats.jit_compiles += uint64_t(k);
  st->stats.jit_ms += ms;
}

// experiment overrides of the planner defaults (also part of the plan-cache key)
void plan_env(PlanOptions* o) {
  if (const char* ev = std::getenv("QGPU_ZSKIP")) o->zskip = std::atoi(ev) != 0;
  if (const char* ev = std::getenv("QGPU_LMIN")) o->l_min = std::atoi(ev);
  if (const char* ev = std::getenv("QGPU_LRELAX")) o->l_relax = std::atoi(ev);
  if (const char* ev = std::getenv("QGPU_REGBITS")) o->reg_bits = std::atoi(ev);
  if (const char* ev = std::getenv("QGPU_MAX_UOPS")) o->max_u_ops = std::atoi(ev);
  if (const char* ev = std::getenv("QGPU_LOOKAHEAD")) o->lookahead = std::atoi(ev);
}

PlanOptions plan_options(const qgpu_config& cfg, bool fuse) {
  PlanOptions o;
  o.fuse_bits = fuse ? cfg.fuse_bits : 0;
  plan_env(&o);
  o.prune = cfg.prune != 0;
  o.rule = cfg.involve_rule;
  return o;
}

}  // namespace

extern "C" {

const char* qgpu_last_error(void) { return g_err.c_str(); }

qgpu_status qgpu_gfc_max_bytes(uint64_t n, uint32_t seg_len, uint64_t* max_bytes) {
  if (!max_bytes) return fail(QGPU_ERR_INVALID_ARG, "max_bytes is NULL");
  if (seg_len == 0 || seg_len % 32) return fail(QGPU_ERR_INVALID_ARG, "seg_len %u is not a positive multiple of 32", seg_len);
  uint64_t total = 0;
  for (uint64_t s = 0; s < n; s += seg_len) {
    const uint64_t c = std::min<uint64_t>(seg_len, n - s);
    const uint64_t b = 8 * c + (c / 32) * 16 + ((c % 32) + 1) / 2;
    total += (b + 15) & ~15ull;
  }
  *max_bytes = total;
  return QGPU_OK;
}

qgpu_status qgpu_gfc_compress(const double* d_in, uint64_t n, uint32_t seg_len, void* d_out, uint64_t out_cap,
                              uint64_t* d_offsets, uint64_t* out_bytes, void* stream) {
  if (!out_bytes || !d_offsets) return fail(QGPU_ERR_INVALID_ARG, "out_bytes/d_offsets is NULL");
  if (seg_len == 0 || seg_len % 32) return fail(QGPU_ERR_INVALID_ARG, "seg_len %u is not a positive multiple of 32", seg_len);
  if (n && (!d_in || !d_out)) return fail(QGPU_ERR_INVALID_ARG, "d_in/d_out is NULL");
  if ((reinterpret_cast<uintptr_t>(d_in) | reinterpret_cast<uintptr_t>(d_out)) % 16)
    return fail(QGPU_ERR_INVALID_ARG, "d_in and d_out must be 16-byte aligned");
  cudaStream_t cs = static_cast<cudaStream_t>(stream);
  const uint64_t nseg = (n + seg_len - 1) / seg_len;
  CK0(cudaMemsetAsync(d_offsets, 0, sizeof(uint64_t), cs));
  *out_bytes = 0;
  if (nseg == 0) {
    CK0(cudaStreamSynchronize(cs));
    return QGPU_OK;
  }
  uint64_t* scratch = nullptr;
  CK0(cudaMallocAsync(reinterpret_cast<void**>(&scratch), gfc_scan_scratch_elems(nseg) * sizeof(uint64_t), cs));
  cudaError_t e = launch_gfc_sizes(cs, d_in, n, seg_len, d_offsets + 1);
  if (e == cudaSuccess) e = launch_scan_u64(cs, d_offsets + 1, nseg, scratch);
  uint64_t total = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&total, d_offsets + nseg, sizeof(uint64_t), cudaMemcpyDeviceToHost, cs);
  cudaFreeAsync(scratch, cs);
  CK0(e);
  CK0(cudaStreamSynchronize(cs));
  *out_bytes = total;
  if (total > out_cap)
    return fail(QGPU_ERR_INVALID_ARG, "out_cap %llu < compressed size %llu", (unsigned long long)out_cap,
                (unsigned long long)total);
  CK0(launch_gfc_encode(cs, d_in, n, seg_len, d_offsets, d_out));
  CK0(cudaStreamSynchronize(cs));
  return QGPU_OK;
}

qgpu_status qgpu_gfc_decompress(const void* d_in, const uint64_t* d_offsets, uint64_t n, uint32_t seg_len,
                                double* d_out, void* stream) {
  if (seg_len == 0 || seg_len % 32) return fail(QGPU_ERR_INVALID_ARG, "seg_len %u is not a positive multiple of 32", seg_len);
  if (n && (!d_in || !d_offsets || !d_out)) return fail(QGPU_ERR_INVALID_ARG, "NULL pointer");
  if (reinterpret_cast<uintptr_t>(d_in) % 16) return fail(QGPU_ERR_INVALID_ARG, "d_in must be 16-byte aligned");
  CK0(launch_gfc_decode(static_cast<cudaStream_t>(stream), d_in, d_offsets, n, seg_len, d_out));
  return QGPU_OK;
}

const char* qgpu_version(void) {
#define QGPU_STR2(x) #x
#define QGPU_STR(x) QGPU_STR2(x)
  return "qgpu abi " QGPU_STR(QGPU_ABI_VERSION) " sm_100a (B200) complex128";
}

qgpu_status qgpu_config_init(qgpu_config* cfg) {
  if (!cfg) return fail(QGPU_ERR_INVALID_ARG, "cfg is NULL");
  std::memset(cfg, 0, sizeof(*cfg));
  cfg->struct_size = sizeof(qgpu_config);
  cfg->world_size = 1;
  cfg->chunk_bits = 21;
  cfg->prune = 1;
  cfg->reorder = 2;
  cfg->fuse_bits = 12;
  cfg->swap_slab_bytes = 256ull << 20;
  cfg->jit = 1;
  return QGPU_OK;
}

qgpu_status qgpu_state_create(int n, const qgpu_config* cfg_in, qgpu_state** out) {
  try {
    if (!out) return fail(QGPU_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    qgpu_config cfg;
    qgpu_config_init(&cfg);
    if (cfg_in) {
      if (cfg_in->struct_size != sizeof(qgpu_config))
        return fail(QGPU_ERR_INVALID_ARG, "qgpu_config.struct_size mismatch (%u != %zu)",
                    cfg_in->struct_size, sizeof(qgpu_config));
      cfg = *cfg_in;
    }
    if (n < 1 || n > kMaxQubits) return fail(QGPU_ERR_INVALID_ARG, "n_qubits %d out of [1, %d]", n, kMaxQubits);
    if (cfg.world_size < 1 || (cfg.world_size & (cfg.world_size - 1)))
      return fail(QGPU_ERR_INVALID_ARG, "world_size %d is not a power of two", cfg.world_size);
    if (cfg.rank < 0 || cfg.rank >= cfg.world_size)
      return fail(QGPU_ERR_INVALID_ARG, "rank %d out of range", cfg.rank);
    if (cfg.host_slice_bits < 0 || cfg.host_slice_bits > 16)
      return fail(QGPU_ERR_INVALID_ARG, "host_slice_bits %d out of [0, 16]", cfg.host_slice_bits);
    if (cfg.host_slice_bits > 0 && (cfg.world_size != 1 || cfg.state_buffer))
      return fail(QGPU_ERR_UNSUPPORTED, "the host tier needs world_size 1 and no state_buffer");
    const int g = cfg.host_slice_bits > 0 ? cfg.host_slice_bits : std::countr_zero(unsigned(cfg.world_size));
    if (n - g < 5) return fail(QGPU_ERR_INVALID_ARG, "need n - log2(world_size) - host_slice_bits >= 5");
    if (cfg.fuse_bits < 0 || cfg.fuse_bits > kMaxTileBits - 1)
      return fail(QGPU_ERR_INVALID_ARG, "fuse_bits %d out of [0, %d]", cfg.fuse_bits, kMaxTileBits - 1);
    if (cfg.fuse_bits > 0 && cfg.fuse_bits < 7)
      return fail(QGPU_ERR_INVALID_ARG, "fuse_bits must be 0 or >= 7");
    if (cfg.reorder < 0 || cfg.reorder > 2) return fail(QGPU_ERR_INVALID_ARG, "reorder must be 0, 1 or 2");
    if (cfg.involve_rule < 0 || cfg.involve_rule > 1) return fail(QGPU_ERR_INVALID_ARG, "involve_rule must be 0 or 1");
    cfg.chunk_bits = std::min(std::max(cfg.chunk_bits, 0), n - g);
    if (const char* ev = std::getenv("QGPU_JIT")) cfg.jit = std::atoi(ev);
    if (cfg.jit < 0 || cfg.jit > 2) return fail(QGPU_ERR_INVALID_ARG, "jit must be 0, 1 or 2");
    auto* st = new qgpu_state();
    st->cfg = cfg;
    st->n = n;
    st->g = g;
    st->m = n - g;
    st->map.init(n, st->m);
    std::memset(&st->stats, 0, sizeof(st->stats));
    st->stats.ops_before_full_involvement = -1;
    auto bail = [&](qgpu_status s) {
      qgpu_state_destroy(st);
      return s;
    };
    cudaError_t e = cudaSetDevice(cfg.device);
    if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "cudaSetDevice(%d): %s", cfg.device, cudaGetErrorString(e)));
    if (cfg.stream) {
      st->stream = static_cast<cudaStream_t>(cfg.stream);
    } else {
      e = cudaStreamCreateWithFlags(&st->stream, cudaStreamNonBlocking);
      if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "cudaStreamCreate: %s", cudaGetErrorString(e)));
      st->own_stream = true;
    }
    const uint64_t need = (1ull << st->m) * sizeof(double2);
    // world_size > 1 without an NCCL id: "virtual ranks", every shard in this process on this
    // GPU (exercises the sharded path -- rank-bit conditions, activation, swaps -- on one GPU)
    st->virt = cfg.world_size > 1 && cfg.nccl_unique_id == nullptr;
    st->host = cfg.host_slice_bits > 0;
    const int nshard = st->host ? (1 << g) : st->virt ? cfg.world_size : 1;
    if (st->virt && cfg.state_buffer) return bail(fail(QGPU_ERR_UNSUPPORTED, "virtual ranks allocate their own shards"));
    if (cfg.host_compress && !cfg.host_slice_bits)
      return bail(fail(QGPU_ERR_INVALID_ARG, "host_compress needs host_slice_bits > 0"));
    if (st->host) {
      // pinned, device-mapped host memory: slices stream through device slots; readout kernels
      // read it in place (zero-copy) through unified addressing
      size_t hbytes = (size_t(1) << n) * sizeof(double2);
      size_t sstride = (size_t(1) << st->m);  // slice stride in amplitudes
      if (cfg.host_compress) {  // each slice holds its worst-case compressed size (>= raw)
        st->hcomp = true;
        const uint64_t nd = 2ull << st->m;
        qgpu_gfc_max_bytes(nd, st->hseg, &st->hcap);
        st->hnseg = (nd + st->hseg - 1) / st->hseg;
        sstride = st->hcap / sizeof(double2);
        hbytes = size_t(st->hcap) << g;
      }
      e = cudaHostAlloc(&st->h_state, hbytes, cudaHostAllocMapped | cudaHostAllocPortable);
      if (e != cudaSuccess) {
        cudaGetLastError();
        st->h_state = nullptr;
        return bail(fail(QGPU_ERR_OUT_OF_MEMORY, "host tier: cudaHostAlloc(%zu): %s", hbytes, cudaGetErrorString(e)));
      }
      double2* dev = nullptr;
      e = cudaHostGetDevicePointer(reinterpret_cast<void**>(&dev), st->h_state, 0);
      if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "cudaHostGetDevicePointer: %s", cudaGetErrorString(e)));
      for (int r = 0; r < nshard; ++r) st->shards.push_back(Shard{r, dev + size_t(r) * sstride, false});
      st->hlive.assign(size_t(nshard), 0);
      st->hraw.assign(size_t(nshard), 1);
      st->hpoor.assign(size_t(nshard), 0);
      if (st->hcomp) {
        e = cudaMallocHost(&st->hoff_base, size_t(nshard) * (st->hnseg + 1) * sizeof(uint64_t));
        if (e != cudaSuccess) return bail(fail(QGPU_ERR_OUT_OF_MEMORY, "host tier offsets: %s", cudaGetErrorString(e)));
        for (int r = 0; r < nshard; ++r) st->hoff.push_back(st->hoff_base + size_t(r) * (st->hnseg + 1));
        e = cudaMallocHost(&st->hsz, qgpu_state::kSzRing * sizeof(uint64_t));
        if (e != cudaSuccess) return bail(fail(QGPU_ERR_OUT_OF_MEMORY, "host tier size ring: %s", cudaGetErrorString(e)));
        st->store_k.assign(size_t(nshard), 0);
      }
      for (cudaStream_t* sp : {&st->s_h2d, &st->s_d2h}) {
        e = cudaStreamCreateWithFlags(sp, cudaStreamNonBlocking);
        if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "cudaStreamCreate: %s", cudaGetErrorString(e)));
      }
      for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
        e = cudaEventCreateWithFlags(&st->ev_loaded[i], cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&st->ev_computed[i], cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&st->ev_stored[i], cudaEventDisableTiming);
      }
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&st->ev_join, cudaEventDisableTiming);
      st->ev_slice.assign(size_t(nshard), nullptr);
      st->slice_seq.assign(size_t(nshard), 0);
      for (int r = 0; r < nshard && e == cudaSuccess; ++r)
        e = cudaEventCreateWithFlags(&st->ev_slice[size_t(r)], cudaEventDisableTiming);
      if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "cudaEventCreate: %s", cudaGetErrorString(e)));
    }
    for (int r = 0; r < nshard && !st->host; ++r) {
      Shard sh;
      sh.rank = st->virt ? r : cfg.rank;
      if (cfg.state_buffer) {
        if (cfg.state_buffer_bytes < need)
          return bail(fail(QGPU_ERR_OUT_OF_MEMORY, "state_buffer has %llu bytes, need %llu",
                           (unsigned long long)cfg.state_buffer_bytes, (unsigned long long)need));
        if (reinterpret_cast<uintptr_t>(cfg.state_buffer) % 16)
          return bail(fail(QGPU_ERR_INVALID_ARG, "state_buffer must be 16-byte aligned"));
        sh.psi = static_cast<double2*>(cfg.state_buffer);
      } else {
        e = cudaMalloc(&sh.psi, need);
        if (e != cudaSuccess) {
          cudaGetLastError();
          return bail(fail(QGPU_ERR_OUT_OF_MEMORY, "cudaMalloc(%llu): %s", (unsigned long long)need,
                           cudaGetErrorString(e)));
        }
        sh.own = true;
      }
      st->shards.push_back(sh);
    }
    st->psi = st->shards[0].psi;
    st->cap_amps = 1ull << st->m;
    e = cudaMalloc(&st->d_zero, sizeof(double2) << kMaxTileBits);
    if (e == cudaSuccess) e = cudaMemset(st->d_zero, 0, sizeof(double2) << kMaxTileBits);
    if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "zero buffer: %s", cudaGetErrorString(e)));
    e = cudaEventCreateWithFlags(&st->ops_evt, cudaEventDisableTiming);
    if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "cudaEventCreate: %s", cudaGetErrorString(e)));
    if (cfg.world_size > 1 && !st->virt) {
      qgpu_status s = comm_create(&st->comm, cfg, st->stream, (1ull << st->m), &g_err);
      if (s) return bail(s);
    }
    qgpu_status s = init_amplitudes(st);
    if (s) return bail(s);
    *out = st;
    return QGPU_OK;
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

qgpu_status qgpu_state_destroy(qgpu_state* st) {
  if (!st) return QGPU_OK;
  if (st->stream) cudaStreamSynchronize(st->stream);
  for (auto& t : st->pending) {
    cudaEventDestroy(t.a);
    cudaEventDestroy(t.b);
  }
  for (auto e : st->event_pool) cudaEventDestroy(e);
  if (st->comm) comm_destroy(st->comm);
  if (st->s_h2d) cudaStreamSynchronize(st->s_h2d);
  if (st->s_d2h) cudaStreamSynchronize(st->s_d2h);
  for (double2* p : st->slots) cudaFree(p);
  for (uint64_t* p : st->doff) cudaFree(p);
  for (uint64_t* p : st->dscan) cudaFree(p);
  for (unsigned char* p : st->dstage) cudaFree(p);
  if (st->hoff_base) cudaFreeHost(st->hoff_base);
  if (st->hsz) cudaFreeHost(st->hsz);
  if (st->h_state) cudaFreeHost(st->h_state);
  for (int i = 0; i < 2; ++i)
    for (cudaEvent_t e : {st->ev_loaded[i], st->ev_computed[i], st->ev_stored[i]})
      if (e) cudaEventDestroy(e);
  if (st->ev_join) cudaEventDestroy(st->ev_join);
  for (cudaEvent_t e : st->ev_slice)
    if (e) cudaEventDestroy(e);
  if (st->s_h2d) cudaStreamDestroy(st->s_h2d);
  if (st->s_d2h) cudaStreamDestroy(st->s_d2h);
  for (Shard& sh : st->shards)
    if (sh.own && sh.psi) cudaFree(sh.psi);
  if (st->d_ops) cudaFree(st->d_ops);
  if (st->h_ops) cudaFreeHost(st->h_ops);
  if (st->d_scratch) cudaFree(st->d_scratch);
  if (st->d_zero) cudaFree(st->d_zero);
  if (st->d_meas) cudaFree(st->d_meas);
  for (CachedPlan& cp : st->plans) {
    if (cp.d_blob) cudaFree(cp.d_blob);
    if (cp.h_blob) cudaFreeHost(cp.h_blob);
  }
  if (st->ops_evt) cudaEventDestroy(st->ops_evt);
  if (st->own_stream && st->stream) cudaStreamDestroy(st->stream);
  delete st;
  return QGPU_OK;
}

qgpu_status qgpu_state_reset(qgpu_state* st) {
  if (qgpu_status s = check_state(st)) return s;
  st->map.init(st->n, st->m);
  st->trace_order.clear();
  st->trace_inv.clear();
  st->gate_counter = 0;
  if (qgpu_status s = drain_timing(st)) return s;
  if (st->hcomp) {  // link bytes of the work before the reset belong to the old statistics
    CK(cudaStreamSynchronize(st->s_d2h));
    host_account_stores(st);
  }
  std::memset(&st->stats, 0, sizeof(st->stats));
  st->stats.ops_before_full_involvement = -1;
  return init_amplitudes(st);
}

qgpu_status qgpu_set_amplitudes(qgpu_state* st, const double* amps) {
  if (qgpu_status s = check_state(st)) return s;
  if (!amps) return fail(QGPU_ERR_INVALID_ARG, "amps is NULL");
  if (st->g > 0 && !st->host) return fail(QGPU_ERR_UNSUPPORTED, "set_amplitudes is single-GPU only");
  if (st->host) {
    CK(cudaStreamSynchronize(st->stream));
    CK(cudaStreamSynchronize(st->s_d2h));
    host_account_stores(st);
    for (size_t r = 0; r < st->shards.size(); ++r)
      std::memcpy(st->shards[r].psi, amps + 2 * (r << st->m), (size_t(1) << st->m) * sizeof(double2));
    std::fill(st->hlive.begin(), st->hlive.end(), 1ull << st->m);
    std::fill(st->hraw.begin(), st->hraw.end(), 1);
  } else {
    st->psi = st->shards[0].psi;
    CK(cudaMemcpyAsync(st->psi, amps, (1ull << st->n) * sizeof(double2), cudaMemcpyHostToDevice, st->stream));
    CK(cudaStreamSynchronize(st->stream));
  }
  st->map.init(st->n, st->m);
  for (int q = 0; q < st->n; ++q) {
    st->map.pos[q] = q;
    st->map.lq[q] = q;
  }
  st->map.kl = st->m;
  st->map.kg = st->n - st->m;
  st->map.involvement = (st->n >= 64) ? ~0ull : ((1ull << st->n) - 1);
  return QGPU_OK;
}

qgpu_status qgpu_synchronize(qgpu_state* st) {
  if (qgpu_status s = check_state(st)) return s;
  CK(cudaStreamSynchronize(st->stream));
  return drain_timing(st);
}

qgpu_status qgpu_state_info(const qgpu_state* st, int* n, int* nl, void** dev) {
  if (!st) return fail(QGPU_ERR_INVALID_ARG, "state is NULL");
  if (n) *n = st->n;
  if (nl) *nl = st->m;
  if (dev) *dev = st->psi;
  return QGPU_OK;
}

qgpu_status qgpu_apply_gate(qgpu_state* st, const double* U, int nt, const int* targets, int nc,
                            const int* controls) {
  try {
    if (qgpu_status s = check_state(st)) return s;
    if (!U || !targets) return fail(QGPU_ERR_INVALID_ARG, "U/targets is NULL");
    if (nt < 1 || nt > 2) return fail(QGPU_ERR_INVALID_ARG, "n_targets must be 1 or 2");
    if (nc < 0 || (nc > 0 && !controls)) return fail(QGPU_ERR_INVALID_ARG, "bad controls");
    Gate g;
    g.nt = nt;
    uint64_t seen = 0;
    for (int j = 0; j < nt + nc; ++j) {
      const int q = j < nt ? targets[j] : controls[j - nt];
      if (q < 0 || q >= st->n) return fail(QGPU_ERR_INVALID_ARG, "qubit %d out of range [0, %d)", q, st->n);
      if (seen >> q & 1) return fail(QGPU_ERR_INVALID_ARG, "qubit %d repeated", q);
      seen |= 1ull << q;
      if (j < nt) g.t[j] = q;
      else g.cmask |= 1ull << q;
    }
    const int dim = 1 << nt;
    for (int i = 0; i < dim * dim; ++i) g.U[i] = cplx{U[2 * i], U[2 * i + 1]};
    g.diag = is_diagonal(g.U, nt);
    g.relabel = false;  // an explicit gate call always moves data
    std::vector<Gate> gs{g};
    std::vector<int> order{0};
    std::vector<Pass> passes;
    std::vector<uint64_t> inv;
    plan_circuit(gs, order, st->map, plan_options(st->cfg, false), &passes, &inv);
    record_trace(st, order, inv, st->gate_counter);
    st->gate_counter++;
    return run_plan(st, passes);
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

}  // extern "C"

namespace {
constexpr int kMeasMax = 12;  // fused measurement: up to 2^12 buckets (32 KiB of shared memory)

// qgpu_apply_circuit; meas_m >= 0 also asks the last fused pass to histogram qubits meas_q
qgpu_status apply_circuit_impl(qgpu_state* st, const qgpu_circuit* c, int meas_m, const int* meas_q) {
  try {
    if (qgpu_status s = check_state(st)) return s;
    if (!c) return fail(QGPU_ERR_INVALID_ARG, "circuit is NULL");
    if (c->c.n > st->n) return fail(QGPU_ERR_INVALID_ARG, "circuit has %d qubits, state %d", c->c.n, st->n);
    const uint64_t key = plan_key(st, c);
    CachedPlan* hit = nullptr;
    for (CachedPlan& cp : st->plans)
      if (cp.key == key) hit = &cp;
    if (!hit) {
      CachedPlan cp;
      cp.key = key;
      cp.order = reorder(c->c.gates, st->cfg.reorder, st->cfg.involve_rule);
      QubitMap map = st->map;
      plan_circuit(c->c.gates, cp.order, map, plan_options(st->cfg, st->cfg.fuse_bits > 0), &cp.passes, &cp.inv);
      cp.map_after = map;
      for (const Gate& g : c->c.gates) cp.relabels += g.relabel ? 1 : 0;
      if (qgpu_status s = upload_plan(st, &cp)) return s;
      if (st->plans.size() >= kMaxPlans) {  // evict the least recently used
        size_t lru = 0;
        for (size_t i = 1; i < st->plans.size(); ++i)
          if (st->plans[i].last_use < st->plans[lru].last_use) lru = i;
        CK(cudaStreamSynchronize(st->stream));
        if (st->plans[lru].d_blob) cudaFree(st->plans[lru].d_blob);
        if (st->plans[lru].h_blob) cudaFreeHost(st->plans[lru].h_blob);
        st->plans.erase(st->plans.begin() + lru);
      }
      st->plans.push_back(std::move(cp));
      hit = &st->plans.back();
      prepare_jit(st, hit->passes);
    }
    if (qgpu_status s = send_plan(st, hit)) return s;
    hit->last_use = ++st->plan_clock;
    record_trace(st, hit->order, hit->inv, 0);
    st->stats.relabels += hit->relabels;
    st->map = hit->map_after;
    std::vector<const unsigned char*> ops(hit->passes.size());
    for (size_t i = 0; i < hit->passes.size(); ++i) ops[i] = hit->d_blob ? hit->d_blob + hit->off[i] : nullptr;
    // fused measurement: the last fused pass writes the final state (only zero-half
    // materialisation may follow it), so it can histogram the amplitudes it stores
    st->meas_pass = nullptr;
    st->meas_done = false;
    if (meas_m >= 0 && st->g == 0 && meas_m <= kMeasMax) {  // single resident state only
      // the map at the end of the last fused pass: undo the qubit relabels (final SWAP layers)
      // planned after it; zero-half materialisation passes do not change amplitudes either
      QubitMap at = hit->map_after;
      int last = -1;
      for (int i = int(hit->passes.size()) - 1; i >= 0; --i) {
        const Pass& pp = hit->passes[size_t(i)];
        if (pp.kind == PK_TILE) { last = i; break; }
        if (pp.kind == PK_RELABEL && pp.rel_a >= 0) { at.swap_positions(pp.rel_a, pp.rel_b); continue; }
        if (pp.kind != PK_ZERO) break;
      }
      // fused only when every requested qubit sits on a bit that is uniform across a warp's
      // stored amplitudes (tile-index or warp bits): then a tile adds one warp-reduced value per
      // warp. Lane and register bits would need an add per amplitude (shared-memory f64 atomics
      // are compare-and-swap loops) -- measured slower than re-reading the state, so those
      // requests take the separate readout kernel.
      if (last >= 0) {
        const Pass& lp = hit->passes[size_t(last)];
        uint64_t nonuni = 0;
        for (int i = 0; i < std::min(5, lp.b); ++i) nonuni |= 1ull << lp.spos[i];  // lane bits
        uint32_t a0 = 0;
        for (const TileOp& op : lp.prog.ops)
          if (op.kind == OP_REMAP) a0 = op.a0;  // the final register-bit mapping
        for (int k = 0; k < lp.prog.nr; ++k) nonuni |= 1ull << lp.spos[(a0 >> (4 * k)) & 15];
        for (int j = 0; j < meas_m; ++j) {
          const int pos = at.pos[meas_q[j]];
          if (pos >= 0 && (nonuni >> pos & 1)) last = -1;
        }
      }
      if (last >= 0) {
        if (!st->d_meas) CK(cudaMalloc(&st->d_meas, (size_t(8) << kMeasMax)));
        CK(cudaMemsetAsync(st->d_meas, 0, size_t(8) << meas_m, st->stream));
        st->meas_pass = &hit->passes[size_t(last)];
        st->meas_m = meas_m;
        for (int j = 0; j < meas_m; ++j) {
          const int pos = at.pos[meas_q[j]];
          st->meas_pos[j] = pos < 0 ? 63 : pos;  // never involved: the bit is 0 everywhere
        }
      }
    }
    qgpu_status s = exec_passes(st, hit->passes, ops);
    st->meas_pass = nullptr;
    return s;
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

}  // namespace

extern "C" {

qgpu_status qgpu_apply_circuit(qgpu_state* st, const qgpu_circuit* c) {
  return apply_circuit_impl(st, c, -1, nullptr);
}

qgpu_status qgpu_apply_circuit_probabilities(qgpu_state* st, const qgpu_circuit* c, int mq, const int* qubits,
                                             double* out) {
  if (qgpu_status s = check_state(st)) return s;
  if (mq < 0 || mq > 30) return fail(QGPU_ERR_INVALID_ARG, "m=%d out of [0, 30]", mq);
  if (!out || (mq > 0 && !qubits)) return fail(QGPU_ERR_INVALID_ARG, "NULL argument");
  uint64_t seen = 0;
  for (int j = 0; j < mq; ++j) {
    const int q = qubits[j];
    if (q < 0 || q >= st->n || (seen >> q & 1)) return fail(QGPU_ERR_INVALID_ARG, "bad qubit %d", q);
    seen |= 1ull << q;
  }
  if (qgpu_status s = apply_circuit_impl(st, c, mq, qubits)) return s;
  if (!st->meas_done) return qgpu_probabilities(st, mq, qubits, out);  // not fusable: read the state
  CK(cudaMemcpyAsync(out, st->d_meas, (size_t(8) << mq), cudaMemcpyDeviceToHost, st->stream));
  st->stats.d2h_bytes += size_t(8) << mq;
  CK(cudaStreamSynchronize(st->stream));
  return drain_timing(st);
}

qgpu_status qgpu_get_amplitudes_device(qgpu_state* st, uint64_t start, uint64_t count, double* dev_out) {
  if (qgpu_status s = check_state(st)) return s;
  if (!dev_out && count) return fail(QGPU_ERR_INVALID_ARG, "dev_out is NULL");
  if (start + count > (1ull << st->n) || start + count < start)
    return fail(QGPU_ERR_INVALID_ARG, "range [%llu, +%llu) outside 2^%d", (unsigned long long)start,
                (unsigned long long)count, st->n);
  if (!count) return QGPU_OK;
  const bool sharded = st->g > 0;
  if (sharded) CK(cudaMemsetAsync(dev_out, 0, count * 2 * sizeof(double), st->stream));
  for (Shard& sh : st->shards) {
    if (sharded && (uint64_t(sh.rank) >> st->map.kg) != 0) continue;  // inactive: all zero
    GatherArgs a{};
    a.psi = sh.psi;
    if (qgpu_status s = host_readable(st, size_t(sh.rank), &a.psi)) return s;
    a.out = reinterpret_cast<double2*>(dev_out);
    a.start = start;
    a.count = count;
    a.n = st->n;
    a.m = st->m;
    a.rank = uint64_t(sh.rank);
    a.only_owned = sharded ? 1 : 0;
    for (int q = 0; q < st->n; ++q) {
      a.pos[q] = st->map.pos[q] < 0 ? 0 : st->map.pos[q];
      if (st->map.pos[q] < 0) a.unassigned |= 1ull << q;
    }
    a.L = live(st, st->map.kl);
    if (st->host) a.L = std::min(a.L, st->hlive[size_t(sh.rank)]);  // zero-copy read of the slice
    CK(launch_gather(st->stream, a));
    st->stats.kernels_launched++;
  }
  if (sharded && st->comm) {  // every rank gets the full range (collective)
    if (qgpu_status s = comm_allreduce_sum(st->comm, dev_out, count * 2, st->stream, &g_err)) return s;
  }
  return QGPU_OK;
}

qgpu_status qgpu_get_amplitudes(qgpu_state* st, uint64_t start, uint64_t count, double* out) {
  if (qgpu_status s = check_state(st)) return s;
  if (!out && count) return fail(QGPU_ERR_INVALID_ARG, "out is NULL");
  const uint64_t chunk = std::min<uint64_t>(count, 1ull << 24);
  if (chunk > st->scratch_cap / 2) {
    CK(cudaStreamSynchronize(st->stream));
    if (st->d_scratch) CK(cudaFree(st->d_scratch));
    st->d_scratch = nullptr;
    CK(cudaMalloc(&st->d_scratch, chunk * 2 * sizeof(double)));
    st->scratch_cap = chunk * 2;
  }
  for (uint64_t done = 0; done < count; done += chunk) {
    const uint64_t c = std::min(chunk, count - done);
    if (qgpu_status s = qgpu_get_amplitudes_device(st, start + done, c, st->d_scratch)) return s;
    CK(cudaMemcpyAsync(out + 2 * done, st->d_scratch, c * 2 * sizeof(double), cudaMemcpyDeviceToHost, st->stream));
    st->stats.d2h_bytes += c * 2 * sizeof(double);
  }
  CK(cudaStreamSynchronize(st->stream));
  return drain_timing(st);
}

qgpu_status qgpu_probabilities(qgpu_state* st, int mq, const int* qubits, double* out) {
  if (qgpu_status s = check_state(st)) return s;
  if (mq < 0 || mq > 30) return fail(QGPU_ERR_INVALID_ARG, "m=%d out of [0, 30]", mq);
  if (!out || (mq > 0 && !qubits)) return fail(QGPU_ERR_INVALID_ARG, "NULL argument");
  ProbArgs a{};
  a.m = mq;
  uint64_t seen = 0;
  for (int j = 0; j < mq; ++j) {
    const int q = qubits[j];
    if (q < 0 || q >= st->n || (seen >> q & 1)) return fail(QGPU_ERR_INVALID_ARG, "bad qubit %d", q);
    seen |= 1ull << q;
    const int p = st->map.pos[q];
    a.ppos[j] = (p < 0 || p >= st->m) ? 63 : p;
  }
  const size_t B = size_t(1) << mq;
  const size_t nsh = st->shards.size();
  const size_t need = B * (nsh > 1 ? 2 : 1) + probs_scratch_doubles(mq);
  if (need > st->scratch_cap) {
    CK(cudaStreamSynchronize(st->stream));
    if (st->d_scratch) CK(cudaFree(st->d_scratch));
    st->d_scratch = nullptr;
    CK(cudaMalloc(&st->d_scratch, need * sizeof(double)));
    st->scratch_cap = need;
  }
  double* acc = st->d_scratch;
  double* tmp = st->d_scratch + B;
  double* part = st->d_scratch + B * (nsh > 1 ? 2 : 1);
  for (size_t i = 0; i < nsh; ++i) {
    const Shard& sh = st->shards[i];
    ProbArgs pa = a;
    pa.psi = sh.psi;
    if (st->host && (uint64_t(sh.rank) >> st->map.kg) == 0)
      if (qgpu_status s = host_readable(st, i, &pa.psi)) return s;
    pa.yfixed = 0;
    for (int j = 0; j < mq; ++j) {  // requested qubits on rank bits: fixed by this rank
      const int p = st->map.pos[qubits[j]];
      if (p >= st->m && ((uint64_t(sh.rank) >> (p - st->m)) & 1)) pa.yfixed |= 1ull << j;
    }
    const bool active = st->g == 0 || (uint64_t(sh.rank) >> st->map.kg) == 0;
    pa.L = active ? live(st, st->map.kl) : 0;
    if (st->host) pa.L = std::min(pa.L, st->hlive[i]);  // zero-copy read of the slice
    pa.out = i == 0 ? acc : tmp;
    CK(launch_probs(st->stream, pa, part));
    st->stats.kernels_launched += 1;
    if (i > 0) CK(launch_add(st->stream, acc, tmp, B));
  }
  if (st->comm) {
    if (qgpu_status s = comm_allreduce_sum(st->comm, acc, B, st->stream, &g_err)) return s;
  }
  CK(cudaMemcpyAsync(out, acc, B * sizeof(double), cudaMemcpyDeviceToHost, st->stream));
  st->stats.d2h_bytes += B * sizeof(double);
  CK(cudaStreamSynchronize(st->stream));
  return drain_timing(st);
}

qgpu_status qgpu_nccl_unique_id(void* out, size_t len) {
  if (!out || len < 128) return fail(QGPU_ERR_INVALID_ARG, "need a 128-byte buffer");
  std::string err;
  qgpu_status s = comm_unique_id(out, &err);
  if (s) return fail(s, "%s", err.c_str());
  return QGPU_OK;
}

qgpu_status qgpu_circuit_from_qasm(const char* text, size_t len, qgpu_circuit** out) {
  try {
    if (!text || !out) return fail(QGPU_ERR_INVALID_ARG, "NULL argument");
    *out = nullptr;
    auto* c = new qgpu_circuit();
    std::string err;
    qgpu_status s = parse_qasm(text, len, &c->c, &err);
    if (s) {
      delete c;
      return fail(s, "%s", err.c_str());
    }
    c->c.hash = circuit_hash(c->c);
    *out = c;
    return QGPU_OK;
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

qgpu_status qgpu_circuit_info(const qgpu_circuit* c, int* n, uint64_t* ng) {
  if (!c) return fail(QGPU_ERR_INVALID_ARG, "circuit is NULL");
  if (n) *n = c->c.n;
  if (ng) *ng = c->c.gates.size();
  return QGPU_OK;
}

qgpu_status qgpu_circuit_destroy(qgpu_circuit* c) {
  delete c;
  return QGPU_OK;
}

qgpu_status qgpu_circuit_reorder(const qgpu_circuit* c, int mode, uint64_t* order, uint64_t cap, uint64_t* n) {
  try {
    if (!c) return fail(QGPU_ERR_INVALID_ARG, "circuit is NULL");
    if ((mode & 3) > 2 || (mode & ~7)) return fail(QGPU_ERR_INVALID_ARG, "mode must be 0, 1 or 2 (+4: refined rule)");
    std::vector<int> o = reorder(c->c.gates, mode & 3, mode >> 2 & 1);
    if (n) *n = o.size();
    if (order)
      for (uint64_t i = 0; i < std::min<uint64_t>(cap, o.size()); ++i) order[i] = uint64_t(o[i]);
    return QGPU_OK;
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

qgpu_status qgpu_circuit_plan(const qgpu_circuit* c, int n, int world, int reorder_mode, int fuse_bits,
                              int64_t* info, uint64_t cap, uint64_t* n_passes) {
  try {
    if (!c) return fail(QGPU_ERR_INVALID_ARG, "circuit is NULL");
    if (n < c->c.n || n > kMaxQubits) return fail(QGPU_ERR_INVALID_ARG, "bad n");
    if (world < 1 || (world & (world - 1))) return fail(QGPU_ERR_INVALID_ARG, "bad world size");
    const int g = std::countr_zero(unsigned(world));
    QubitMap map;
    map.init(n, n - g);
    PlanOptions o;
    o.fuse_bits = fuse_bits;
    plan_env(&o);
    o.rule = reorder_mode >> 2 & 1;
    std::vector<Pass> passes;
    plan_circuit(c->c.gates, reorder(c->c.gates, reorder_mode & 3, o.rule), map, o, &passes, nullptr);
    if (n_passes) *n_passes = passes.size();
    for (uint64_t i = 0; info && i < std::min<uint64_t>(cap, passes.size()); ++i) {
      const Pass& p = passes[i];
      uint64_t S = 0;
      for (int j = 0; j < p.b; ++j) S |= 1ull << p.spos[j];
      int64_t* r = info + 8 * i;
      r[0] = p.first; r[1] = p.count; r[2] = p.kind; r[3] = p.k_in; r[4] = p.k_out; r[5] = p.b;
      r[6] = int64_t(S & 0xffffffffull);
      r[7] = int64_t(S >> 32);
    }
    return QGPU_OK;
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

qgpu_status qgpu_circuit_plan_text(const qgpu_circuit* c, int n, int world, int reorder_mode, int fuse_bits,
                                   char* buf, size_t cap, size_t* len) {
  try {
    if (!c) return fail(QGPU_ERR_INVALID_ARG, "circuit is NULL");
    if (n < c->c.n || n > kMaxQubits) return fail(QGPU_ERR_INVALID_ARG, "bad n");
    if (world < 1 || (world & (world - 1))) return fail(QGPU_ERR_INVALID_ARG, "bad world size");
    const int g = std::countr_zero(unsigned(world));
    if (n - g < 3) return fail(QGPU_ERR_INVALID_ARG, "too few local qubits");
    QubitMap map;
    map.init(n, n - g);
    PlanOptions o;
    o.fuse_bits = fuse_bits;
    plan_env(&o);
    o.rule = reorder_mode >> 2 & 1;
    std::vector<Pass> passes;
    plan_circuit(c->c.gates, reorder(c->c.gates, reorder_mode & 3, o.rule), map, o, &passes, nullptr);
    std::string t;
    char line[512];
    for (const Pass& p : passes) {
      std::snprintf(line, sizeof(line), "P %d %d %d %d %d %d", p.kind, p.k_in, p.k_out, p.kg, p.kg_from, p.nswap);
      t += line;
      for (int i = 0; i < p.nswap; ++i) {
        std::snprintf(line, sizeof(line), " %d %d", p.swap_global[i], p.swap_local[i]);
        t += line;
      }
      t += "\n";
      for (const PhysGate& pg : p.gates) {
        std::snprintf(line, sizeof(line), "G %d %d %d %llu %d", pg.nt, pg.p[0], pg.p[1],
                      static_cast<unsigned long long>(pg.pc), pg.diag ? 1 : 0);
        t += line;
        const int dim = 1 << pg.nt;
        for (int e = 0; e < dim * dim; ++e) {
          std::snprintf(line, sizeof(line), " %.17g %.17g", pg.U[e].re, pg.U[e].im);
          t += line;
        }
        t += "\n";
      }
    }
    t += "M";
    for (int q = 0; q < n; ++q) t += " " + std::to_string(map.pos[q]);
    t += "\n";
    if (len) *len = t.size();
    if (buf && cap) {
      const size_t k = std::min(cap - 1, t.size());
      std::memcpy(buf, t.data(), k);
      buf[k] = 0;
    }
    return QGPU_OK;
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

qgpu_status qgpu_circuit_jit_check(const qgpu_circuit* c, int n, int reorder_mode, int fuse_bits,
                                   int* n_compiled) {
  try {
    if (!c || n < c->c.n || n > kMaxQubits) return fail(QGPU_ERR_INVALID_ARG, "bad arguments");
    if (n_compiled) *n_compiled = 0;
    QubitMap map;
    map.init(n, n);
    PlanOptions o;
    o.fuse_bits = fuse_bits;
    plan_env(&o);
    o.rule = reorder_mode >> 2 & 1;
    std::vector<Pass> passes;
    plan_circuit(c->c.gates, reorder(c->c.gates, reorder_mode & 3, o.rule), map, o, &passes, nullptr);
    std::string cubin, log;
    for (const Pass& p : passes) {
      if (p.kind != PK_TILE) continue;
      if (!jit_cubin_cached(tile_jit_source(p), &cubin, &log, nullptr)) {
        if (log == "libnvrtc not found") return fail(QGPU_ERR_UNSUPPORTED, "%s", log.c_str());
        return fail(QGPU_ERR_CUDA, "NVRTC: %s\n--- source ---\n%s", log.c_str(), tile_jit_source(p).c_str());
      }
      if (n_compiled) (*n_compiled)++;
    }
    return QGPU_OK;
  } catch (const std::exception& ex) {
    return fail(QGPU_ERR_OUT_OF_MEMORY, "exception: %s", ex.what());
  }
}

qgpu_status qgpu_get_involvement(qgpu_state* st, uint64_t* mask) {
  if (!st || !mask) return fail(QGPU_ERR_INVALID_ARG, "NULL argument");
  *mask = st->map.involvement;
  return QGPU_OK;
}

qgpu_status qgpu_get_chunk_bitmap(qgpu_state* st, int c, uint64_t* words, uint64_t n_words) {
  if (!st || !words) return fail(QGPU_ERR_INVALID_ARG, "NULL argument");
  if (c < 0 || c > st->n) return fail(QGPU_ERR_INVALID_ARG, "chunk_bits out of range");
  const uint64_t nch = 1ull << (st->n - c);
  if (n_words < (nch + 63) / 64) return fail(QGPU_ERR_INVALID_ARG, "n_words too small");
  std::memset(words, 0, n_words * sizeof(uint64_t));
  const uint64_t full = (st->n >= 64) ? ~0ull : ((1ull << st->n) - 1);
  const uint64_t uninv = ~st->map.involvement & full;
  // bit j set iff ((j << c) & ~involvement) == 0 (Alg.1 l.7)
  for (uint64_t j = 0; j < nch; ++j)
    if (((j << c) & uninv) == 0) words[j >> 6] |= 1ull << (j & 63);
  return QGPU_OK;
}

qgpu_status qgpu_get_schedule(qgpu_state* st, uint64_t* order, uint64_t* inv, uint64_t cap, uint64_t* n) {
  if (!st) return fail(QGPU_ERR_INVALID_ARG, "state is NULL");
  const uint64_t len = st->trace_order.size();
  if (n) *n = len;
  for (uint64_t i = 0; i < std::min(cap, len); ++i) {
    if (order) order[i] = st->trace_order[i];
    if (inv) inv[i] = st->trace_inv[i];
  }
  return QGPU_OK;
}

qgpu_status qgpu_get_qubit_map(qgpu_state* st, int* pos) {
  if (!st || !pos) return fail(QGPU_ERR_INVALID_ARG, "NULL argument");
  for (int q = 0; q < st->n; ++q) pos[q] = st->map.pos[q];
  return QGPU_OK;
}

qgpu_status qgpu_get_stats(qgpu_state* st, qgpu_stats* out) {
  if (!st || !out) return fail(QGPU_ERR_INVALID_ARG, "NULL argument");
  if (!st->pending.empty()) {
    if (qgpu_status s = drain_timing(st)) return s;
  }
  if (st->hcomp) {  // compressed link bytes are known once the stores have completed
    CK(cudaStreamSynchronize(st->s_d2h));
    host_account_stores(st);
  }
  *out = st->stats;
  return QGPU_OK;
}

qgpu_status qgpu_reset_stats(qgpu_state* st) {
  if (!st) return fail(QGPU_ERR_INVALID_ARG, "state is NULL");
  if (qgpu_status s = drain_timing(st)) return s;
  const int64_t obf = st->stats.ops_before_full_involvement;
  std::memset(&st->stats, 0, sizeof(st->stats));
  st->stats.ops_before_full_involvement = obf;
  return QGPU_OK;
}

}  // extern "C"
