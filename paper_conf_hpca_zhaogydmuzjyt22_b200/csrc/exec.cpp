// Pass execution of libqgpu: resident fused / per-gate passes, global-local swaps (a10), and the
// host-memory tier's streaming sweeps (NEXT-2, with the GFC link of NEXT-3). Called from api.cpp.
#include <nvtx3/nvToolsExt.h>

#include "state.h"

namespace qgpu_impl {

// NVTX range per pass / swap / sweep (visible in Nsight timelines; header-only NVTX3,
// a no-op unless a tool is attached)
struct PassRange {
  explicit PassRange(const Pass& p) {
    static const char* const kinds[] = {"tile", "pair", "quad", "diag", "relabel", "swap", "activate", "zero"};
    char name[96];
    if (p.kind == PK_SWAP)
      std::snprintf(name, sizeof(name), "qgpu swap %d-bit k%d", p.nswap, p.k_in);
    else
      std::snprintf(name, sizeof(name), "qgpu %s k%d->%d gates %d", kinds[p.kind & 7], p.k_in, p.k_out, p.count);
    nvtxRangePushA(name);
  }
  ~PassRange() { nvtxRangePop(); }
};

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
    if (t.prof) {
      t.rec.ms = ms;
      st->prof.push_back(t.rec);
    }
    st->event_pool.push_back(t.a);
    st->event_pool.push_back(t.b);
  }
  st->pending.clear();
  return QGPU_OK;
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

// Global-local swap (a10): the pass's s pairs (rank bit swap_global - m <-> local position
// swap_local) as ONE batched all-to-all inside each group of 2^s ranks, over the live prefix only
// (amplitudes beyond 2^kl are zero on every rank and stay zero). NCCL: comm_swap (pipelined slabs,
// two streams). Virtual ranks (every shard on this GPU): the same geometry, pack / unpack kernels
// and slab loop, with device-to-device copies between the shards' staging as the transport.
qgpu_status exec_swap(qgpu_state* st, const Pass& p, uint64_t* bytes) {
  const int m = st->m;
  const uint64_t L = live(st, p.k_in);
  const uint64_t active = 1ull << p.kg;
  int j[8], l[8];
  for (int i = 0; i < p.nswap; ++i) {
    j[i] = p.swap_global[i] - m;
    l[i] = p.swap_local[i];
  }
  const uint64_t slab_req = std::max<uint64_t>(32, st->cfg.swap_slab_bytes / 16 / ((1ull << p.nswap) - 1));
  uint64_t sent = 0;
  if (!st->virt) {
    for (Shard& sh : st->shards) {
      if (uint64_t(sh.rank) >= active) continue;
      SwapGeom g;
      g.init(sh.rank, p.nswap, j, l, L);
      qgpu_status s = comm_swap(st->comm, sh.psi, g, slab_req, st->stream, &sent, &g_err);
      if (s) {
        st->poisoned = true;
        return s;
      }
    }
  } else {
    std::vector<SwapGeom> geo(st->shards.size());
    for (Shard& sh : st->shards)
      if (uint64_t(sh.rank) < active) geo[size_t(sh.rank)].init(sh.rank, p.nswap, j, l, L);
    const SwapGeom& g0 = geo[0];
    const uint64_t slab = std::max<uint64_t>(1, std::min(slab_req, g0.rest));
    const size_t need = size_t(slab) * size_t(g0.nb);
    if (need > st->vstage_cap) {
      CK(cudaStreamSynchronize(st->stream));
      for (double2* b : st->vstage) CK(cudaFree(b));
      st->vstage.assign(2 * st->shards.size(), nullptr);
      for (double2*& b : st->vstage) CK(cudaMalloc(&b, need * sizeof(double2)));
      st->vstage_cap = need;
    }
    for (uint64_t t0 = 0; t0 < g0.rest; t0 += slab) {
      const uint64_t cnt = std::min(slab, g0.rest - t0);
      BlockArgs a{};
      for (Shard& sh : st->shards) {  // pack every active shard's slab
        if (uint64_t(sh.rank) >= active) continue;
        const SwapGeom& g = geo[size_t(sh.rank)];
        a.psi = sh.psi;
        a.buf = st->vstage[2 * size_t(sh.rank)];
        a.nins = g.nins;
        for (int k = 0; k < g.nins; ++k) a.ins[k] = g.ins[k];
        a.t0 = t0;
        a.cnt = cnt;
        a.nb = g.nb;
        for (int b = 0; b < g.nb; ++b) a.pat[b] = g.pat[b];
        CK(launch_pack_blocks(st->stream, a));
        st->stats.kernels_launched++;
      }
      for (Shard& sh : st->shards) {  // transport: block b of rank r -> peer's slot for r's block
        if (uint64_t(sh.rank) >= active) continue;
        const SwapGeom& g = geo[size_t(sh.rank)];
        for (int b = 0; b < g.nb; ++b) {
          const SwapGeom& gp = geo[size_t(g.peer[b])];
          double2* dst = st->vstage[2 * size_t(g.peer[b]) + 1] + size_t(gp.slot(g.e)) * cnt;
          const double2* src = st->vstage[2 * size_t(sh.rank)] + size_t(b) * cnt;
          CK(cudaMemcpyAsync(dst, src, cnt * sizeof(double2), cudaMemcpyDeviceToDevice, st->stream));
        }
        if (sh.rank == 0) sent += 16 * cnt * uint64_t(g.nb);
      }
      for (Shard& sh : st->shards) {  // unpack the received blocks in place
        if (uint64_t(sh.rank) >= active) continue;
        const SwapGeom& g = geo[size_t(sh.rank)];
        a.psi = sh.psi;
        a.buf = st->vstage[2 * size_t(sh.rank) + 1];
        a.nins = g.nins;
        for (int k = 0; k < g.nins; ++k) a.ins[k] = g.ins[k];
        a.t0 = t0;
        a.cnt = cnt;
        a.nb = g.nb;
        for (int b = 0; b < g.nb; ++b) a.pat[b] = g.pat[b];
        CK(launch_unpack_blocks(st->stream, a));
        st->stats.kernels_launched++;
      }
    }
  }
  *bytes += sent;
  st->stats.swaps++;
  st->stats.swap_bits += uint64_t(p.nswap);
  st->stats.swap_bytes += sent;
  return QGPU_OK;
}

// Rank activation (PK_ACTIVATE): ranks [2^kg_from, 2^kg) start to hold live amplitudes. A copy
// activation (a fresh qubit placed on a rank bit by an uncontrolled 1-qubit gate, §8e) gives each
// new rank the live prefix of rank r - 2^kg_from; otherwise the new ranks are zeroed.
qgpu_status exec_activate(qgpu_state* st, const Pass& p) {
  const uint64_t active = 1ull << p.kg, from = 1ull << p.kg_from;
  if (!p.act_copy) {
    for (Shard& sh : st->shards)
      if (uint64_t(sh.rank) >= from && uint64_t(sh.rank) < active) {
        qgpu_status s = zero_fill(st, sh.psi, 0, 1ull << st->m);
        if (s) return s;
      }
    return QGPU_OK;
  }
  const uint64_t L = live(st, p.k_in);
  if (!st->virt) {
    qgpu_status s = comm_activate_copy(st->comm, st->shards[0].psi, p.kg_from, p.kg, L, st->stream, &g_err);
    if (s) st->poisoned = true;
    // the rest of a newly active buffer is read as zeros only through the live prefix: with
    // prune = 0 the copy covers the whole buffer (L = 2^m)
    return s;
  }
  for (Shard& sh : st->shards)
    if (uint64_t(sh.rank) >= from && uint64_t(sh.rank) < active)
      CK(cudaMemcpyAsync(sh.psi, st->shards[size_t(sh.rank) - size_t(from)].psi, L * sizeof(double2),
                         cudaMemcpyDeviceToDevice, st->stream));
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
    a.umat_n = int(std::min(P.pool.size(), size_t(kUmatParam)));
    if (P.pool.size() <= size_t(kUmatParam))
      for (size_t i = 0; i < P.pool.size(); ++i) a.umat[i] = make_double2(P.pool[i].re, P.pool[i].im);
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
    // tiles whose base selects a skipped zero half (zout) do no work: leave them out of the tile
    // enumeration (tile-index bit i <-> the i-th non-tile position below k_out)
    a.nzs = 0;
    const char* zd = std::getenv("QGPU_ZOUT_DEAL");  // 0: enumerate (and skip) them (A/B)
    if (st->cfg.prune && p.zout && !(zd && zd[0] == '0')) {
      uint64_t S = 0;
      for (int i = 0; i < p.b; ++i) S |= 1ull << p.spos[i];
      int ti = 0;
      for (int q = 0; q < kout; ++q) {
        if (S >> q & 1) continue;
        if (p.zout >> q & 1) a.zs_pos[a.nzs++] = ti;
        ++ti;
      }
      a.ntiles >>= a.nzs;
    }
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
    // FP64-heavy passes (pass_two_cta, default on): two single-buffered CTAs per SM at <= 128
    // registers (NVRTC kernels only)
    const bool two_cta = pass_two_cta(p) && (st->cfg.jit == 2 || (st->cfg.jit == 1 && p.k_out >= jit_min_bits()));
    if (two_cta) a.nbuf = 1;
    // optional bulk stores (staged tile, async copies per run; QGPU_BSTORE)
    const int bs = bstore_mode();
    if (bs == 2 || (bs == 1 && a.remaps)) a.nbuf = 3;
    if (tile_smem_bytes(a) > 227 * 1024) a.nbuf = 2;
    if (const char* nb = std::getenv("QGPU_NBUF"))  // experiments: fewer tile buffers
      if (a.remaps && !two_cta) a.nbuf = std::max(1, std::min(a.nbuf, std::atoi(nb)));
    a.bstore = (a.nbuf == 3 && (bs == 2 || (bs == 1 && a.remaps))) ? 1 : 0;
    if (st->meas_pass == &p && !a.bstore) {  // fused measurement, if its histogram fits in smem
      TileArgs h = a;
      h.hist = st->d_meas;
      h.hm = st->meas_m;
      h.hacc = st->meas_hacc;
      h.hlred = st->meas_hlred;
      for (int j = 0; j < st->meas_m; ++j) h.hpos[j] = st->meas_pos[j];
      // mode 2's per-warp private histograms (2^m doubles per warp) must not cost the pass CTAs
      // per SM: a two-CTA pass (<= 113 KiB each) or one that would not fit at all adds straight
      // to the global histogram instead (QGPU_HGLOB=0: never, 2: always)
      if (tile_smem_bytes(h) > 227 * 1024 && h.nbuf == 3) h.nbuf = 2;  // make room: double buffering
      if (h.hacc == 2) {
        const char* hg = std::getenv("QGPU_HGLOB");
        const int hgm = hg ? std::atoi(hg) : 1;
        const size_t cap = two_cta ? 113 * 1024 : 227 * 1024;
        h.hglob = (hgm == 2 || (hgm == 1 && tile_smem_bytes(h) > cap)) ? 1 : 0;
      }
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

// Amplitudes a pass's program runs on in one shard: a fused pass skips the tiles whose base
// lies in the zero region of an expansion (a non-tile position >= k_in set) or selects a
// skipped zero half (zin / zout positions); the per-gate kernels touch the live range.
uint64_t computed_amps(const qgpu_state* st, const Pass& p) {
  const int kin = st->cfg.prune ? p.k_in : st->m, kout = st->cfg.prune ? p.k_out : st->m;
  if (p.kind != PK_TILE) return 1ull << kout;
  uint64_t S = 0;
  for (int i = 0; i < p.b; ++i) S |= 1ull << p.spos[i];
  const uint64_t z = st->cfg.prune ? (p.zin | p.zout) : 0;
  int free_bits = 0;
  for (int q = 0; q < kout; ++q)
    if (!(S >> q & 1) && q < kin && !(z >> q & 1)) ++free_bits;
  return 1ull << (free_bits + p.b);
}

// Execute one planned pass: compute passes on every active local shard (ranks >= 2^kg hold
// only zeros and skip the work), swaps through the communicator, activations as memsets.
qgpu_status exec_pass(qgpu_state* st, const Pass& p, const unsigned char* d_ops, bool own_timing = true,
                      uint64_t* bytes_out = nullptr) {
  PassRange nvtx_range(p);
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
  if (p.kind == PK_ACTIVATE) return exec_activate(st, p);
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
    if (st->cfg.timing == 2) {
      tl.prof = true;
      tl.rec.kind = p.kind;
      tl.rec.k_in = kin;
      tl.rec.k_out = kout;
      tl.rec.n_gates = p.count;
      tl.rec.bytes = bytes;
      tl.rec.amps_computed = p.kind == PK_SWAP ? 0 : computed_amps(st, p);
      tl.rec.fp64_ops = p.fp64_per_amp * double(tl.rec.amps_computed);
      if (p.kind == PK_TILE)
        for (size_t i = 1; i < p.prog.ops.size(); ++i) {
          const int k = p.prog.ops[i].kind;
          tl.rec.lane_ops += k == OP_U1L;
          tl.rec.remaps += k == OP_REMAP || k == OP_SMEM1 || k == OP_SMEM2;
        }
    }
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
  nvtxRangePushA("qgpu host-tier sweep");
  struct Pop {
    ~Pop() { nvtxRangePop(); }
  } pop;
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
    st->stats.swap_bits++;
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
    const bool group = st->cfg.timing == 1 && st->shards.size() == 1;
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


}  // namespace qgpu_impl
