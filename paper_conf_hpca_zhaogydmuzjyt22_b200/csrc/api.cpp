// C ABI of libqgpu (include/qgpu.h): state management, planning and plan cache, readout,
// statistics. No exception crosses the ABI; every CUDA error is mapped to a status. Pass
// execution lives in exec.cpp.
#include <cstdarg>

#include "state.h"

namespace qgpu_impl {

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
  if (const char* ev = std::getenv("QGPU_GLOBAL_FIRST")) mix(uint64_t(std::atoi(ev) + 1) << 20);
  if (const char* ev = std::getenv("QGPU_AUTO_LANES")) mix(uint64_t(std::atoi(ev) + 1) << 28);
  if (const char* ev = std::getenv("QGPU_PASS_SCHED")) mix(uint64_t(std::atoi(ev) + 1) << 16);
  if (const char* ev = std::getenv("QGPU_SCHED_ROLLOUT")) mix(uint64_t(std::atoi(ev) + 1) << 12);
  if (const char* ev = std::getenv("QGPU_GLOBAL_MIN_LOCAL")) mix(uint64_t(std::atoi(ev) + 1) << 24);
  return h;
}

PlanOptions plan_options(const qgpu_config& cfg, bool fuse);

// Content equality of two circuits (everything the planner reads; the source line is not)
bool same_circuit(int an, const std::vector<Gate>& ag, const Circuit& b) {
  if (an != b.n || ag.size() != b.gates.size()) return false;
  for (size_t i = 0; i < ag.size(); ++i) {
    const Gate& x = ag[i];
    const Gate& y = b.gates[i];
    if (x.nt != y.nt || x.t[0] != y.t[0] || (x.nt == 2 && x.t[1] != y.t[1]) || x.cmask != y.cmask ||
        x.diag != y.diag || x.relabel != y.relabel)
      return false;
    if (std::memcmp(x.U, y.U, sizeof(cplx) << (2 * x.nt)) != 0) return false;
  }
  return true;
}

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
  if (const char* ev = std::getenv("QGPU_LMIN")) {  // a fixed lane policy (experiments)
    o->l_min = std::atoi(ev);
    o->auto_lanes = false;
  }
  if (const char* ev = std::getenv("QGPU_LRELAX")) {
    o->l_relax = std::atoi(ev);
    o->auto_lanes = false;
  }
  if (const char* ev = std::getenv("QGPU_AUTO_LANES")) o->auto_lanes = o->auto_lanes && std::atoi(ev) != 0;
  if (const char* ev = std::getenv("QGPU_SCHED_ROLLOUT")) o->sched_rollout = std::atoi(ev) != 0;
  // pass-aware execution order: 0 off, 1 tried by plan_circuit_auto (default), 2 always (no auto)
  if (const char* ev = std::getenv("QGPU_PASS_SCHED")) {
    const int v = std::atoi(ev);
    o->auto_sched = v == 1;
    if (v == 2) {
      o->pass_sched = true;
      o->auto_lanes = false;
    }
  }
  if (const char* ev = std::getenv("QGPU_REGBITS")) o->reg_bits = std::atoi(ev);
  if (const char* ev = std::getenv("QGPU_MAX_UOPS")) o->max_u_ops = std::atoi(ev);
  if (const char* ev = std::getenv("QGPU_LOOKAHEAD")) o->lookahead = std::atoi(ev);
  if (const char* ev = std::getenv("QGPU_GLOBAL_FIRST")) o->global_first = o->global_first && std::atoi(ev) != 0;
  if (const char* ev = std::getenv("QGPU_GLOBAL_MIN_LOCAL")) o->global_min_local = std::atoi(ev);
}

PlanOptions plan_options(const qgpu_config& cfg, bool fuse) {
  PlanOptions o;
  o.fuse_bits = fuse ? cfg.fuse_bits : 0;
  // sharded over ranks (NCCL or virtual): cross-rank first-touch expand; the host tier folds its
  // swaps into streaming sweeps over <= 4 slices, so it keeps local-first placement, 2-bit swaps
  o.global_first = cfg.world_size > 1 && cfg.host_slice_bits == 0;
  if (cfg.host_slice_bits > 0) o.max_swap_bits = 2;
  plan_env(&o);
  o.prune = cfg.prune != 0;
  o.rule = cfg.involve_rule;
  return o;
}

}  // namespace qgpu_impl

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
    if (cfg.timing < 0 || cfg.timing > 2) return fail(QGPU_ERR_INVALID_ARG, "timing must be 0, 1 or 2");
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
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess) return bail(fail(QGPU_ERR_CUDA, "cudaGetDeviceCount: %s", cudaGetErrorString(e)));
    if (cfg.device < 0 || cfg.device >= ndev)
      return bail(fail(QGPU_ERR_INVALID_ARG, "device %d out of [0, %d)", cfg.device, ndev));
    QGPU_ON_DEVICE(st);
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
  QGPU_ON_DEVICE(st);
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
  for (double2* b : st->vstage)
    if (b) cudaFree(b);
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
  QGPU_ON_DEVICE(st);
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
  st->prof.clear();
  return init_amplitudes(st);
}

qgpu_status qgpu_set_amplitudes(qgpu_state* st, const double* amps) {
  QGPU_ON_DEVICE(st);
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

qgpu_status qgpu_set_timing(qgpu_state* st, int mode) {
  if (qgpu_status s = check_state(st)) return s;
  if (mode < 0 || mode > 2) return fail(QGPU_ERR_INVALID_ARG, "timing must be 0, 1 or 2");
  st->cfg.timing = mode;
  return QGPU_OK;
}

qgpu_status qgpu_synchronize(qgpu_state* st) {
  QGPU_ON_DEVICE(st);
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
    QGPU_ON_DEVICE(st);
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
constexpr int kMeasMax = 12;
// QGPU_HACC=0 turns the per-slot fused measurement off (A/B against the separate readout);
// QGPU_HACC=2 fuses mode 2 even when lane bits need the run-time butterfly, 3: mode 2 never with
// unrequested lane bits (the round-2 rule, A/B)
bool hacc_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("QGPU_HACC");
    return !(e && e[0] == '0');
  }();
  return on;
}  // fused measurement: up to 2^12 buckets (32 KiB of shared memory)

// qgpu_apply_circuit; meas_m >= 0 also asks the last fused pass to histogram qubits meas_q
qgpu_status apply_circuit_impl(qgpu_state* st, const qgpu_circuit* c, int meas_m, const int* meas_q) {
  try {
    QGPU_ON_DEVICE(st);
    if (qgpu_status s = check_state(st)) return s;
    if (!c) return fail(QGPU_ERR_INVALID_ARG, "circuit is NULL");
    if (c->c.n > st->n) return fail(QGPU_ERR_INVALID_ARG, "circuit has %d qubits, state %d", c->c.n, st->n);
    const uint64_t key = plan_key(st, c);
    CachedPlan* hit = nullptr;
    // QGPU_PLAN_CACHE=0 (read per call; bench.py's cold end-to-end number): every apply
    // re-runs the Alg.2/3 reorder and the pass planning (the NVRTC kernel cache stays warm)
    const char* pc_env = std::getenv("QGPU_PLAN_CACHE");
    const bool use_cache = !(pc_env && pc_env[0] == '0');
    for (CachedPlan& cp : st->plans)
      if (use_cache && cp.key == key && same_circuit(cp.circ_n, cp.circ_gates, c->c)) hit = &cp;
    if (!hit) {
      CachedPlan cp;
      cp.key = key;
      cp.circ_n = c->c.n;
      cp.circ_gates = c->c.gates;
      cp.order = reorder(c->c.gates, st->cfg.reorder, st->cfg.involve_rule);
      QubitMap map = st->map;
      plan_circuit_auto(c->c.gates, cp.order, map, plan_options(st->cfg, st->cfg.fuse_bits > 0), &cp.passes, &cp.inv);
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
      // how the last pass histograms (TileArgs::hacc): every requested qubit on a tile bit of
      // the final mapping -> a slot's bucket is the same in every tile: per-slot register sums,
      // one add per slot at the end of the kernel (1); all on bits uniform across a warp's
      // stored amplitudes (tile-index or warp bits) -> one warp-reduced add per warp and tile
      // (0); otherwise lane / register bits mixed with tile-index bits -> per-warp private
      // histograms in shared memory, plain adds by the lanes whose buckets differ (2; shared-
      // memory f64 atomics are compare-and-swap loops, measured slower than re-reading the
      // state). If the private histograms do not fit in shared memory, the separate readout.
      st->meas_hacc = 0;
      if (last >= 0) {
        const Pass& lp = hit->passes[size_t(last)];
        uint64_t tilebits = 0;
        for (int i = 0; i < lp.b; ++i) tilebits |= 1ull << lp.spos[i];
        bool on_tile = true;
        for (int j = 0; j < meas_m; ++j) {
          const int pos = at.pos[meas_q[j]];
          if (pos >= 0 && !(tilebits >> pos & 1)) on_tile = false;
        }
        if (on_tile && meas_m > 0 && hacc_enabled()) st->meas_hacc = 1;
      }
      if (last >= 0 && !st->meas_hacc) {
        const Pass& lp = hit->passes[size_t(last)];
        uint64_t nonuni = 0;
        for (int i = 0; i < std::min(5, lp.b); ++i) nonuni |= 1ull << lp.spos[i];  // lane bits
        uint32_t a0 = 0;
        for (const TileOp& op : lp.prog.ops)
          if (op.kind == OP_REMAP) a0 = op.a0;  // the final register-bit mapping
        for (int k = 0; k < lp.prog.nr; ++k) nonuni |= 1ull << lp.spos[(a0 >> (4 * k)) & 15];
        bool uni = true;
        for (int j = 0; j < meas_m; ++j) {
          const int pos = at.pos[meas_q[j]];
          if (pos >= 0 && (nonuni >> pos & 1)) uni = false;
        }
        if (!uni) {
          if (hacc_enabled()) {  // per-warp private histograms (mode 2)
            st->meas_hacc = 2;
            st->meas_hlred = 0;
            for (int k = 0; k < std::min(5, lp.b); ++k) {
              bool req = false;
              for (int j = 0; j < meas_m; ++j) req = req || at.pos[meas_q[j]] == lp.spos[k];
              if (!req) st->meas_hlred |= 1u << k;
            }
            // an unrequested lane bit cost the run-time epilogue a shuffle butterfly on every
            // stored slot, with one lane in 2^u adding: measured on QAOA_32 (one such bit) it
            // added 15 ms to a 23 ms pass while the separate readout reads the 64 GiB state in
            // 9.4 ms. The NVRTC variants compile the masks in and reduce-scatter instead
            // (tile_driver, Body::kHistRS): mode 2 is fused with unrequested lane bits only when
            // the last pass runs an NVRTC kernel (QGPU_HACC=2 forces it, QGPU_HACC=3 never)
            const char* he = std::getenv("QGPU_HACC");
            const bool jit_last = (st->cfg.jit == 2 || (st->cfg.jit == 1 && lp.k_out >= jit_min_bits())) &&
                                  jit_available(nullptr);
            if (st->meas_hlred != 0u && !(he && he[0] == '2') && (!jit_last || (he && he[0] == '3'))) last = -1;
          } else {
            last = -1;
          }
        }
      }
      if (std::getenv("QGPU_DEBUG_HIST"))
        std::fprintf(stderr, "fused measurement: last fused pass %d, mode %d, unrequested lane bits %x\n", last,
                     st->meas_hacc, st->meas_hlred);
      if (last >= 0) {
        if (!st->d_meas) CK(cudaMalloc(&st->d_meas, (size_t(8) << kMeasMax)));
        CK(cudaMemsetAsync(st->d_meas, 0, size_t(8) << meas_m, st->stream));
        st->meas_pass = &hit->passes[size_t(last)];
        st->meas_m = meas_m;
        // bucket bit order inside the kernel: requested lane bits first, in lane order, so the
        // lanes of a warp add to consecutive shared-memory words (mode 2 without bank
        // conflicts); meas_perm maps a kernel bucket bit back to the caller's bit
        int jj = 0;
        const Pass& lp = hit->passes[size_t(last)];
        for (int k = 0; k < std::min(5, lp.b); ++k)
          for (int j = 0; j < meas_m; ++j)
            if (at.pos[meas_q[j]] == lp.spos[k]) st->meas_perm[jj++] = j;
        for (int j = 0; j < meas_m; ++j) {
          bool lane = false;
          for (int k = 0; k < std::min(5, lp.b); ++k) lane = lane || at.pos[meas_q[j]] == lp.spos[k];
          if (!lane) st->meas_perm[jj++] = j;
        }
        for (int j = 0; j < meas_m; ++j) {
          const int pos = at.pos[meas_q[st->meas_perm[j]]];
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
  QGPU_ON_DEVICE(st);
  if (qgpu_status s = apply_circuit_impl(st, c, mq, qubits)) return s;
  if (!st->meas_done) return qgpu_probabilities(st, mq, qubits, out);  // not fusable: read the state
  CK(cudaMemcpyAsync(out, st->d_meas, (size_t(8) << mq), cudaMemcpyDeviceToHost, st->stream));
  st->stats.d2h_bytes += size_t(8) << mq;
  CK(cudaStreamSynchronize(st->stream));
  bool ident = true;
  for (int j = 0; j < mq; ++j) ident = ident && st->meas_perm[j] == j;
  if (!ident) {  // kernel bucket bit j' holds the caller's bit meas_perm[j']
    std::vector<double> k(out, out + (size_t(1) << mq));
    for (uint64_t y = 0; y < (uint64_t(1) << mq); ++y) {
      uint64_t yk = 0;
      for (int j = 0; j < mq; ++j) yk |= ((y >> st->meas_perm[j]) & 1) << j;
      out[y] = k[yk];
    }
  }
  return drain_timing(st);
}

namespace {
// GatherArgs of rank `rank` for the logical range [start, start + count)
GatherArgs gather_args(const qgpu_state* st, const double2* psi, uint64_t rank, uint64_t start, uint64_t count,
                       double* dev_out) {
  GatherArgs a{};
  a.psi = psi;
  a.out = reinterpret_cast<double2*>(dev_out);
  a.start = start;
  a.count = count;
  a.n = st->n;
  a.m = st->m;
  a.rank = rank;
  for (int q = 0; q < st->n; ++q) {
    a.pos[q] = st->map.pos[q] < 0 ? 0 : st->map.pos[q];
    if (st->map.pos[q] < 0) a.unassigned |= 1ull << q;
  }
  a.L = live(st, st->map.kl);
  return a;
}
}  // namespace

// Sharded readout, point to point: the owner of each logical index is the rank whose
// bits the index has on the qubits at rank-bit positions. Every rank compacts the amplitudes it
// owns in the range (owner flags -> inclusive scan -> slot), sends its compact list to every other
// rank and receives theirs (grouped ncclSend / ncclRecv: each rank moves only what it owns, once
// per peer), then scatters every list into the output. All ranks share the qubit map, so each
// computes every rank's list length locally. Virtual ranks run the same kernels with the shards'
// compact lists read in place.
qgpu_status sharded_gather(qgpu_state* st, uint64_t start, uint64_t count, double* dev_out) {
  const uint64_t nact = 1ull << st->map.kg;
  const int world = int(uint64_t(1) << st->g);
  uint64_t *pos = nullptr, *scr = nullptr;
  double2 *own = nullptr, *rcv = nullptr;
  cudaStream_t s = st->stream;
  auto cleanup = [&]() {
    for (void* p : {static_cast<void*>(pos), static_cast<void*>(scr), static_cast<void*>(own), static_cast<void*>(rcv)})
      if (p) cudaFreeAsync(p, s);
  };
  cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&pos), count * sizeof(uint64_t), s);
  if (e == cudaSuccess)
    e = cudaMallocAsync(reinterpret_cast<void**>(&scr), std::max<uint64_t>(1, gfc_scan_scratch_elems(count)) * sizeof(uint64_t), s);
  if (e == cudaSuccess) e = cudaMallocAsync(reinterpret_cast<void**>(&own), count * sizeof(double2), s);
  if (e != cudaSuccess) {
    cleanup();
    CK(e);
  }
  CK(cudaMemsetAsync(dev_out, 0, count * 2 * sizeof(double), s));
  auto scan_for = [&](uint64_t r) -> cudaError_t {
    GatherArgs a = gather_args(st, nullptr, r, start, count, dev_out);
    cudaError_t x = launch_owner_flags(s, a, pos);
    if (x == cudaSuccess) x = launch_scan_u64(s, pos, count, scr);
    return x;
  };
  if (st->virt) {
    for (Shard& sh : st->shards) {
      if (uint64_t(sh.rank) >= nact) continue;  // inactive: all zero
      GatherArgs a = gather_args(st, sh.psi, uint64_t(sh.rank), start, count, dev_out);
      cudaError_t x = scan_for(uint64_t(sh.rank));
      if (x == cudaSuccess) x = launch_owned_compact(s, a, pos, own);
      if (x == cudaSuccess) x = launch_owned_scatter(s, a, pos, own);
      if (x != cudaSuccess) {
        cleanup();
        CK(x);
      }
      st->stats.kernels_launched += 5;
    }
    cleanup();
    return QGPU_OK;
  }
  // NCCL: list lengths of every rank (host), this rank's compact list, the exchange, the scatter
  const Shard& me = st->shards[0];
  std::vector<uint64_t> n_of(size_t(world), 0);
  uint64_t* tot = nullptr;
  CK(cudaMallocHost(&tot, sizeof(uint64_t) * size_t(world)));
  for (int r = 0; r < world; ++r) {
    if (uint64_t(r) >= nact) continue;
    cudaError_t x = scan_for(uint64_t(r));
    if (x == cudaSuccess) x = cudaMemcpyAsync(tot + r, pos + count - 1, sizeof(uint64_t), cudaMemcpyDeviceToHost, s);
    if (x == cudaSuccess && r == me.rank)
      x = launch_owned_compact(s, gather_args(st, me.psi, uint64_t(r), start, count, dev_out), pos, own);
    if (x != cudaSuccess) {
      cudaFreeHost(tot);
      cleanup();
      CK(x);
    }
  }
  CK(cudaStreamSynchronize(s));
  uint64_t recv_total = 0;
  for (int r = 0; r < world; ++r) {
    n_of[size_t(r)] = uint64_t(r) < nact ? tot[r] : 0;
    if (r != me.rank) recv_total += n_of[size_t(r)];
  }
  cudaFreeHost(tot);
  if (recv_total) CK(cudaMallocAsync(reinterpret_cast<void**>(&rcv), recv_total * sizeof(double2), s));
  std::vector<int> peer;
  std::vector<const double*> sb;
  std::vector<double*> rb;
  std::vector<size_t> sc, rc;
  std::vector<uint64_t> roff(size_t(world), 0);
  uint64_t off = 0;
  for (int r = 0; r < world; ++r) {
    if (r == me.rank) continue;
    peer.push_back(r);
    sb.push_back(reinterpret_cast<const double*>(own));
    sc.push_back(size_t(2 * n_of[size_t(me.rank)]));
    roff[size_t(r)] = off;
    rb.push_back(reinterpret_cast<double*>(rcv + off));
    rc.push_back(size_t(2 * n_of[size_t(r)]));
    off += n_of[size_t(r)];
  }
  if (qgpu_status x = comm_exchange(st->comm, int(peer.size()), peer.data(), sb.data(), sc.data(), rb.data(), rc.data(),
                                    s, &g_err)) {
    st->poisoned = true;
    cleanup();
    return x;
  }
  for (int r = 0; r < world; ++r) {
    if (!n_of[size_t(r)]) continue;
    GatherArgs a = gather_args(st, nullptr, uint64_t(r), start, count, dev_out);
    cudaError_t x = scan_for(uint64_t(r));
    if (x == cudaSuccess) x = launch_owned_scatter(s, a, pos, r == me.rank ? own : rcv + roff[size_t(r)]);
    if (x != cudaSuccess) {
      cleanup();
      CK(x);
    }
  }
  cleanup();
  return QGPU_OK;
}

qgpu_status qgpu_get_amplitudes_device(qgpu_state* st, uint64_t start, uint64_t count, double* dev_out) {
  QGPU_ON_DEVICE(st);
  if (qgpu_status s = check_state(st)) return s;
  if (!dev_out && count) return fail(QGPU_ERR_INVALID_ARG, "dev_out is NULL");
  if (start + count > (1ull << st->n) || start + count < start)
    return fail(QGPU_ERR_INVALID_ARG, "range [%llu, +%llu) outside 2^%d", (unsigned long long)start,
                (unsigned long long)count, st->n);
  if (!count) return QGPU_OK;
  if (st->g > 0 && !st->host) return sharded_gather(st, start, count, dev_out);
  if (st->g > 0) CK(cudaMemsetAsync(dev_out, 0, count * 2 * sizeof(double), st->stream));  // host tier slices
  for (Shard& sh : st->shards) {
    if (st->g > 0 && (uint64_t(sh.rank) >> st->map.kg) != 0) continue;  // host tier: inactive slice
    GatherArgs a = gather_args(st, sh.psi, uint64_t(sh.rank), start, count, dev_out);
    if (qgpu_status s = host_readable(st, size_t(sh.rank), &a.psi)) return s;
    a.only_owned = st->g > 0 ? 1 : 0;
    if (st->host) a.L = std::min(a.L, st->hlive[size_t(sh.rank)]);  // zero-copy read of the slice
    CK(launch_gather(st->stream, a));
    st->stats.kernels_launched++;
  }
  return QGPU_OK;
}

qgpu_status qgpu_get_amplitudes(qgpu_state* st, uint64_t start, uint64_t count, double* out) {
  QGPU_ON_DEVICE(st);
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
  QGPU_ON_DEVICE(st);
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
    if (qgpu_status s = comm_allreduce_sum(st->comm, acc, B, st->stream, &g_err)) {
      st->poisoned = true;  // an NCCL failure leaves the communicator unusable
      return s;
    }
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
    o.global_first = world > 1;
    plan_env(&o);
    o.rule = reorder_mode >> 2 & 1;
    std::vector<Pass> passes;
    plan_circuit_auto(c->c.gates, reorder(c->c.gates, reorder_mode & 3, o.rule), map, o, &passes, nullptr);
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
    o.global_first = world > 1;
    plan_env(&o);
    o.rule = reorder_mode >> 2 & 1;
    std::vector<Pass> passes;
    plan_circuit_auto(c->c.gates, reorder(c->c.gates, reorder_mode & 3, o.rule), map, o, &passes, nullptr);
    std::string t;
    char line[512];
    for (const Pass& p : passes) {
      std::snprintf(line, sizeof(line), "P %d %d %d %d %d %d", p.kind, p.k_in, p.k_out, p.kg,
                    p.kind == PK_ACTIVATE && p.act_copy ? -1 - p.kg_from : p.kg_from, p.nswap);
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
    plan_circuit_auto(c->c.gates, reorder(c->c.gates, reorder_mode & 3, o.rule), map, o, &passes, nullptr);
    std::string cubin, log;
    for (const Pass& p : passes) {
      if (p.kind != PK_TILE) continue;
      if (!jit_cubin_cached(tile_jit_source(p), &cubin, &log, nullptr)) {
        if (log == "libnvrtc not found") return fail(QGPU_ERR_UNSUPPORTED, "%s", log.c_str());
        return fail(QGPU_ERR_CUDA, "NVRTC: %s\n--- source ---\n%s", log.c_str(), tile_jit_source(p).c_str());
      }
      if (n_compiled) (*n_compiled)++;
    }
    // QGPU_JIT_CHECK_HIST=<key>: also the fused-measurement variants of the last tile pass (modes
    // 0 and 1, mode 2 with run-time masks, and mode 2 with the compile-time masks `key`, see
    // hist_rs_key: low 8 bits unrequested lane bits, bits 8..11 dead register bits)
    if (const char* ev = std::getenv("QGPU_JIT_CHECK_HIST")) {
      const uint32_t key = uint32_t(std::strtoul(ev, nullptr, 0));
      for (int i = int(passes.size()) - 1; i >= 0; --i) {
        const Pass& p = passes[size_t(i)];
        if (p.kind != PK_TILE) continue;
        for (int v = 0; v < 4; ++v) {
          const std::string src = tile_jit_source(p, v < 3 ? v : 2, v < 3 ? ~0u : key);
          if (!jit_cubin_cached(src, &cubin, &log, nullptr))
            return fail(QGPU_ERR_CUDA, "NVRTC: %s\n--- source ---\n%s", log.c_str(), src.c_str());
          if (n_compiled) (*n_compiled)++;
        }
        break;
      }
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
  QGPU_ON_DEVICE(st);
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

qgpu_status qgpu_get_pass_profile(qgpu_state* st, qgpu_pass_profile* out, uint64_t cap, uint64_t* n) {
  QGPU_ON_DEVICE(st);
  if (!st) return fail(QGPU_ERR_INVALID_ARG, "state is NULL");
  CK(cudaStreamSynchronize(st->stream));
  if (qgpu_status s = drain_timing(st)) return s;
  if (n) *n = st->prof.size();
  for (uint64_t i = 0; out && i < std::min<uint64_t>(cap, st->prof.size()); ++i) out[i] = st->prof[i];
  if (out) st->prof.clear();  // a size query (out = NULL) keeps the records
  return QGPU_OK;
}

qgpu_status qgpu_measure_fp64_peak(int device, double* fma_per_s) {
  if (!fma_per_s) return fail(QGPU_ERR_INVALID_ARG, "fma_per_s is NULL");
  int ndev = 0;
  CK0(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return fail(QGPU_ERR_INVALID_ARG, "device %d out of range", device);
  DeviceGuard guard(device);
  CK0(probe_fp64(fma_per_s));
  return QGPU_OK;
}

qgpu_status qgpu_reset_stats(qgpu_state* st) {
  QGPU_ON_DEVICE(st);
  if (!st) return fail(QGPU_ERR_INVALID_ARG, "state is NULL");
  if (qgpu_status s = drain_timing(st)) return s;
  const int64_t obf = st->stats.ops_before_full_involvement;
  std::memset(&st->stats, 0, sizeof(st->stats));
  st->stats.ops_before_full_involvement = obf;
  return QGPU_OK;
}

}  // extern "C"
