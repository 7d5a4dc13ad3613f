// Internal (not part of the ABI): the state object and the helpers shared by api.cpp (the C ABI,
// planning, readout) and exec.cpp (pass execution: resident passes, global-local swaps, the
// host-memory tier's streaming sweeps).
#pragma once
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

namespace qgpu_impl {
// A planned circuit for a given starting qubit map: passes (with their resolved JIT kernels)
// and their packed programs (pinned host blob + device copy). Reused when the same circuit is
// applied again from the same map (e.g. after qgpu_state_reset): no host planning; the packed
// gate data (matrices, phases, conditions) is re-sent host->device on every apply, an async
// copy of a few KB that keeps each apply's inputs flowing like an uncached run.
struct CachedPlan {
  uint64_t key = 0;
  // the planned circuit: a key hit is reused only if the content matches too
  int circ_n = 0;
  std::vector<Gate> circ_gates;
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
}  // namespace qgpu_impl

namespace qgpu_impl {

// QGPU_BSTORE: 0 (default) per-thread stores from registers, 1 bulk stores for programs with
// remaps, 2 bulk stores for every tile pass. Measured on B200 (profiles/r01/README.md): bulk
// stores of 1-8 KiB runs are 1.5-1.8x slower than the per-thread stores, so they stay off.
inline int bstore_mode() {
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
inline bool host_zc_decode() {
  static const bool v = [] {
    const char* ev = std::getenv("QGPU_HOST_ZC_DECODE");
    return ev && std::atoi(ev) != 0;
  }();
  return v;
}

// QGPU_HOST_SWEEP_PER_PASS=1 (ablation): the host tier streams the slices once per pass, as the
// paper traverses every chunk once per gate, instead of once per run of passes
inline bool host_sweep_per_pass() {
  const char* ev = std::getenv("QGPU_HOST_SWEEP_PER_PASS");  // read per call: ablations flip it
  return ev && std::atoi(ev) != 0;
}

// jit=1: specialise fused passes whose live range is >= 2^jit_min_bits amplitudes (default 12;
// read per call, so a test can run the same circuits at the library default and above it)
inline int jit_min_bits() {
  const char* ev = std::getenv("QGPU_JIT_MIN_BITS");
  return ev ? std::atoi(ev) : 12;
}


extern thread_local std::string g_err;

qgpu_status fail(qgpu_status s, const char* fmt, ...);

constexpr int kHostSweep = 100;  // TimedLaunch kind of a host-tier streaming sweep

struct TimedLaunch {
  cudaEvent_t a, b;
  int kind;
  uint64_t bytes;
  int count = 1;  // launches between a and b (a run of consecutive fused passes: one interval)
  // timing = 2: the pass this interval times (qgpu_get_pass_profile)
  bool prof = false;
  qgpu_pass_profile rec = {};
};

}  // namespace qgpu_impl

using namespace qgpu_impl;

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
  std::vector<qgpu_pass_profile> prof;  // timing = 2: completed per-pass records
  std::vector<cudaEvent_t> event_pool;
  Comm* comm = nullptr;
  // virtual ranks: per shard a send and a receive staging buffer of vstage_cap amplitudes (the
  // device-copy transport of the batched swap)
  std::vector<double2*> vstage;
  size_t vstage_cap = 0;
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
  int meas_perm[30] = {};              // kernel bucket bit j -> the caller's qubit index j
  int meas_hacc = 0;                   // TileArgs::hacc (see apply_circuit_impl)
  uint32_t meas_hlred = 0;             // TileArgs::hlred: lane bits not requested
  double* d_meas = nullptr;            // 2^kMeasMax doubles
  bool meas_done = false;
};


// Every entry point that touches a state runs on the state's device and restores the caller's
// current device on return (a state may be used from a thread whose current device differs, or
// next to states on other devices in the same process).
struct DeviceGuard {
  int prev = -1;
  bool changed = false;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) changed = cudaSetDevice(dev) == cudaSuccess;
  }
  ~DeviceGuard() {
    if (changed) cudaSetDevice(prev);
  }
  DeviceGuard(const DeviceGuard&) = delete;
  DeviceGuard& operator=(const DeviceGuard&) = delete;
};
#define QGPU_ON_DEVICE(st) DeviceGuard qgpu_device_guard_((st) ? (st)->cfg.device : 0)

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

namespace qgpu_impl {
// exec.cpp
cudaEvent_t get_event(qgpu_state* st);
qgpu_status drain_timing(qgpu_state* st);
inline uint64_t live(const qgpu_state* st, int k) {
  return st->cfg.prune ? (1ull << k) : (1ull << st->m);
}
void account(qgpu_state* st, uint64_t L_out, uint64_t bytes);
void sorted_positions(uint64_t mask, int* out, int* n);
qgpu_status zero_fill(qgpu_state* st, double2* psi, uint64_t from, uint64_t to);
qgpu_status exec_passes(qgpu_state* st, const std::vector<Pass>& passes,
                        const std::vector<const unsigned char*>& ops);
qgpu_status ensure_slots(qgpu_state* st, int unit, int* ngroups);
qgpu_status host_readable(qgpu_state* st, size_t r, const double2** psi);
void host_account_stores(qgpu_state* st);
}  // namespace qgpu_impl
using namespace qgpu_impl;
