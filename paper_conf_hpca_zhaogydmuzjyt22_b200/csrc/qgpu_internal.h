// Internal declarations of libqgpu (not part of the ABI).
//
// Layering:
//   qasm.cpp    a1  OpenQASM-2 subset -> circuit IR (gate matrices in gates.cpp)
//   sched.cpp   a2  dependency DAG + Alg.2 / Alg.3 reorder
//               a3  involvement flags, first-touch qubit placement, chunk bitmap
//               a4  pass planner: cuts the order into consecutive fused HBM passes
//   kernels.cu  a5-a9, a11  sm_100a kernels (pair, quad, diag, fused tile, gather, reduce)
//   comm.cpp    a10 global-local swaps over NCCL (sharded mode)
//   exec.cpp    pass execution: resident passes, swaps, host-memory tier sweeps (NEXT-2/3)
//   api.cpp     the C ABI (include/qgpu.h): state, plan cache, readout (state.h: shared types)
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "../../include/qgpu.h"
#include "tile_common.cuh"

namespace qgpu {

struct cplx {
  double re, im;
};

constexpr int kMaxQubits = 40;

// ------------------------------------------------------------------------------------ IR
// One gate after lowering: target matrix U (2^nt x 2^nt, row-major, bit j of
// the row/column index <-> t[j]) acting where every control in cmask is |1>.
struct Gate {
  int nt = 1;
  int t[2] = {0, 0};
  uint64_t cmask = 0;
  cplx U[16];
  bool diag = false;     // U is diagonal (z s t p rz cp cz crz rzz ...)
  bool relabel = false;  // uncontrolled SWAP: executed as a qubit-map relabel
  int line = 0;
  uint64_t tmask() const {
    uint64_t m = 1ull << t[0];
    if (nt == 2) m |= 1ull << t[1];
    return m;
  }
  uint64_t qmask() const { return tmask() | cmask; }  // qubits it involves (P:229 l.11)
};

struct Circuit {
  int n = 0;
  std::vector<Gate> gates;
  uint64_t hash = 0;  // content hash (gates, matrices), set by the parser / on demand
};
uint64_t circuit_hash(const Circuit& c);

qgpu_status parse_qasm(const char* text, size_t len, Circuit* out, std::string* err);
// Lower a gate name: fills the arity and the target matrix; false if the name is unknown.
bool gate_matrix(const std::string& name, const std::vector<double>& p, int* n_params,
                 int* n_qubits, int* n_controls, cplx* U, bool build);
bool is_diagonal(const cplx* U, int nt);
bool is_swap_matrix(const cplx* U, int nt);

// ------------------------------------------------------------------------------ schedule
// Qubits a gate involves when executed with involvement I (logical masks).
//   rule 0 (the paper, reading Q7): every operand, P:229 l.11;
//   rule 1 (refined; exact by P:221): a gate with a control outside I acts
//   as the identity (every amplitude has that bit 0) and a diagonal gate maps the zero
//   amplitudes to zero, so neither involves anything; other gates involve every operand.
inline uint64_t involving(const Gate& g, uint64_t I, int rule) {
  if (rule == 0) return g.qmask();
  if ((g.cmask & ~I) || g.diag) return 0;
  return g.qmask();
}
// mode 0 program order, 1 greedy (Alg.2), 2 forward-looking (Alg.3); costs use `rule`
std::vector<int> reorder(const std::vector<Gate>& gates, int mode, int rule = 0);

// Qubit map + involvement (a3). Physical positions 0..m-1 are local index bits, m..n-1 are
// global (rank) bits when sharded. Positions are handed out in first-touch order, local ones
// first, so the live part of every active rank's buffer is the prefix [0, 2^kl).
struct QubitMap {
  int n = 0, m = 0;              // total and local qubits
  int pos[kMaxQubits];           // logical -> physical, -1 = never involved
  int lq[kMaxQubits];            // physical -> logical, -1 = free
  int kl = 0;                    // assigned local positions (live local size 2^kl)
  int kg = 0;                    // assigned global positions (active ranks 2^kg)
  uint64_t involvement = 0;      // P:223 flags (logical)
  void init(int n_, int m_);
  // Set involvement bits (P:229 l.11) and place the not-yet-placed qubits of `mask`
  // (ascending logical index).
  void touch(uint64_t mask);
  uint64_t phys_mask(uint64_t logical_mask) const;
  void swap_positions(int pa, int pb);  // exchange the logical qubits at two positions
  void place_global(int q);             // place a never-involved qubit on the next rank bit
};

// --------------------------------------------------------------------------- device ops
// Device-side program structures (TileOp, RunEntry, PhaseTerm, Pattern) live in
// tile_common.cuh, shared with the kernels and the NVRTC-compiled pass kernels.
struct TileProgram {
  std::vector<TileOp> ops;
  std::vector<RunEntry> entries;
  std::vector<Pattern> patterns;
  std::vector<PhaseTerm> terms;
  std::vector<PhaseTerm> scalar;   // tile-uniform diagonal terms (commute with the whole pass)
  std::vector<cplx> pool;          // U matrices
  std::vector<cplx> tlo;           // [pattern][2^lb] products of the low-tile-index-bit terms
  int nr = 0, nw = 0;
  int lb = 0;                      // tile-index bits covered by tlo
  int spat = -1;                   // pattern of the scalar terms (-1: none)
  // byte offsets of each region inside the blob (all multiples of 16)
  size_t off_entries = 0, off_patterns = 0, off_terms = 0, off_scalar = 0, off_pool = 0, off_tlo = 0,
         bytes = 0;
  void layout();
  void pack(unsigned char* dst) const;
};


// A gate in physical positions at its execution time.
struct PhysGate {
  int gate = -1;          // index into the circuit
  int nt = 1;
  int p[2] = {0, 0};      // physical targets
  uint64_t pc = 0;        // physical control mask (may include global positions)
  cplx U[16];
  bool diag = false;
  bool expands_target = false;  // a target was first touched by this gate
};

enum PassKind : int {
  PK_TILE = 0, PK_PAIR = 1, PK_QUAD = 2, PK_DIAG = 3, PK_RELABEL = 4, PK_SWAP = 5,
  PK_ACTIVATE = 6,  // ranks [2^kg_from, 2^kg) become active: zeroed, or (act_copy) each receives a
                    // copy of the live prefix of rank r - 2^kg_from (cross-rank first-touch expand)
  PK_ZERO = 7       // write zeros over the live amplitudes that have a bit of `zmask` set
};

struct Pass {
  int kind = PK_TILE;
  int first = 0, count = 0;     // range in the execution order
  int k_in = 0, k_out = 0;      // log2 local live size before / after the pass
  // fused tile pass
  int b = 0, l = 0;
  int spos[kMaxTileBits];
  std::vector<PhysGate> gates;  // gates of the pass (tile) or the single gate (pair/quad/diag)
  TileProgram prog;             // built at pass close (tile)
  int n_est = 0;                // op-count estimate while the pass is open
  int kg = 0;                   // active ranks 2^kg while the pass runs (sharded)
  // swap pass (sharded): exchange global positions swap_global[i] with local swap_local[i]
  int nswap = 0;
  int swap_global[8], swap_local[8];
  int kg_from = 0;              // activation pass
  int act_copy = 0;             // activation by copy (a fresh qubit placed on a rank bit, §8e)
  mutable void* jit_fn = nullptr;  // specialised kernel, resolved at the first launch
  mutable void* jit_fn_hist[3] = {nullptr, nullptr, nullptr};  // fused-measurement variants, per mode
  mutable uint32_t jit_hist_key = ~0u;  // the mode-2 variant's compile-time masks (hist_rs_key)
  uint64_t unfused_bytes = 0;   // bytes the pass's gates would move one gate per pass
  double fp64_per_amp = 0.0;    // FP64 pipe instructions per computed amplitude (roofline model,
                                // fp64_model() in sched.cpp)
  double fp64_dense = 0.0;      // the same without zero-slot skipping / scalar folding (two-CTA rule)
  // zero-position skipping (tile passes): physical positions p whose bit-p = 1 half of the live
  // state is exactly zero and NOT materialised in memory -- on input (zin: loads read zeros
  // instead) and on output (zout: those amplitudes are not stored); PK_ZERO materialises zmask
  uint64_t zin = 0, zout = 0, zmask = 0;
  int rel_a = -1, rel_b = -1;   // PK_RELABEL: the two physical positions whose qubits it swapped
};

struct PlanOptions {
  int fuse_bits = 12;   // b
  int l_min = 5;        // minimum contiguous low tile bits (2^5 * 16 B = 512 B runs)
  int l_relax = 0;      // > 0: a gate may join an open pass with only this many (QGPU_LRELAX)
  int max_u_ops = 32;   // non-diagonal ops per fused pass (rqc_30: 24 -> 32 = 149.5 -> 145.6 ms)
  int max_ops = 256;    // all ops per fused pass
  int reg_bits = 4;     // register bits per thread (2^reg_bits amplitudes in registers)
  bool peephole = true; // fuse CX . D . CX into a diagonal (exact)
  int lookahead = 192;  // fusion lookahead window (gates); 0: passes are runs of `order`
  // pass-aware execution order (pass_schedule in sched.cpp): the gates are re-ordered, within
  // the commutation DAG, pass by pass -- each pass takes the closure of the ready gates over a
  // tile set chosen greedily by gain; single resident state, involvement rule 0, no relabels
  bool pass_sched = false;
  bool sched_rollout = true;  // near the full live size, choose each pass's kmax by a rollout
  bool prune = true;
  int rule = 0;         // involvement rule (see involving())
  // skip the halves of positions that a first touch left zero (placed by a diagonal gate or as
  // a control) until a non-diagonal op targets them; single resident state, fused passes only
  bool zskip = true;
  // sharded (m < n): place fresh qubits first touched by an uncontrolled 1-qubit non-diagonal
  // gate on the rank bits (up to log2 G of them) once >= global_min_local local positions are
  // assigned, so every rank holds live amplitudes from early on (cross-rank expand, §8e)
  bool global_first = false;
  int global_min_local = 10;
  int max_swap_bits = 8;  // rank bits per batched swap (the host tier's sweeps fold at most 2)
  // plan_circuit_auto: try the lane-bit policies (l_min, l_relax) = (5, 0) (5, 4) (5, 3) (4, 0)
  // (3, 0) and keep the plan with the lowest modelled time
  bool auto_lanes = true;
  // plan_circuit_auto also tries pass_sched = true (QGPU_PASS_SCHED=0 turns it off)
  bool auto_sched = true;
};

// Cut `gates` into passes, updating `map` (involvement, placement) exactly as the execution
// will. The execution order is `order` with fusion lookahead (later commuting gates that join
// the open tile pass are pulled forward) and passes are consecutive runs of it -- or, with
// opt.pass_sched, the pass-aware order of pass_schedule (sched.cpp) cut at its pass boundaries.
// inv_after[k] = involvement after the k-th gate of `order` (the paper's trace).
void plan_circuit(const std::vector<Gate>& gates, const std::vector<int>& order, QubitMap& map,
                  const PlanOptions& opt, std::vector<Pass>* passes,
                  std::vector<uint64_t>* inv_after);
// plan_circuit over candidate lane-bit policies (opt.l_min / opt.l_relax), with and without the
// pass-aware order (opt.auto_sched), when opt.auto_lanes: every candidate is planned from a copy
// of `map` (concurrently, on host threads), its passes costed by pass_cost_model(), and the
// cheapest plan is kept (map, passes, inv_after as plan_circuit leaves them).
void plan_circuit_auto(const std::vector<Gate>& gates, const std::vector<int>& order, QubitMap& map,
                       const PlanOptions& opt, std::vector<Pass>* passes, std::vector<uint64_t>* inv_after);
// Modelled seconds of one pass on one B200: max(HBM bytes / (copy peak x efficiency of its
// contiguous run length 16 * 2^l B), modelled FP64 instructions / (FP64 peak x issue efficiency))
// plus a launch gap.
double pass_cost_model(const Pass& p, int m);
// Two single-buffered CTAs per SM at <= 128 registers for this pass's NVRTC kernel (instead of
// one triple-buffered CTA at <= 255): QGPU_2CTA=1 every pass, 2 passes whose program runs >= 40
// FP64 instructions per amplitude (the latency-bound ones), 4 (default) those and the passes
// whose program remaps at >= 20 FP64 per amplitude, 0 none (read per call).
bool pass_two_cta(const Pass& p);
// Build the device ops of a tile pass from its gates and tile positions.
void build_tile_ops(Pass& p, int m, int reg_bits = 4);
// Unfused byte model of one gate on live size 2^k.
uint64_t unfused_gate_bytes(const PhysGate& g, int k_in, int k_out);
// FP64 instructions per amplitude a pass's program executes (fused tile pass) or its single
// gate needs (pair / quad / diagonal kernels): the FP64 side of the per-pass roofline.
// zero_aware: count what the NVRTC body executes (zero slots of a first-touch expansion skipped,
// the tile-uniform scalar folded into a run); else the dense count (the two-CTA thresholds)
double fp64_model(const Pass& p, bool zero_aware = true);

}  // namespace qgpu
