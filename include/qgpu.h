/* qgpu.h -- C ABI of the B200-native Q-GPU hot path (libqgpu.so).
 *
 * Implements the data-parallel hot path of Q-GPU (Zhao et al., "Q-GPU: A Recipe of
 * Optimizations for Quantum Circuit Simulation Using GPUs", HPCA 2022; cited as P:<line> of
 * /root/reference/PAPER.md): applying 1- and 2-qubit, optionally controlled, gates to a 2^n
 * complex128 state vector (Eq.8), with zero-amplitude pruning driven by the
 * per-qubit `involvement` flags (Algorithm 1), dependency-aware reordering that
 * delays qubit involvement (Algorithms 2/3), and -- B200-specific, not in the
 * paper -- a resident-in-HBM state whose live part is a contiguous prefix (first-touch qubit
 * placement), fused multi-gate HBM passes, and global-local qubit swaps across GPUs.
 *
 * Conventions (readings listed in DESIGN.md):
 *  - Qubit q is bit q of the amplitude index (little-endian, Eq.8).
 *  - Amplitudes are complex128 stored as interleaved (re, im) doubles.
 *  - A gate matrix U is 2^t x 2^t, row-major, as (re, im) pairs; bit j of the row/column
 *    index refers to targets[j]. Controls fire on |1> only. Targets and controls are
 *    distinct and in [0, n).
 *  - All status codes are returned; a human-readable detail is in qgpu_last_error().
 *    No C++ exception or abort() crosses the ABI. On an argument error the state is left
 *    unchanged.
 *  - Apply calls are asynchronous on the state's stream; readout calls synchronise it. An
 *    asynchronous CUDA failure surfaces at the next synchronising call as QGPU_ERR_CUDA and
 *    marks the state QGPU_ERR_STATE.
 *  - Sharded mode (world_size > 1): every call is a collective, made by all ranks in the
 *    same order (SPMD); readout results are valid on every rank.
 *  - Thread safety: a state must not be used from two threads at once.
 */
#ifndef QGPU_H
#define QGPU_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define QGPU_ABI_VERSION 2

typedef enum {
  QGPU_OK = 0,
  QGPU_ERR_INVALID_ARG = 1,    /* bad argument; nothing was changed                         */
  QGPU_ERR_OUT_OF_MEMORY = 2,  /* device allocation failed or buffer too small              */
  QGPU_ERR_UNSUPPORTED = 3,    /* valid request outside the supported subset                */
  QGPU_ERR_PARSE = 4,          /* QASM syntax error; detail has line:col                    */
  QGPU_ERR_CUDA = 5,           /* CUDA runtime error                                        */
  QGPU_ERR_NCCL = 6,           /* NCCL error (sharded mode)                                 */
  QGPU_ERR_STATE = 7           /* state poisoned by an earlier asynchronous failure         */
} qgpu_status;

typedef struct qgpu_state qgpu_state;       /* opaque; owned by the library */
typedef struct qgpu_circuit qgpu_circuit;   /* opaque; owned by the library */

typedef struct {
  uint32_t struct_size;       /* = sizeof(qgpu_config); ABI guard                           */
  int device;                 /* CUDA device ordinal                                       */
  void* stream;               /* cudaStream_t to enqueue on; NULL = library-owned stream   */
  void* state_buffer;         /* optional caller-owned device memory (e.g. a torch tensor) */
  uint64_t state_buffer_bytes;/* its size; must be >= 16 * 2^(n - log2 world_size)          */
  int rank, world_size;       /* world_size = 2^g GPUs; 1 = single GPU                     */
  const void* nccl_unique_id; /* 128-byte ncclUniqueId (world_size > 1), same on all ranks.
                                 NULL with world_size > 1: "virtual ranks" -- all 2^g shards
                                 live in this process on `device` (tests the sharded path,
                                 rank-bit conditions and swaps, on one GPU)               */
  int chunk_bits;             /* c: bitmap/pruning unit 2^c amplitudes;
                                 default 21, clamped to [0, n]                             */
  int prune;                  /* 1 (default): pruning + delayed involvement;
                                 0: every pass over the full local range (ablation)        */
  int reorder;                /* qgpu_apply_circuit order: 0 program, 1 greedy (Alg.2),
                                 2 forward-looking (Alg.3, default)            */
  int fuse_bits;              /* b: tile qubits per fused HBM pass (default 12);
                                 0 = one kernel per gate (pair/quad/diag kernels)          */
  int timing;                 /* 1: time passes with CUDA events into the statistics (a run
                                 of consecutive fused passes is one interval); 2: every pass its
                                 own interval, recorded for qgpu_get_pass_profile          */
  uint64_t swap_slab_bytes;   /* staging bytes per all-to-all slab (sharded mode)          */
  int jit;                    /* fused passes: 0 = generic tile kernel only; 1 (default) = NVRTC-
                                 specialised kernel for passes whose live output range is >=
                                 2^12 amplitudes (env QGPU_JIT_MIN_BITS overrides the 12);
                                 2 = always. Falls back to the generic kernel if NVRTC is
                                 unavailable                                               */
  int host_slice_bits;        /* h: host-memory tier (the paper's setting,
                                 P:185-191). 0 (default) = state resident in HBM. h > 0
                                 (world_size = 1 only): the 2^n amplitudes live in pinned host
                                 memory as 2^h slices of 2^(n-h); the circuit is planned as
                                 for 2^h virtual ranks (slice index = top h physical bits) and
                                 each run of passes between global-local swaps streams the
                                 active slices through device slots (H2D, passes, D2H on three
                                 streams, double-buffered). Pruning skips never-active slices
                                 and moves only each slice's live prefix across the link.
                                 Device memory: 4-8 slots of 16 * 2^(n-h) bytes              */
  int involve_rule;           /* which qubits a gate involves:
                                 0 (default) = the paper's rule, every operand (P:229 l.11);
                                 1 = refined: a gate with a control on a never-involved qubit
                                 is the identity on the current state and is skipped; a
                                 diagonal gate on a never-involved target is restricted to that
                                 bit = 0 (a global phase becomes a scalar on the live part);
                                 neither involves anything. Exact. Also changes the
                                 Alg.2/3 costs (new qubits a gate would involve)            */
  int host_compress;          /* host tier only: 1 = slices cross the host link GFC-compressed
                                 (SURVEY §8f NEXT-3 on the NEXT-2 link): each stored
                                 live prefix is compressed on the device and written straight
                                 into pinned host memory, and decompressed on the device when
                                 it is loaded again. Lossless (bit-exact). Host memory: 2^h
                                 slices of gfc_max_bytes(2 * 2^(n-h), 4096) bytes            */
} qgpu_config;

typedef struct {
  uint64_t gates_applied;      /* gates executed (SWAPs handled as relabels included)        */
  uint64_t passes;             /* HBM passes (kernel launches over the state)                */
  uint64_t kernels_launched;   /* every kernel launched by the library                       */
  uint64_t relabels;           /* SWAP gates executed as qubit-map relabels (no data moved)  */
  uint64_t amps_processed;     /* sum over passes of live local amplitudes written           */
  uint64_t amps_full;          /* sum over passes of 2^(n-g) (what an unpruned pass touches) */
  uint64_t chunks_processed;   /* sum over passes of live chunks (2^c granularity)           */
  uint64_t chunks_skipped;     /* sum over passes of all-zero chunks skipped         */
  uint64_t algo_bytes;         /* algorithmic HBM bytes: reads of live input + writes        */
  uint64_t unfused_bytes;      /* bytes the same gates would move one gate per pass          */
  uint64_t swaps;              /* batched global-local swaps (sharded mode; one all-to-all each) */
  uint64_t swap_bytes;         /* amplitude bytes sent by this rank in swaps                  */
  int64_t ops_before_full_involvement; /* Table II statistic, -1 if never    */
  double kernel_ms;            /* timing=1: summed CUDA-event time of pass kernels           */
  double tile_kernel_ms;       /* timing=1: time of fused tile kernels only                  */
  uint64_t tile_kernel_launches;
  uint64_t tile_algo_bytes;    /* algorithmic bytes of fused tile kernels only               */
  double swap_ms;              /* timing=1: time in swaps                                    */
  uint64_t h2d_bytes;          /* host->device bytes copied by the library (ops, amplitudes) */
  uint64_t d2h_bytes;          /* device->host bytes copied by readout calls                 */
  uint64_t jit_launches;       /* fused passes run by an NVRTC-specialised kernel            */
  uint64_t jit_compiles;       /* kernels compiled (cache misses)                            */
  double jit_ms;               /* host time spent compiling                                  */
  /* host-memory tier (host_slice_bits > 0) */
  uint64_t host_h2d_bytes;     /* slice bytes copied host -> device (live prefixes only)      */
  uint64_t host_d2h_bytes;     /* slice bytes copied device -> host                           */
  uint64_t host_slice_loads;   /* slices streamed through the device                         */
  uint64_t host_slice_skips;   /* slice visits skipped because the slice is all zero  */
  uint64_t host_runs;          /* runs of passes (one streaming sweep over the slices each)  */
  double host_ms;              /* timing=1: CUDA-event time of the streaming sweeps          */
  uint64_t swap_bits;          /* rank bits exchanged by the swaps (sum of their widths s)   */
} qgpu_stats;

/* One pass of the last qgpu_apply_circuit / qgpu_apply_gate call when cfg.timing = 2 (every
 * pass timed by its own CUDA events): the per-pass roofline inputs. */
typedef struct qgpu_pass_profile {
  int32_t kind;                /* as qgpu_circuit_plan: 0 tile, 1 pair, 2 quad, 3 diag, 5 swap, 7 zero */
  int32_t k_in, k_out;         /* log2 live local size before / after                          */
  int32_t n_gates;             /* gates fused into the pass                                    */
  double ms;                   /* CUDA-event time of the pass (all local shards)               */
  uint64_t bytes;              /* algorithmic HBM bytes (live input read + output written)     */
  uint64_t amps_computed;      /* amplitudes the program ran on (zero tiles excluded)          */
  double fp64_ops;             /* FP64 pipe instructions (DFMA/DMUL/DADD) by the pass model    */
  int32_t lane_ops;            /* fused pass: 1-qubit ops on lane bits (4 warp shuffles per amplitude) */
  int32_t remaps;              /* fused pass: remaps / shared-memory ops (32 B of shared memory per amplitude) */
} qgpu_pass_profile;

/* ---- configuration and state ---------------------------------------------------------- */

/* Fill *cfg with defaults (device 0, own stream, prune=1, reorder=2, chunk_bits=21,
 * fuse_bits=12, world_size=1). Returns INVALID_ARG if cfg is NULL. */
qgpu_status qgpu_config_init(qgpu_config* cfg);

/* Create an n-qubit state |0...0> (all qubits start in |0>). cfg may be NULL
 * (defaults). The device buffer is cudaMalloc'ed unless cfg->state_buffer is given, in which
 * case it stays caller-owned and must outlive the state. No memset of the full buffer is done:
 * the live part grows by first-touch expansion, which writes the new half explicitly.
 * Errors: INVALID_ARG (n < 1, n > 40, bad world size), OUT_OF_MEMORY, CUDA, NCCL.
 * *out receives an owned handle; release it with qgpu_state_destroy. */
qgpu_status qgpu_state_create(int n_qubits, const qgpu_config* cfg, qgpu_state** out);

/* Destroy a state (synchronises its stream, frees library-owned memory). NULL is a no-op. */
qgpu_status qgpu_state_destroy(qgpu_state* st);

/* Return the state to |0...0> and clear involvement, qubit map, schedule trace and stats.
 * O(1) device work (one 16-byte write), asynchronous. */
qgpu_status qgpu_state_reset(qgpu_state* st);

/* Overwrite the full logical state from host memory: amps = 2 * 2^n doubles (re, im) in
 * logical index order. Marks every qubit involved (nothing left to prune). Synchronises.
 * Single-GPU or host tier (UNSUPPORTED when sharded over ranks). */
qgpu_status qgpu_set_amplitudes(qgpu_state* st, const double* amps);

/* Change cfg.timing (0 off, 1 grouped, 2 per pass) for the calls that follow. */
qgpu_status qgpu_set_timing(qgpu_state* st, int mode);

/* Block until all work enqueued on the state's stream is done; reports async errors. */
qgpu_status qgpu_synchronize(qgpu_state* st);

/* Number of qubits, local qubits (n - log2 world, or n - host_slice_bits) and the pointer of
 * the local buffer (device memory; with the host tier: the pinned host state, device-accessible
 * through unified addressing -- raw amplitudes only with host_compress = 0). */
qgpu_status qgpu_state_info(const qgpu_state* st, int* n_qubits, int* n_local, void** dev_ptr);

/* ---- gate application (the hot path) --------------------------------------------------- */

/* Apply one gate (Eq.8): U is (2^t x 2^t) row-major complex128 as 2*4^t
 * doubles (copied on call), t = n_targets in {1, 2}; targets[j] <-> bit j of U's index;
 * controls (n_controls >= 0, may be NULL when 0) must all be |1>. Updates `involvement`
 * with targets and controls (P:229 l.11), places first-touched qubits, and launches one pair
 * (t=1), quad (t=2) or diagonal kernel over the live prefix only (pruning).
 * Errors: INVALID_ARG (range, duplicates, NULL), STATE. Asynchronous. */
qgpu_status qgpu_apply_gate(qgpu_state* st, const double* U, int n_targets, const int* targets,
                            int n_controls, const int* controls);

/* Apply a parsed circuit: reorder (cfg.reorder: Alg.2/Alg.3), update involvement and qubit
 * placement per gate, cut the order into consecutive fused passes (cfg.fuse_bits) -- or, when
 * the pass cost model prefers it (single resident state, involve_rule 0, no SWAP gates), plan
 * the passes over the commutation DAG, keeping Alg.3's priority among ready gates (DESIGN.md
 * §4 "Pass scheduling") -- execute SWAP gates as qubit relabels, and launch. The result equals
 * program-order application up to floating-point rounding; the schedule and the
 * involvement trace reported by qgpu_get_schedule follow Alg.3's order exactly. The circuit
 * must have n_qubits <= the state's n. Errors: INVALID_ARG, STATE, CUDA, NCCL. Asynchronous. */
qgpu_status qgpu_apply_circuit(qgpu_state* st, const qgpu_circuit* c);

/* Apply a circuit and measure at its end (marginal probabilities as in
 * qgpu_probabilities, Eq.1): out[y] = sum over i with bits_Q(i) = y of |psi_i|^2 after the
 * circuit, qubits[0] <-> bit 0 of y, 0 <= m <= 30, out = 2^m doubles (host). When the plan ends
 * with a fused pass over the whole live state (single resident state, m <= 12) that pass
 * accumulates the histogram from the amplitudes it stores (no extra read of the state; in
 * shared memory, or with global f64 reductions when per-warp histograms would not fit beside
 * the tile buffers); otherwise this is qgpu_apply_circuit + qgpu_probabilities.
 * The state is left as qgpu_apply_circuit leaves it. Synchronises. Errors as both calls. */
qgpu_status qgpu_apply_circuit_probabilities(qgpu_state* st, const qgpu_circuit* c, int m,
                                             const int* qubits, double* out);

/* ---- readout (synchronising) ------------------------------------------------------------ */

/* Copy amplitudes [start, start+count) of the LOGICAL index space to host out[2*count]
 * (re, im). Handles the qubit map; never-involved qubits read as |0>. */
qgpu_status qgpu_get_amplitudes(qgpu_state* st, uint64_t start, uint64_t count, double* out);

/* Same into caller-owned DEVICE memory dev_out[2*count] (no host copy). Asynchronous. */
qgpu_status qgpu_get_amplitudes_device(qgpu_state* st, uint64_t start, uint64_t count,
                                       double* dev_out);

/* Marginal probabilities (Eq.1): out[y] = sum_{i: bits_Q(i)=y} |psi_i|^2, with
 * qubits[0] <-> bit 0 of y; 0 <= m <= 30; out has 2^m doubles (host). m = 0 gives the norm. */
qgpu_status qgpu_probabilities(qgpu_state* st, int m, const int* qubits, double* out);

/* ---- circuits ---------------------------------------------------------------------------- */

/* Parse an OpenQASM-2 subset. Errors: PARSE (with line:col),
 * UNSUPPORTED (gate definitions, reset, if, unknown gates), INVALID_ARG. *out is owned by
 * the caller; release with qgpu_circuit_destroy. */
qgpu_status qgpu_circuit_from_qasm(const char* text, size_t len, qgpu_circuit** out);
qgpu_status qgpu_circuit_info(const qgpu_circuit* c, int* n_qubits, uint64_t* n_gates);
qgpu_status qgpu_circuit_destroy(qgpu_circuit* c);

/* Host-only (no GPU needed): the execution order chosen by `mode` (0 program, 1 greedy
 * Alg.2, 2 forward-looking Alg.3; + 4 = costs under the refined involvement rule, see
 * qgpu_config.involve_rule) as gate indices into order[cap]. *n = number of gates. The
 * `reorder` argument of the plan / plan_text / jit_check diagnostics takes the same +4 flag. */
qgpu_status qgpu_circuit_reorder(const qgpu_circuit* c, int mode, uint64_t* order, uint64_t cap,
                                 uint64_t* n);

/* Host-only pass plan summary for diagnostics/tests: for each pass p (up to cap),
 * info[8p..8p+7] = {first gate position, gate count, kind, log2 L_in, log2 L_out, tile bits,
 * tile position mask (low 32 bits), high 32 bits of the mask}. kind: 0 tile, 1 pair, 2 quad,
 * 3 diag, 4 relabel, 5 swap. */
qgpu_status qgpu_circuit_plan(const qgpu_circuit* c, int n_qubits, int world_size, int reorder,
                              int fuse_bits, int64_t* info, uint64_t cap, uint64_t* n_passes);

/* Host-only (no GPU needed): the physical plan as text, for diagnostics and for executing the
 * sharded protocol independently in tests. One line per pass
 *   "P kind k_in k_out kg kg_from nswap g0 l0 g1 l1 ..." (kind as in qgpu_circuit_plan; 6 =
 *   activation of ranks [2^kg_from, 2^kg): zeroed, or -- written as kg_from' = -1 - kg_from --
 *   each receiving a copy of rank r - 2^kg_from's live prefix [0, 2^k_in) (cross-rank expand);
 *   5 = ONE batched swap: rank bit position g_i <-> local position l_i for all i at once),
 * followed by one line per gate of the pass in physical positions at execution time
 *   "G nt p0 p1 control_mask diag re im re im ..." (the (2^nt)^2 matrix, row-major),
 * and a final "M pos_0 ... pos_{n-1}" with the final qubit map (-1 = never involved).
 * Writes at most cap bytes (NUL-terminated); *len = bytes needed (without the NUL). */
qgpu_status qgpu_circuit_plan_text(const qgpu_circuit* c, int n_qubits, int world_size, int reorder,
                                   int fuse_bits, char* buf, size_t cap, size_t* len);

/* Host-only (no GPU needed): generate the NVRTC-specialised kernel source of every fused pass of
 * the plan (as qgpu_circuit_plan) and compile it for sm_100a into the on-disk cubin cache
 * ($QGPU_JIT_CACHE, else <dir of libqgpu.so>/build/jitcache). *n_compiled = passes compiled.
 * Returns UNSUPPORTED if NVRTC cannot be loaded, CUDA (with the NVRTC log in
 * qgpu_last_error) if a pass fails to compile. */
qgpu_status qgpu_circuit_jit_check(const qgpu_circuit* c, int n_qubits, int reorder, int fuse_bits,
                                   int* n_compiled);

/* ---- scheduler state (tests / diagnostics) ---------------------------------------------- */

/* Current `involvement` flags, bit q = logical qubit q has been acted on. */
qgpu_status qgpu_get_involvement(qgpu_state* st, uint64_t* mask);

/* Logical chunk bitmap for chunk size 2^chunk_bits: bit j (word j/64, bit j%64) = 1 iff
 * chunk j may hold a non-zero amplitude, i.e. ((j << c) & ~involvement) == 0.
 * n_words must be >= ceil(2^(n-c) / 64). */
qgpu_status qgpu_get_chunk_bitmap(qgpu_state* st, int chunk_bits, uint64_t* words,
                                  uint64_t n_words);

/* Execution trace since the last reset: order[k] = program index (within its circuit, or a
 * running gate counter for qgpu_apply_gate) of the k-th executed gate and
 * involvement_after[k] the flags after it. Either output may be NULL. *n = trace length. */
qgpu_status qgpu_get_schedule(qgpu_state* st, uint64_t* order, uint64_t* involvement_after,
                              uint64_t cap, uint64_t* n);

/* Physical position of each logical qubit (-1 = never involved), pos[n_qubits]. */
qgpu_status qgpu_get_qubit_map(qgpu_state* st, int* pos);

qgpu_status qgpu_get_stats(qgpu_state* st, qgpu_stats* out);
qgpu_status qgpu_reset_stats(qgpu_state* st);

/* Per-pass profile (cfg.timing = 2) of the passes executed since the last call of this
 * function with out != NULL or qgpu_state_reset: out[0..min(cap, n)), *n = records available
 * (out = NULL: size query, the records are kept). Synchronises.
 * Diagnostic (bench.py's per-pass binding bound, max(bytes / HBM peak, FP64 / FP64 peak)). */
qgpu_status qgpu_get_pass_profile(qgpu_state* st, qgpu_pass_profile* out, uint64_t cap, uint64_t* n);

/* Measure this device's FP64 FMA throughput: a kernel of independent DFMA chains on every SM,
 * timed with CUDA events (best of 3). *fma_per_s = thread-level DFMA per second (a DFMA is 2
 * flops). The FP64 peak of the per-pass roofline. Synchronous; ~0.1 s. */
qgpu_status qgpu_measure_fp64_peak(int device, double* fma_per_s);

/* Host: a fresh 128-byte ncclUniqueId (rank 0 creates it, the caller broadcasts it, e.g. with
 * torch.distributed). UNSUPPORTED if libnccl.so.2 cannot be loaded ($QGPU_NCCL_LIB). */
qgpu_status qgpu_nccl_unique_id(void* out, size_t len);

/* ---- GFC lossless compression of amplitude data ----------
 * The paper compresses every state chunk on the GPU before it crosses the host link: segments
 * of `seg_len` doubles are compressed independently, one warp per segment, as micro-chunks of
 * 32 doubles whose residual against the previous micro-chunk is stored as a 4-bit prefix (sign
 * + count of leading zero bytes) plus the remaining bytes. Byte format (readings
 * G1-G5): residual = w - prev on the 64-bit patterns (mod 2^64), prev = 0 for a
 * segment's first micro-chunk; nibble = sign << 3 | min(7, leading zero bytes of |residual|),
 * payload = the 8 - count low-order bytes of |residual|, little-endian; a micro-chunk of cnt
 * values = ceil(cnt/2) nibble bytes (value i in byte i/2, low nibble for even i) followed by the
 * payloads in order; a segment stream is zero-padded to a multiple of 16 bytes; the output is
 * the segment streams in order and offsets[s] = byte offset of segment s (offsets[0] = 0,
 * offsets[n_seg] = total). Lossless for every bit pattern (NaN payloads, -0.0).
 * All pointers except `out_bytes` / `max_bytes` are DEVICE memory owned by the caller; `d_out`
 * and `d_in` must be 16-byte aligned; `stream` is a cudaStream_t (NULL = legacy default).
 * seg_len must be a positive multiple of 32; n = number of doubles (2 per amplitude). */

/* Host: the largest possible compressed size of n doubles (every value 8 payload bytes). */
qgpu_status qgpu_gfc_max_bytes(uint64_t n, uint32_t seg_len, uint64_t* max_bytes);

/* Compress d_in[0..n) into d_out (capacity out_cap bytes) and d_offsets[0..n_seg], n_seg =
 * ceil(n / seg_len). Synchronises `stream` (the size is data dependent) and returns the total
 * in *out_bytes. If out_cap is too small: QGPU_ERR_INVALID_ARG, *out_bytes = the size needed,
 * d_offsets valid, d_out untouched. */
qgpu_status qgpu_gfc_compress(const double* d_in, uint64_t n, uint32_t seg_len, void* d_out,
                              uint64_t out_cap, uint64_t* d_offsets, uint64_t* out_bytes,
                              void* stream);

/* Inverse: d_out[0..n) from the stream d_in and d_offsets produced by qgpu_gfc_compress with
 * the same n and seg_len. Asynchronous on `stream`. */
qgpu_status qgpu_gfc_decompress(const void* d_in, const uint64_t* d_offsets, uint64_t n,
                                uint32_t seg_len, double* d_out, void* stream);

/* Thread-local detail of the last error on this thread (valid until the next call). */
const char* qgpu_last_error(void);

/* Library version / build string (ABI version, arch). */
const char* qgpu_version(void);

#ifdef __cplusplus
}
#endif
#endif /* QGPU_H */
