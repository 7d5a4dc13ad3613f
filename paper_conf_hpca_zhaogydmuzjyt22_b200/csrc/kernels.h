// Kernel argument blocks and launchers (kernels.cu). Passed by value as kernel parameters.
#pragma once

#include <cuda_runtime.h>

#include "qgpu_internal.h"

namespace qgpu {

struct PairArgs {
  double2* psi;
  double2 u[4];            // row-major 2x2
  int t;                   // target position
  int nins;                // inserted zero positions for pair enumeration (target + controls)
  int ins[kMaxQubits];
  int nins_c;              // controls only (shuffle variant: per-amplitude enumeration)
  int ins_c[kMaxQubits];
  uint64_t cset;           // local control bits forced to 1
  uint64_t npairs;         // live pairs with controls satisfied
  uint64_t L_in;           // reads at index >= L_in are implicit zeros (first-touch expand)
};

struct QuadArgs {
  double2* psi;
  double2 u[16];
  int t0, t1;              // bit 0 / bit 1 of U's index
  int nins;
  int ins[kMaxQubits];
  uint64_t cset;
  uint64_t nquads;
  uint64_t L_in;
};

struct PhaseArgs {
  double2* psi;
  double2 d[4];            // diagonal entries indexed by target bits
  int nt, t0, t1;
  int nins;
  int ins[kMaxQubits];     // positions fixed by `fixed`
  uint64_t fixed;          // bits forced to 1 (controls, and targets in the single-term form)
  uint64_t count;          // amplitudes enumerated
};

struct GatherArgs {
  const double2* psi;
  double2* out;
  uint64_t start, count;
  int n, m;
  uint64_t rank;
  int pos[kMaxQubits];
  uint64_t unassigned;     // logical qubits never involved (their |1> half is zero)
  uint64_t L;              // live local size
  int only_owned;          // sharded: write only the amplitudes this rank owns
};

// Sharded readout by point-to-point exchange (qgpu_get_amplitudes): for the logical
// range [start, start + count), flags[x] = 1 where rank `rank` owns x (x's bits on the qubits at
// rank-bit positions equal the rank, no bit on a never-involved qubit); after an inclusive scan
// flags[x] - 1 is x's slot in that rank's compact list. compact: the owner writes its amplitudes
// (psi, live prefix L) to their slots; scatter: a receiver places a rank's compact list.
cudaError_t launch_owner_flags(cudaStream_t st, const GatherArgs& a, uint64_t* flags);
cudaError_t launch_owned_compact(cudaStream_t st, const GatherArgs& a, const uint64_t* pos, double2* compact);
cudaError_t launch_owned_scatter(cudaStream_t st, const GatherArgs& a, const uint64_t* pos, const double2* compact);

struct ProbArgs {
  const double2* psi;
  uint64_t L;
  int m;
  int ppos[32];            // physical position of each requested qubit (63 = never set)
  uint64_t yfixed;         // bucket bits given by this rank's bits (requested qubits on rank bits)
  double* out;
  double* partial;
};

size_t tile_smem_bytes(const TileArgs& a);
int device_num_sms();
size_t probs_scratch_doubles(int m);
cudaError_t launch_pair(cudaStream_t st, const PairArgs& a, bool shfl);
cudaError_t launch_quad(cudaStream_t st, const QuadArgs& a);
cudaError_t launch_phase(cudaStream_t st, const PhaseArgs& a);
cudaError_t launch_tile(cudaStream_t st, const TileArgs& a);
cudaError_t launch_gather(cudaStream_t st, const GatherArgs& a);
cudaError_t launch_probs(cudaStream_t st, ProbArgs a, double* scratch);
cudaError_t launch_set_amp(cudaStream_t st, double2* psi, uint64_t i, double re, double im);
// FP64 peak probe (qgpu_measure_fp64_peak): thread-level DFMA per second on the current device
cudaError_t probe_fp64(double* fma_per_s);
cudaError_t launch_zero_where(cudaStream_t st, double2* psi, uint64_t L, uint64_t mask);
// sharded swaps (a10)
cudaError_t launch_swap_halves(cudaStream_t st, double2* a, double2* b, int lp, uint64_t half);
// a10 batched global-local swap of s rank bits with s local positions: the live local amplitudes
// split into 2^s blocks by their bits at the local positions; block d (all but the rank's own)
// goes to the peer whose rank bits are d. A slab is the rest-index range [t0, t0 + cnt) of every
// block (rest index = the live index with the swapped local positions removed); pack gathers it
// into buf[b * cnt + t], unpack scatters buf back (in place: a received block lands in the slots
// of the block that was sent to the same peer).
constexpr int kMaxSwapBlocks = 63;  // 2^6 - 1: up to 64 ranks in one batched swap
struct BlockArgs {
  double2* psi;
  double2* buf;
  int nins;
  int ins[8];       // the swapped local positions, ascending
  uint64_t t0, cnt;
  int nb;           // blocks in the slab
  uint64_t pat[kMaxSwapBlocks];  // block b's bits at the swapped local positions
};
cudaError_t launch_pack_blocks(cudaStream_t st, const BlockArgs& a);
cudaError_t launch_unpack_blocks(cudaStream_t st, const BlockArgs& a);
cudaError_t launch_add(cudaStream_t st, double* out, const double* in, uint64_t count);

// GFC compression (gfc.cu): per-segment padded sizes, encode at scanned offsets,
// decode; in-place inclusive scan of uint64 (scratch: gfc_scan_scratch_elems(n) elements)
cudaError_t launch_gfc_sizes(cudaStream_t st, const double* in, uint64_t n, uint32_t seg, uint64_t* sizes);
cudaError_t launch_gfc_encode(cudaStream_t st, const double* in, uint64_t n, uint32_t seg, const uint64_t* offsets,
                              void* out);
cudaError_t launch_gfc_decode(cudaStream_t st, const void* in, const uint64_t* offsets, uint64_t n, uint32_t seg,
                              double* out);
uint64_t gfc_scan_scratch_elems(uint64_t n);
cudaError_t launch_scan_u64(cudaStream_t st, uint64_t* a, uint64_t n, uint64_t* scratch);

}  // namespace qgpu
