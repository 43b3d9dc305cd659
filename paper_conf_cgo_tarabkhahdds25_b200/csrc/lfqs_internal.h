// lfqs_internal.h -- internal types of the B200 LFQS library (not part of the ABI).
//
// Citations: "P:N" = PAPER.md line N (Tarabkhah et al., CGO'25).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <memory>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/lfqs.h"

#include <nvtx3/nvToolsExt.h>

namespace lfqs {

// NVTX range over a host-side phase (a circuit run, an exchange, canonicalisation,
// a measurement) for nsys / ncu --nvtx timelines (SURVEY §5 tracing); header-only NVTX3,
// a no-op unless a tool is attached.
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

// Thrown inside the library, converted to lfqs_status at the ABI boundary.
struct Error : std::runtime_error {
  lfqs_status status;
  Error(lfqs_status s, const std::string& m) : std::runtime_error(m), status(s) {}
};

#define LFQS_CUDA_CHECK(expr)                                                              \
  do {                                                                                     \
    cudaError_t _e = (expr);                                                               \
    if (_e != cudaSuccess)                                                                 \
      throw ::lfqs::Error(LFQS_ERR_CUDA, std::string(#expr) + ": " + cudaGetErrorString(_e)); \
  } while (0)

inline void require(bool ok, const std::string& msg) {
  if (!ok) throw Error(LFQS_ERR_INVALID_ARG, msg);
}

struct cplx {
  double re, im;
};

// ---------------------------------------------------------------------------
// Host-side gate decode (a1 in SURVEY §8(a)): kind -> matrix and sparsity class,
// the static matrix specialisation of P:441-445.
// ---------------------------------------------------------------------------
enum class GClass : int {
  NOOP,       // identity (I, or a diagonal of ones)
  DIAG,       // diagonal: a[k] *= d[loc(k)]          (Z, S, T, Rz, Phase, CZ, CPhase, MC-Z)
  PERM_X,     // pair swap                             (X, CNOT, Toffoli)
  PERM_Y,     // pair swap with +-i                    (Y)
  PERM_SWAP,  // exchange a[k|2^t0] <-> a[k|2^t1]      (SWAP)
  DENSE       // 2^m x 2^m matvec per group            (H, Rx, Ry, U3, UNITARYm)
};

struct Decoded {
  int kind = 0;
  int m = 1;                 // number of targets
  int targets[3] = {0, 0, 0};// targets[0] = MSB of the local index (reading R2)
  uint64_t cmask = 0;        // control mask
  GClass cls = GClass::DENSE;
  bool is_h = false;         // Hadamard: sq2r*(s1 +- s2) (Fig. 12c / Fig. 14)
  cplx M[64];                // 2^m x 2^m row-major
};

// Validates and decodes one gate; throws Error(INVALID_ARG) on bad input.
Decoded decode_gate(int n, int kind, const int* targets, int n_targets, uint64_t cmask,
                    const double* params, int n_params, const double* matrix);
int kind_arity(int kind);
int kind_nparams(int kind);

// ---------------------------------------------------------------------------
// Kernel-side parameter blocks (passed by value)
// ---------------------------------------------------------------------------
constexpr int kMaxInsert = 40;

// Free index -> amplitude index: insert a 0 bit at each pos[] (ascending), then
// OR `ones` (Fig. 3b, Fig. 14 id1 = rR + 2 rL Rs, generalised
// to several inserted bits: Fig. 8's three loops Ls/Gs/Rs).
struct InsertPlan {
  int np;
  int pos[kMaxInsert];
  uint64_t ones;
};

struct Options {
  // Warp-shuffle path for targets < 5.  Measured equal-or-slower than the
  // generic 32-byte path on B200 (profiles/r01_gate_sweep.md), so off by default.
  bool lowq_shuffle = false;
  bool wide256 = true;       // two adjacent groups per item, 32-byte accesses
  bool line_reads = true;    // fixed bits 1-2 -> store predicate, whole-line reads (apply_kernels.cu)
  // Global-qubit exchanges overlapped with local work (state.cu execute): the
  // exchange is split into 2^exchange_chunk_bits parts by as many local qubits; the last
  // local ops before it and the first after it run part by part on the compute stream
  // while the parts move on the exchange stream.  0 bits: serial exchanges.
  int exchange_chunk_bits = 2;
  bool exchange_chunk_select = true;  // chunk qubits chosen per exchange (state.cu choose_chunk)
  int exchange_ctas = 0;     // grid of the (device / P2P) exchange swap kernels; 0: full grid
  int exchange_rate_gbs = 0; // > 0: the swap kernel paced to this many GB/s per direction
                             // (a link-rate emulation for the one-GPU virtual partition)
  int fuse_tile_qubits = 12;
  int fuse_low_qubits = 0;   // contiguous low qubits of a fused tile (chunk = 2^L amps);
                             // 0: auto, 7 or 6 by planned pass count (fused_kernels.cu)
  bool fuse_reorder = true;  // commutation-aware scheduling of fused passes
  // Tiles with more chunks load/store directly (no TMA).  Measured on B200 at
  // n=30 (profiles/r01_fused_variants.md): TMA with parallel issue from warp 0
  // beats direct loads for every chunk count up to 128, so TMA is the default.
  int fuse_tma_max_chunks = 256;
  int items_per_thread = 0;  // 0 = library default
  int jit_threads = 0;       // threads per CTA of compiled passes (128, 256, 512; 0: per pass)
  int lane_group = 1;  // 1: dense 4x4 on qubits {1, 2} via k_lanegroup; 2: every dense 4x4/8x8
                       // with targets in [1, 5] (test / measurement); 0: never
  int stream_max_prefix = 0;  // lfqs_run_circuit_streamed: max gates run per piece (0: all)
  bool fuse_phase_split = false;     // phase tables: tile-invariant / tile-dependent groups
  bool fuse_merge_commuting = true;  // merge same-qubit 1-target gates across commuting gates
  int auto_extra_passes = 0;  // internal: passes planned outside the auto-tiled run
  int fuse_perm = 1;         // trailing SWAP runs as one bit-permutation pass (k_bitperm)
                             // with at most this many tile bits (0: off, 1: auto)
  bool exchange_wide = true;  // device / P2P transports: exchanges at any local position >= 3
  bool canon_fuse = true;     // canonicalising SWAP passes fused (State::canonicalize)
  bool fuse_phase_extract = true;  // global phases of dense 1-target gates (extract_phases)
  bool fuse_h_scale = true;   // Hadamard scales of a fused pass folded into one (fold_h_scales)
  bool fuse_merge_2q = true;  // fold dense 1-target gates into neighbouring 2-target gates
  bool jit_lane_move = true;     // compiled passes may move lane bits >= 3 into registers
  bool jit_greedy_place = true;  // compiled passes: remaps fill every register position
  bool jit_partial_rt = true;    // compiled passes: round trips move only re-placed amplitudes
  bool jit_lane_pool = false;    // compiled passes: movable lanes serve gates like registers
  bool jit_lane_reg2 = true;     // compiled passes: SWAP/U4 on a lane bit + a register bit by shuffles
};

// One launch worth of work on a contiguous shard.
struct LaunchCtx {
  void* amps;              // interleaved shard: complex128 (double2) or complex64 (float2)
  int n_local;             // qubits in the shard
  cudaStream_t stream;
  uint64_t* launch_counter;
  const Options* opt;
  bool c64;                // amplitudes are complex64 (NEXT-4 precision variant)
  // LFQS_FUSE_PHASE: runs of diagonal gates in a fused pass are merged into
  // per-tile phase tables (one lookup + one multiply per amplitude per table).
  bool phase_tables = false;
  // LFQS_FUSE_JIT: each fused pass runs as its own compiled kernel (jit.cpp).
  bool jit = false;
  // Plan and compile only (lfqs_jit_precompile): no kernel is launched.
  bool dry_run = false;
  // Count the passes of the fused schedule only (no programs, no launches).
  bool plan_only = false;
  // Structure-of-arrays shard (LFQS_STATE_SOA): real plane, then imaginary plane.
  bool soa = false;
};

// Raises a kernel's dynamic shared memory limit once per device.
void ensure_smem_attr(const void* kernel, int bytes);

// Applies one decoded gate whose targets are all < n_local (controls < n_local).
void launch_gate(const LaunchCtx& ctx, const Decoded& g);
// The same on a structure-of-arrays shard (soa_kernels.cu).
void launch_gate_soa(const LaunchCtx& ctx, const Decoded& g);
// Half-shard swap for the global-qubit exchange: the l=1 half of the shard at
// ctx.amps with the l=0 half of the shard partner_offset_amps further on, restricted to
// the amplitudes whose bits fix_zero are 0 and fix_one are 1 (a block of an overlapped
// exchange, or one rank's share of the pairs; <= 4 fixed bits, none at l).
// ctas > 0: a grid of at most that many CTAs (persistent grid-stride kernel) -- for
// exchanges overlapped with local passes on another stream.
void launch_half_swap(const LaunchCtx& ctx, int l, uint64_t partner_offset_amps, int ctas = 0,
                      uint64_t fix_zero = 0, uint64_t fix_one = 0);

// Fused staging of gates[begin..): applies the longest prefix that fits one tile
// program in one HBM pass; false if fewer than two gates fuse (fused_kernels.cu).
bool run_fused_circuit(const LaunchCtx& ctx, const std::vector<Decoded>& gates, size_t begin,
                       size_t end, int tile_qubits, size_t* consumed);
// Whole-list fused execution with exact-commutation reordering (fused_kernels.cu).
void run_fused_schedule(const LaunchCtx& ctx, const std::vector<Decoded>& gates, int tile_qubits);

// A qubit permutation that is an involution (a run of disjoint-cycle SWAPs: QFT's final
// bit reversal) applied in one pass (fused_kernels.cu k_bitperm): the tile bits are closed
// under it, so tile t's data goes to tile sigma(t) with its bits permuted inside the tile.
struct PermArgs {
  int ns = 0, nf = 0;      // tile bits, tile-index bits
  uint8_t sbit[16] = {};   // element bit k <-> position sbit[k] (ascending)
  uint8_t sdst[16] = {};   // element bit k of the source goes to element bit sdst[k]
  uint8_t fbit[48] = {};   // tile-index bit k <-> position fbit[k] (ascending)
  uint8_t fdst[48] = {};   // tile-index bit k goes to tile-index bit fdst[k]
  int f0 = -1;             // >= 0: the tile-index bits are positions f0 .. f0 + nf - 1
  int rev = 0;             // 1: sigma reverses the tile-index bits (fdst[k] = nf - 1 - k)
  int s_lo = -1, s_h0 = 0; // >= 0: tile bits = positions [0, s_lo) and [s_h0, s_h0 + ns - s_lo)
  int srev = 0;            // 1: the tile bits are reversed too (sdst[k] = ns - 1 - k)
};

// One pass of a fused schedule: a single gate's class kernel, a fused tile program, or a
// bit-permutation pass.
struct FProg;  // fused_prog.h
struct FusedPass {
  std::shared_ptr<PermArgs> perm;  // bit-permutation pass (a trailing run of SWAPs)
  int gate = -1;                 // single-gate pass: index into the gate list
  std::shared_ptr<FProg> prog;   // fused pass (tile program)
  std::string key;               // compiled-pass cache key (LFQS_FUSE_JIT), else empty
  int K = 0;                     // tile qubits of prog
  uint64_t qmask = 0;            // qubits the pass's gates touch (targets | controls)
  uint64_t nd_mask = 0;          // targets of its non-diagonal gates (the qubits it mixes)
};
// Plans (and for LFQS_FUSE_JIT compiles) the passes run_fused_schedule would launch.
void plan_fused_schedule(const LaunchCtx& ctx, const std::vector<Decoded>& gates, int tile_qubits,
                         std::vector<FusedPass>& out);
// Launches one planned pass on ctx: the whole shard, or any block of it (amps offset,
// n_local) that contains every qubit in ps.qmask.
void launch_fused_pass(const LaunchCtx& ctx, const std::vector<Decoded>& gates,
                       const FusedPass& ps);
// Block v of the chunk qubits `chunk` (<= 3 positions of the shard): the amplitudes whose
// chunk bits, read in ascending position order, spell v.  A pass can run block by block
// when it does not mix the chunk qubits (pass_blockwise): a fused pass whose tile holds
// none of them (they are fixed bits of its tile index), or a single gate when the chunk
// qubits are the top ones of the shard (a contiguous block).  Controls and diagonal
// entries on them are resolved for the block -- exactly the ops the whole-shard pass
// applies to these amplitudes, with the same kernels and formulas.
bool pass_blockwise(const FusedPass& ps, uint64_t chunk, int n_local);
void launch_fused_pass_part(const LaunchCtx& ctx, const std::vector<Decoded>& gates,
                            const FusedPass& ps, uint64_t chunk, uint64_t v);

// Reductions (C9): d_out[v], v < 2^nq (nq <= 20, bit s of v = bit qubits[s]); one read
// pass over the shard whatever nq is; deterministic (fixed grid and summation order).
// d_partials must hold probs_partials_doubles(ctx.n_local, qubits, nq) doubles.
void launch_probs(const LaunchCtx& ctx, const int* qubits, int nq, double* d_partials,
                  size_t partials_doubles, double* d_out);
size_t probs_partials_doubles(int n_local, const int* qubits, int nq);

// Projective collapse: a[k] = (k & mask) == pat ? scale * a[k] : 0 (all zero if
// zero_all: the rank's global bits do not match the outcome).
void launch_collapse(const LaunchCtx& ctx, uint64_t mask, uint64_t pat, double scale, bool zero_all);

// Initialisers.
void launch_init_basis(const LaunchCtx& ctx, int64_t local_index);  // -1: all zero
void launch_init_random(const LaunchCtx& ctx, uint64_t seed, uint64_t global_offset);

}  // namespace lfqs
