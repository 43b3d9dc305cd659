/*
 * lfqs.h -- C ABI of the B200-native LFQS state-vector gate-application library.
 *
 * What it computes: the state after each gate of a circuit,
 *     S_out = G . S_in                                   (Eq. 2)
 *     G     = I_L (x) M (x) I_R                          (Eq. 1)
 *     G_q1q2 = sum_ij X_ij (x) I_N (x) U_ij              (Eq. 5, non-adjacent)
 *     CU    = |0><0| (x) I + |1><1| (x) U                (Fig. 1)
 * applied in place to a 2^n complex128 Array-of-Structs state
 * (PAPER.md:503), gate after gate (Eq. 3), followed by
 * measurement probabilities.  Every gate is one pass over the
 * changed part of the state -- the matrix is never built (vector fusion,
 * PAPER.md:401-407) -- with code specialised per sparsity class (static matrix
 * specialisation): diagonal, permutation, dense 2x2/4x4/8x8.
 *
 * Conventions (readings R1, R2, R7):
 *   - qubit q is bit q of the amplitude index (little-endian).  The paper's
 *     Kronecker-left qubit i is q = n-1-i.
 *   - an m-target gate's local index is j = sum_s bit(t_s) << (m-1-s):
 *     targets[0] is the most significant bit (Eq. 5's q1).
 *   - controls: the gate acts where every control bit is 1.  No negative controls.
 *   - amplitudes are interleaved (re, im) doubles, 16 bytes each.
 *
 * Errors: every call returns lfqs_status (0 = OK) and never throws or aborts
 * across the ABI.  On failure lfqs_last_error() (thread-local) describes it.
 * lfqs_apply_gate / lfqs_run_circuit / lfqs_state_init_* are ASYNCHRONOUS on the
 * state's CUDA stream: kernel faults surface as LFQS_ERR_CUDA at the next
 * synchronising call (lfqs_measure_probs, lfqs_copy_out, lfqs_synchronize).
 * There is no CPU fallback: without a usable CUDA device every call that needs
 * one returns LFQS_ERR_CUDA.
 *
 * Ownership: states returned by lfqs_state_create* own their device memory;
 * lfqs_state_wrap borrows it (the caller keeps it alive until destroy).  Every
 * pointer argument is read or written only during the call.  Output buffers are
 * caller-allocated with explicit lengths.
 */
#ifndef LFQS_ABI_INCLUDED_
#define LFQS_ABI_INCLUDED_
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LFQS_ABI_VERSION 1

typedef enum {
  LFQS_OK = 0,
  LFQS_ERR_INVALID_ARG = -1,   /* bad qubit / arity / params / buffer length / handle */
  LFQS_ERR_OUT_OF_MEMORY = -2, /* 16 * 2^n_local bytes do not fit on the device */
  LFQS_ERR_CUDA = -3,          /* CUDA runtime or kernel error, or no device */
  LFQS_ERR_NCCL = -4,          /* NCCL error (distributed states) */
  LFQS_ERR_UNSUPPORTED = -5    /* valid request this build does not implement */
} lfqs_status;

/* Gate kinds.  Matrices: Fig. 1 for X, Y, Z, H, T, I, SWAP;
 * Nielsen & Chuang (cited PAPER.md:120) for the rest (R7):
 *   S = diag(1, i), SDG = diag(1, -i), T = diag(1, e^{i pi/4}), TDG = conj,
 *   RX(t) = [[c, -i s], [-i s, c]], RY(t) = [[c, -s], [s, c]],
 *   RZ(t) = diag(e^{-i t/2}, e^{i t/2})   (c = cos(t/2), s = sin(t/2)),
 *   PHASE(p) = diag(1, e^{i p}),
 *   U3(t, p, l) = [[c, -e^{i l} s], [e^{i p} s, e^{i(p+l)} c]]  (OpenQASM 2),
 *   SWAP |ij> = |ji>, UNITARYm = caller matrix, m = 1..3 targets.
 * Controlled forms: CNOT = X + 1 control, Toffoli = X + 2, CZ = Z + 1,
 * CPhase = PHASE + 1, CU = UNITARY1 + 1 control, MC-Z = Z + (n-1) controls. */
typedef enum {
  LFQS_I = 0, LFQS_X, LFQS_Y, LFQS_Z, LFQS_H, LFQS_S, LFQS_SDG, LFQS_T, LFQS_TDG,
  LFQS_RX, LFQS_RY, LFQS_RZ, LFQS_PHASE, LFQS_U3,
  LFQS_SWAP,
  LFQS_UNITARY1, LFQS_UNITARY2, LFQS_UNITARY3,
  LFQS_NUM_KINDS
} lfqs_gate_kind;

/* One gate of a circuit (72 bytes).  control_mask bit q = control on qubit q.
 * params: RX/RY/RZ/PHASE use params[0]; U3 uses (theta, phi, lambda).
 * matrix: UNITARYm only, 2^m x 2^m row-major interleaved (re, im), borrowed for
 * the duration of the call. */
typedef struct {
  int32_t kind;
  int32_t n_targets;
  int32_t n_controls;       /* must equal popcount(control_mask) */
  int32_t _pad0;
  int32_t targets[3];
  int32_t _pad1;
  uint64_t control_mask;
  double params[3];
  const double* matrix;
} lfqs_gate;

/* lfqs_run_circuit flags */
#define LFQS_FUSE_NONE      0u  /* one pass per gate: every intermediate state exists */
#define LFQS_FUSE_LOW       1u  /* shared-memory staging of consecutive low-qubit / diagonal gates */
/* With LFQS_FUSE_LOW: inside a fused pass, runs of diagonal gates (which
 * commute, P:441-445 classes) are merged into per-tile phase tables -- each
 * table entry is the product of the run's factors for one pattern of <= 8 tile
 * bits, built once per tile; every amplitude then takes one lookup and one
 * complex multiply per table instead of one per gate.  The product is the same
 * diagonal (Eq. 3), rounded in a different order, so diagonal
 * results are then within rounding (<= 1e-12 abs), not value-exact. */
#define LFQS_FUSE_PHASE     2u
/* With LFQS_FUSE_LOW: every fused pass is compiled into its own kernel (the
 * pass's gate program emitted as PTX with indices, predicates and op types
 * resolved, coefficients left as a kernel parameter; compiled in-process,
 * in parallel, and cached by structure) instead of being interpreted per tile
 * -- the paper's compile-the-circuit approach applied to
 * fused passes.  Results are bit-identical to the interpreted passes; the
 * first run of a new circuit structure pays the compile time (~0.1-1 s per
 * pass, on all host cores).  Compile failure: LFQS_ERR_CUDA. */
#define LFQS_FUSE_JIT       4u
#define LFQS_FUSE_DEFAULT   LFQS_FUSE_LOW

typedef struct lfqs_state lfqs_state;  /* opaque */

/* ---- lifetime ------------------------------------------------------------- */
/* Allocates 16 * 2^n bytes on `device` (cudaMalloc) and initialises |0...0>.
 * n_qubits in [1, 36].  stream: a cudaStream_t the state's work is ordered on,
 * or NULL for a library-created non-blocking stream.
 * LFQS_ERR_OUT_OF_MEMORY if it does not fit. */
lfqs_status lfqs_state_create(int n_qubits, int device, void* cuda_stream, lfqs_state** out);
/* Borrow caller device memory (e.g. a torch complex128 tensor of 2^n elements).
 * dev_ptr must be 32-byte aligned: the kernels read and write two adjacent
 * amplitudes per 32-B vector access (LDG/STG.256) and move tiles with TMA bulk
 * copies; a merely element-aligned view (torch t[1:]) returns
 * LFQS_ERR_INVALID_ARG.  cudaMalloc / torch allocations are 256-B aligned.
 * The contents are left as they are; the caller keeps ownership and must keep
 * the buffer alive until lfqs_state_destroy. */
lfqs_status lfqs_state_wrap(int n_qubits, int device, void* dev_ptr, void* cuda_stream,
                            lfqs_state** out);
/* Precision / partition variants (NEXT-4).  flags: LFQS_STATE_C64 stores
 * complex64 amplitudes (8 bytes: float re, im) instead of complex128 -- half
 * the HBM traffic per gate and one more qubit per GPU; arithmetic is fp32 (the
 * diagonal multiply RN without FMA, as in complex128).  world >= 2 creates a
 * single-GPU virtual partition (see lfqs_state_create_virtual).  The paper does
 * not state its precision (R5); complex128 stays the default. */
#define LFQS_STATE_C64 1u
/* LFQS_STATE_SOA: structure-of-arrays layout -- the paper's layout study (§6.6,
 * PAPER.md:501-505, 605-613): the real plane re[0, 2^n) followed by the
 * imaginary plane im[0, 2^n) in one allocation (a borrowed buffer holds the
 * same two planes), instead of interleaved (re, im) pairs.  Single shard only
 * (world >= 2: LFQS_ERR_UNSUPPORTED); gates run one pass each (lfqs_apply_gate,
 * lfqs_run_circuit with LFQS_FUSE_NONE; fused runs return
 * LFQS_ERR_UNSUPPORTED); copy_in/out keep interleaved host buffers;
 * probabilities, sampling and collapse are layout-independent (bit-identical
 * probabilities to an AOS state holding the same amplitudes). */
#define LFQS_STATE_SOA 2u
lfqs_status lfqs_state_create_ex(int n_qubits, int world, int device, void* cuda_stream,
                                 uint32_t flags, lfqs_state** out);
/* Borrow caller memory with the precision given by flags (LFQS_STATE_C64: a
 * torch complex64 tensor of 2^n elements).  Alignment: 32 B for complex128,
 * 16 B for complex64 (two amplitudes per vector access), else
 * LFQS_ERR_INVALID_ARG. */
lfqs_status lfqs_state_wrap_ex(int n_qubits, int device, void* dev_ptr, void* cuda_stream,
                               uint32_t flags, lfqs_state** out);
lfqs_status lfqs_state_destroy(lfqs_state* s);
/* Re-targets subsequent work to another stream (NULL = the library stream). */
lfqs_status lfqs_state_set_stream(lfqs_state* s, void* cuda_stream);

/* ---- distributed (one process per GPU, SPMD) ---------------- */
/* rank 0 creates an NCCL unique id (128 bytes); broadcast it (torch.distributed)
 * and pass it to lfqs_state_create_dist on every rank.  world must be a power of
 * two; rank r owns the 2^(n - log2 world) amplitudes whose top log2(world) bits
 * equal r ("global" qubits).  Gates on global qubits are handled transparently:
 * diagonal ones and controls rank-locally, others by a qubit-swap remap over
 * NCCL send/recv of half-shards. */
lfqs_status lfqs_dist_unique_id(uint8_t uid[128]);
lfqs_status lfqs_state_create_dist(int n_qubits, int rank, int world, const uint8_t uid[128],
                                   int device, void* cuda_stream, lfqs_state** out);
/* Peer-memory (CUDA IPC) sharding, NEXT-3: the same planner, with every global-
 * qubit exchange done by ONE in-place swap kernel that loads and stores the
 * partner's shard directly over NVLink / NVSwitch (no staging buffer, no NCCL),
 * each partner swapping half of the pairs, ordered by device-side flags.
 * Measurement histograms are summed across ranks in rank order (deterministic).
 * Setup, on every rank (SPMD):
 *   1. lfqs_state_create_p2p(n, rank, world, device, stream, flags, &s)
 *      (flags: 0 or LFQS_STATE_C64; the shard is |0..0>'s part, synchronised);
 *   2. lfqs_state_p2p_handle(s, blob) -> LFQS_P2P_HANDLE_BYTES opaque bytes;
 *   3. all-gather the blobs in rank order (e.g. torch.distributed) and pass the
 *      world * LFQS_P2P_HANDLE_BYTES bytes to lfqs_state_p2p_attach(s, all).
 * Ranks may share a GPU (tests) or not; with different GPUs they must be
 * peer-capable (NVLink).  A rank that stops participating makes its partners'
 * barrier kernels time out after 30 s: the next synchronising call returns
 * LFQS_ERR_CUDA.  lfqs_state_destroy is collective (a barrier precedes the
 * unmapping).  Not capturable by lfqs_circuit_compile. */
#define LFQS_P2P_HANDLE_BYTES 256
lfqs_status lfqs_state_create_p2p(int n_qubits, int rank, int world, int device,
                                  void* cuda_stream, uint32_t flags, lfqs_state** out);
lfqs_status lfqs_state_p2p_handle(lfqs_state* s, uint8_t* blob);
lfqs_status lfqs_state_p2p_attach(lfqs_state* s, const uint8_t* all_blobs);
/* Single-GPU "virtual" partition: the same remap planner and exchange code
 * path with `world` shards in one allocation and device-to-device copies as the
 * transport.  For testing the distributed logic on one GPU. */
lfqs_status lfqs_state_create_virtual(int n_qubits, int world, int device, void* cuda_stream,
                                      lfqs_state** out);

/* ---- state contents -------------------------------------------------------- */
/* |index> (global index). */
lfqs_status lfqs_state_init_basis(lfqs_state* s, uint64_t index);
/* Unnormalised counter-based random state: amplitude k = (u(2k), u(2k+1)) with
 * u(i) = (SplitMix64_output_i(seed) >> 11) * 2^-53 * 2 - 1 (same formula as
 * workloads/__init__.py).  Input generation for tests and benchmarks only. */
lfqs_status lfqs_state_init_random(lfqs_state* s, uint64_t seed);
/* Host <-> device copies of amplitudes [offset, offset+count) in canonical
 * (logical) qubit order; host buffers hold 2*count doubles.  Synchronous. */
lfqs_status lfqs_copy_in(lfqs_state* s, uint64_t offset, uint64_t count, const double* host);
lfqs_status lfqs_copy_out(lfqs_state* s, uint64_t offset, uint64_t count, double* host);
/* Same for complex64 states without conversion: 2*count floats (re, im).
 * LFQS_ERR_INVALID_ARG on a complex128 state.  (lfqs_copy_in/out also work on
 * complex64 states, converting on the host.) */
lfqs_status lfqs_copy_in_c64(lfqs_state* s, uint64_t offset, uint64_t count, const float* host);
lfqs_status lfqs_copy_out_c64(lfqs_state* s, uint64_t offset, uint64_t count, float* host);

/* ---- gates ------------------------------------------------------------------ */
/* One gate, one pass (no fusion).  targets/controls are qubit lists; params has
 * n_params doubles (must equal the kind's count); matrix for UNITARYm. */
lfqs_status lfqs_apply_gate(lfqs_state* s, int kind, const int* targets, int n_targets,
                            const int* controls, int n_controls, const double* params,
                            int n_params, const double* matrix);
/* Applies gates[0..n_gates) in order.  flags: LFQS_FUSE_*.  With
 * LFQS_FUSE_NONE the result equals n_gates lfqs_apply_gate calls bit for bit;
 * with fusion, permutation/diagonal results are still value-exact and dense
 * results agree within rounding (<= 1e-12 abs per amplitude); adding
 * LFQS_FUSE_PHASE moves diagonal results into the rounding class too.
 * Unknown flag bits: LFQS_ERR_INVALID_ARG. */
lfqs_status lfqs_run_circuit(lfqs_state* s, const lfqs_gate* gates, size_t n_gates, uint32_t flags);
/* Loads the whole state from host memory and runs a circuit, overlapping the upload with
 * the computation (the state's input is 2^n interleaved complex128 values -- for a sharded
 * state (one shard per rank, NCCL or p2p) this rank's 2^n_local amplitudes, every rank
 * calling with the same circuit -- host_interleaved
 * [2*k] = Re a_k, [2*k+1] = Im a_k, read during the call's asynchronous execution: keep it
 * alive and unchanged until the next synchronising call; page-locked memory for the copies
 * to overlap).  The state is uploaded in 2^chunk_bits pieces (split by its top chunk_bits
 * qubits, chunk_bits in [0, 8], < n_local) on an internal copy stream; each gate of the longest
 * prefix of the circuit whose targets and controls all lie below n_local - chunk_bits acts inside
 * each piece (Eq. 1: I on the piece index (x) the gate), so every piece runs that prefix as
 * soon as it has landed while later pieces are still being copied; the remaining gates run
 * on the whole state (sharded: through the planner's exchanges).  The qubit map is reset to
 * canonical.  Result: with LFQS_FUSE_NONE bit-identical to lfqs_copy_in of the
 * whole state followed by lfqs_run_circuit; with fusion the prefix and the rest are fused
 * separately, so (as for fusion itself) permutation/diagonal results stay value-exact and
 * dense ones agree within rounding.  Asynchronous like lfqs_run_circuit.  complex128 AOS
 * states, not virtual partitions (else LFQS_ERR_INVALID_ARG). */
lfqs_status lfqs_run_circuit_streamed(lfqs_state* s, const double* host_interleaved,
                                      const lfqs_gate* gates, size_t n_gates, uint32_t flags,
                                      int chunk_bits);

/* ---- captured circuits (CUDA graphs) ----------------------------------------- */
/* The circuit runner of Eq. 3 replayed without host work: the
 * launches lfqs_run_circuit(s, gates, n_gates, flags) would issue are captured
 * once into a CUDA graph; each lfqs_circuit_launch applies the whole circuit
 * again (same kernels, same arguments, so bit-identical to lfqs_run_circuit)
 * on the state's current stream, asynchronously.  For launch-bound sizes
 * (n <= ~20) this removes the per-gate host and launch cost.
 *   - compile issues no GPU work (the state is unchanged); a virtual partition
 *     is canonicalised first and the graph ends canonical, so replays compose;
 *   - distributed (NCCL) states: LFQS_ERR_UNSUPPORTED;
 *   - the circuit borrows the state: destroy it before lfqs_state_destroy;
 *   - *kernels_out (may be NULL) = kernels one launch replays. */
typedef struct lfqs_circuit lfqs_circuit;  /* opaque */
lfqs_status lfqs_circuit_compile(lfqs_state* s, const lfqs_gate* gates, size_t n_gates,
                                 uint32_t flags, lfqs_circuit** out, uint64_t* kernels_out);
lfqs_status lfqs_circuit_launch(lfqs_circuit* c);
lfqs_status lfqs_circuit_destroy(lfqs_circuit* c);

/* ---- measurement -------------------------------------------- */
/* probs_out[v] = sum over k with bit qubits[s] of k == bit s of v of |a_k|^2,
 * v in [0, 2^n_q).  n_q = 0 gives the squared norm.  n_q <= 20 (one
 * streaming pass per 10 measured qubits' worth of bins beyond the first 10).  Deterministic
 * (fixed reduction order).  probs_len >= 2^n_q.  Synchronous. */
lfqs_status lfqs_measure_probs(lfqs_state* s, const int* qubits, int n_q, double* probs_out,
                               size_t probs_len);

/* Sampling without collapse (reading R15: the paper's "followed by measurement",
 * P:122).  With p = lfqs_measure_probs(qubits) and c[v] = p[0] + ... + p[v]
 * (ascending), shot i returns the smallest v with u_i * c[last] < c[v].  The
 * uniforms u_i in [0, 1) are caller-provided (the random numbers the method draws
 * are inputs).  outcomes has `shots` entries.  Synchronous. */
lfqs_status lfqs_measure_sample(lfqs_state* s, const int* qubits, int n_q, const double* uniforms,
                                size_t shots, uint64_t* outcomes);
/* Projective measurement with a chosen outcome (mid-circuit measurement):
 * amplitudes whose measured bits differ from `outcome` become 0, the others are
 * multiplied by 1/sqrt(P(outcome)).  *probability (optional) receives P(outcome).
 * LFQS_ERR_INVALID_ARG if P(outcome) == 0.  Synchronous. */
lfqs_status lfqs_measure_collapse(lfqs_state* s, const int* qubits, int n_q, uint64_t outcome,
                                  double* probability);

/* ---- planning (host only: no GPU needed) ------------------------------------ */
/* The distributed planner as a query: the physical
 * operations rank `rank` of `world` performs for gates[0..n_gates), in order.
 *   kind = LFQS_PLAN_LOCAL: apply `gate` to the rank's shard of n - log2(world)
 *     local qubits.  The gate is already rank-specialised (global controls
 *     resolved, diagonals on global qubits folded) and always expressed as
 *     UNITARYm with gate.matrix pointing at this op's `matrix` (row-major
 *     interleaved).  Ranks whose global controls are 0 get no op.
 *   kind = LFQS_PLAN_EXCHANGE: swap local bit position l with global position g:
 *     this rank exchanges, in place, its amplitudes whose bit l equals
 *     1 - bit (g - n_local) of `rank` with the same positions of partner rank
 *     rank ^ 2^(g - n_local).
 * canonicalize: bit 0 appends the ops that restore the identity qubit map; bit 1
 * (LFQS_PLAN_WIDE) plans with the device / P2P transports' exchange window (any local
 * position >= 3, LFQS_OPT_EXCHANGE_WIDE) instead of the NCCL-sized top window.
 * Returns LFQS_ERR_INVALID_ARG with *n_ops = required length if capacity is
 * too small.  The ops array must outlive any use of gate.matrix. */
#define LFQS_PLAN_LOCAL 0
#define LFQS_PLAN_EXCHANGE 1
#define LFQS_PLAN_WIDE 2
typedef struct {
  int32_t kind;
  int32_t l;
  int32_t g;
  int32_t _pad;
  lfqs_gate gate;
  double matrix[128];
} lfqs_plan_op;
lfqs_status lfqs_plan_circuit(int n_qubits, int world, int rank, const lfqs_gate* gates,
                              size_t n_gates, int canonicalize, lfqs_plan_op* ops,
                              size_t capacity, size_t* n_ops);

/* Ahead-of-time compile for LFQS_FUSE_JIT (host only, no device needed): plans the
 * fused passes lfqs_run_circuit(s, gates, n_gates, flags) would run on a
 * single-GPU n_qubits state (complex64 if c64 != 0, default tile options) and
 * compiles every pass not yet in the process-wide cache, in parallel.
 * *n_passes (may be NULL) receives the number of passes of the plan.
 * flags must contain LFQS_FUSE_LOW | LFQS_FUSE_JIT. */
lfqs_status lfqs_jit_precompile(int n_qubits, int c64, const lfqs_gate* gates, size_t n_gates,
                                uint32_t flags, uint64_t* n_passes);

/* ---- misc ------------------------------------------------------------------- */
lfqs_status lfqs_synchronize(lfqs_state* s);
/* n_qubits, local qubits, rank, world, and the device pointer of the local shard. */
lfqs_status lfqs_state_info(const lfqs_state* s, int* n_qubits, int* n_local, int* rank,
                            int* world, void** dev_ptr);
/* Global-qubit exchanges this state has issued so far (sharded states; 0 on one
 * GPU) and the bytes each one sends per rank and direction (16 or 8 * 2^(n_local-1)),
 * summed.  Counted when the exchange is enqueued (host side, no synchronisation). */
lfqs_status lfqs_state_exchange_stats(const lfqs_state* s, uint64_t* exchanges,
                                      uint64_t* bytes_per_rank);
/* Overlapped-exchange accounting (cumulative; benchmark / test use):
 * exchanges run in parts (LFQS_OPT_EXCHANGE_CHUNK_BITS > 0), local passes run block by block
 * around them (summed over the state's shards), exchanges whose chunk qubits were not the
 * top local qubits (LFQS_OPT_EXCHANGE_CHUNK_SELECT), and exchanges chained onto the
 * previous one (the whole run between them ran block by block).  Any pointer may be NULL. */
lfqs_status lfqs_state_overlap_stats(const lfqs_state* s, uint64_t* overlapped_exchanges,
                                     uint64_t* block_passes, uint64_t* strided_exchanges,
                                     uint64_t* chained_exchanges);
/* Number of kernels this state has launched so far (for benchmark accounting). */
lfqs_status lfqs_kernel_launches(const lfqs_state* s, uint64_t* count);
/* Number of state passes this state has run so far: one per fused pass or per single-gate
 * class kernel of lfqs_apply_gate / lfqs_run_circuit (an exchange's swap kernels and
 * a pass run block by block around an overlapped exchange count once) -- the
 * denominator of the per-pass HBM roofline (benchmark accounting). */
lfqs_status lfqs_state_pass_count(const lfqs_state* s, uint64_t* passes);
/* Tuning knobs (benchmark / test use): LFQS_OPT_LOWQ_SHUFFLE (1: warp-shuffle
 * path for targets < 5; default 0, measured no faster than the 32-byte path), LFQS_OPT_FUSE_TILE_QUBITS (k of the staging
 * tile, default 12). */
#define LFQS_OPT_LOWQ_SHUFFLE 1
#define LFQS_OPT_FUSE_TILE_QUBITS 2
#define LFQS_OPT_ITEMS_PER_THREAD 3
#define LFQS_OPT_WIDE256 4 /* 1: two adjacent groups per thread, 32-byte accesses (default 1) */
#define LFQS_OPT_FUSE_LOW_QUBITS 5 /* contiguous low qubits of a fused tile, [3, 12], or 0
                                      (default): 7, or 6 when planning the circuit with 6
                                      saves >= 20 % of the passes; the other tile qubits
                                      are claimed by the fused gates */
#define LFQS_OPT_FUSE_TMA_MAX_CHUNKS 6 /* tiles of at most this many chunks move by TMA bulk
                                          copies, larger ones by direct loads (default 256) */
#define LFQS_OPT_FUSE_REORDER 7 /* 1: fused passes may take later gates that commute exactly
                                   with the skipped ones (default 1); 0: prefixes only */
#define LFQS_OPT_JIT_THREADS 8 /* threads per CTA of LFQS_FUSE_JIT passes: 256 (default), 512
                                   (twice the warps per SM, half the amplitudes per thread) or
                                   128 (one more register-held tile bit, 3 CTAs per SM) */
#define LFQS_OPT_JIT_LANE_MOVE 9 /* 1 (default): compiled passes may move the lane tile bits >= 3
                                     (complex64: >= 4) into register positions, so 1-target
                                     gates on them run in registers instead of by warp
                                     shuffles; bit-identical results either way */
#define LFQS_OPT_FUSE_MERGE_COMMUTING 10 /* 1 (default): inside a fused pass, a 1-target gate
                                     merges (host matrix product) into the last earlier gate
                                     touching any of its qubits when that is a 1-target gate on
                                     the same target with the same controls and one of the two
                                     is dense; 0: only directly adjacent runs merge.  Changes
                                     rounding only (dense tolerance class) */
#define LFQS_OPT_JIT_GREEDY_PLACE 11 /* 1 (default): a compiled pass's tile round trip moves
                                     into register positions the targets of the longest run
                                     of upcoming gates that fit them (fewest round trips);
                                     0: only the current gate's targets (furthest-next-use
                                     eviction).  Bit-identical results either way */
#define LFQS_OPT_LANE_GROUP 12 /* 1 (default): per-gate dense 4x4 gates on qubits {1, 2}
                                  run as coalesced warp chunks with shuffle exchange (the
                                  group kernel's accesses are 128-B strided there); 2: also
                                  every other dense 4x4 / 8x8 gate with targets in 1..5;
                                  0: never.  Bit-identical results either way */
#define LFQS_OPT_JIT_LANE_REG2 13 /* 1 (default): in a compiled pass, a SWAP / 2-target dense
                                     gate with one target on a lane bit (0-4) and the other
                                     on a register-held tile bit runs by warp shuffles in
                                     registers instead of as a shared-memory op; 0: shared
                                     memory.  Bit-identical results either way */
#define LFQS_OPT_JIT_LANE_POOL 14 /* 1: with greedy placement, lane-move and lane/register
                                     2-target gates on, the movable lane positions serve
                                     1-target and 2-target gates by shuffles like register
                                     positions (more tile bits per placement, fewer tile
                                     round trips); 0 (default): registers only.
                                     Bit-identical results either way */
#define LFQS_OPT_JIT_PARTIAL_RT 15 /* 1 (default): a compiled pass's tile round trip stores
                                      and reloads only the amplitudes whose (thread, slot)
                                      changes (a swap of k tile-bit positions moves 1 - 2^-k
                                      of the tile; complex128 states only -- measured
                                      slower for complex64); 0: the whole tile.
                                      Bit-identical */
#define LFQS_OPT_FUSE_PHASE_SPLIT 16 /* 1: LFQS_FUSE_PHASE groups the tile-invariant
                                        and the tile-dependent diagonals of a run separately
                                        (the latter -- e.g. QFT CPhases controlled from
                                        outside the tile -- become tables of few entries);
                                        0 (default; measured 1-9 % faster): one greedy
                                        grouping in program order.  Changes the rounding
                                        order only (phase-table tolerance) */
#define LFQS_OPT_STREAM_MAX_PREFIX 17 /* lfqs_run_circuit_streamed: at most this many prefix
                                         gates run piece by piece (0, default: the whole
                                         piece-local prefix); the rest run on the whole
                                         state.  Enough to cover the upload keeps the GPU
                                         busy with fewer, larger launches.  Same results */
#define LFQS_OPT_L2_FETCH_GRANULARITY 18 /* device-wide L2 fetch granularity hint in bytes
                                            (cudaLimitMaxL2FetchGranularity: 0, 32, 64 or
                                            128) for the state's device; measurement knob */
#define LFQS_OPT_LINE_READS 19 /* 1 (default): per-gate kernels whose gate fixes qubit 1 or 2
                                  (a control, or the pattern of a one-entry diagonal) read
                                  whole 128-B lines coalesced and store only the touched
                                  groups (DRAM reads whole lines anyway:
                                  tools/probe_sparse.cu); 0: read only the touched groups.
                                  Bit-identical results either way */
#define LFQS_OPT_EXCHANGE_CHUNK_BITS 20 /* sharded states: each global-qubit exchange is
                                  split into 2^value parts (value in [0, 3]) by `value`
                                  local "chunk" qubits (LFQS_OPT_EXCHANGE_CHUNK_SELECT; the
                                  planner never uses the top 2 as exchange positions,
                                  whatever the value, so the plan does not depend on it;
                                  an exchange at a position among the top `value` runs
                                  serially when the chunk qubits are the top ones);
                                  the local passes right before it and right after it that
                                  do not mix those qubits run part by part on the state's
                                  stream while the parts move on an exchange stream (NCCL:
                                  the communicator's stream) -- exchange overlapped with
                                  local work.  Default 2; 0: serial exchanges.  The same
                                  passes and per-amplitude arithmetic as serial exchanges:
                                  bit-identical results */
#define LFQS_OPT_EXCHANGE_CTAS 21 /* grid of the device / P2P exchange swap kernels (a
                                     persistent grid-stride kernel); 0 (default): one
                                     thread per pair.  A small grid saturates NVLink and
                                     leaves the SMs to the overlapped local passes */
#define LFQS_OPT_FUSE_MERGE_2Q 22 /* 1 (default): inside a fused pass, a dense 1-target gate
                                     adjacent (in commuting order) to a 2-target gate on a
                                     superset of its qubit is multiplied into the 4x4 on the
                                     host, and two 2-target gates on the same pair are
                                     multiplied, when the product has no more complex
                                     multiply-adds per amplitude than the separate gates
                                     (e.g. Sycamore-like 1-target layers into fSim).
                                     Rounding changes only (dense tolerance class) */
#define LFQS_OPT_EXCHANGE_CHUNK_SELECT 23 /* 1 (default): fused runs on the device / P2P
                                  transports choose each exchange's chunk qubits among the
                                  local qubits at or above the fused tile size, the ones
                                  left unmixed by the most planned ops around the exchange
                                  (and keep the previous exchange's when the run between
                                  the two leaves them unmixed: the run then flows block by
                                  block from one exchange into the next); rank-independent
                                  (decided from the plan).  0, per-gate runs and NCCL: the
                                  top local qubits.  Bit-identical results either way */
#define LFQS_OPT_EXCHANGE_RATE_GBS 24 /* > 0: the device / P2P exchange swap kernel (grid
                                  LFQS_OPT_EXCHANGE_CTAS, 64 if 0) paces itself to this many
                                  GB/s per direction -- a link-rate emulation, so that the
                                  one-GPU virtual partition shows how much of an NVLink
                                  exchange the overlapped local passes hide; default 0
                                  (unpaced).  Same results */
#define LFQS_OPT_FUSE_H_SCALE 25 /* 1 (default): in a fused pass with k >= 2 unpredicated
                                  Hadamards, one carries the whole scale (1/sqrt 2)^k and the
                                  others compute the unscaled butterfly (a + b, a - b): 2 FP64
                                  multiplies per amplitude fewer per Hadamard.  Rounding
                                  changes only (dense tolerance class) */
#define LFQS_OPT_FUSE_PHASE_EXTRACT 26 /* 1 (default): a fused pass's uncontrolled dense
                                  1-target gates that are a global phase times a real matrix
                                  or a real-diagonal / imaginary-off-diagonal one (sqrt X,
                                  sqrt Y, ...) run in that 4-operation form, the phases
                                  multiplied into one other dense 1-target gate of the pass.
                                  Rounding changes only (dense tolerance class) */
#define LFQS_OPT_CANON_FUSE 27 /* sharded states, 1 (default): the local SWAP / X passes
                                  that restore the canonical qubit map (copy_in / copy_out /
                                  the end of a compiled circuit) run fused, a run of them in
                                  one tile pass, and their exchanges overlap like a circuit's;
                                  0: one pass per SWAP.  Moves only: bit-identical */
#define LFQS_OPT_FUSE_PERM 28 /* 1 (default, auto tile size): a fused run ending in >= 3
                                  uncontrolled SWAPs whose composition is an involution
                                  (QFT's bit reversal) applies them as one bit-permutation
                                  pass (tile pairs closed under the permutation); 8..12: that
                                  many tile bits at most; 0: off.  Moves only: bit-identical */
#define LFQS_OPT_EXCHANGE_WIDE 29 /* sharded states on the device / P2P transports, 1
                                  (default): the planner may exchange a global qubit with any
                                  local position >= 3 (Belady over all of them; the swap kernel
                                  moves any block in place), and canonicalisation needs no
                                  SWAP pass to bring a low qubit to the top first; 0: the top
                                  window the NCCL transport uses.  Results within tolerance
                                  (a different plan) */
lfqs_status lfqs_set_option(lfqs_state* s, int option, int64_t value);
const char* lfqs_last_error(void);
int lfqs_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* LFQS_ABI_INCLUDED_ */
