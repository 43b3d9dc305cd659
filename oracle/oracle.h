/*
 * oracle.h -- plain, slow, obviously-correct CPU oracle for LFQS state-vector
 * gate application (Tarabkhah, Delavar, Doosti, Shaikhha, CGO'25).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or constant with the CUDA library under
 * paper_conf_cgo_tarabkhahdds25_b200/ and neither includes the other.
 *
 * Citations: "P:N" = /root/reference/PAPER.md line N.
 *
 * Semantics (readings R1, R2, R7):
 *   - state: 2^n complex128, interleaved (re, im) = Array-of-Structs.
 *     basis index k, qubit q = bit q of k.  The paper's Kronecker-left qubit i is
 *     q = n-1-i (Eq. 1, verified against G_{0,2} at P:316-325).
 *   - a gate is an m-target matrix M (2^m x 2^m, m = 1..3); its local index is
 *     j = sum_s b_{t_s} 2^{m-1-s} (targets[0] = MSB, Eq. 5's q1).
 *   - controls: the gate acts on the subspace where every control bit is 1
 *     (CU = |0><0| (x) I + |1><1| (x) U).
 *   - pinned arithmetic (reading R8): complex multiply (ac - bd, ad + bc), every
 *     op round-to-nearest, no FMA (built with -ffp-contract=off), sums ascending
 *     from (+0, +0).
 */
#ifndef LFQS_ORACLE_H
#define LFQS_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Gate kinds (the oracle's own numbering; the Python wrapper maps names). */
enum {
  OR_I = 0, OR_X, OR_Y, OR_Z, OR_H, OR_S, OR_SDG, OR_T, OR_TDG,
  OR_RX, OR_RY, OR_RZ, OR_PHASE, OR_U3,
  OR_SWAP,
  OR_UNITARY1, OR_UNITARY2, OR_UNITARY3,
  OR_NKINDS
};

typedef struct {
  int32_t kind;
  int32_t n_targets;
  int32_t n_controls;     /* informational; control_mask is authoritative */
  int32_t _pad0;
  int32_t targets[3];
  int32_t _pad1;
  uint64_t control_mask;  /* bit q set = control on qubit q */
  double params[3];
  const double* matrix;   /* UNITARYm: 2^m x 2^m row-major interleaved re,im */
} oracle_gate;

/* Return codes: 0 ok, -1 invalid argument, -2 out of memory. */

/* Gate table (Fig. 1 + Nielsen & Chuang [27] for the rest).
 * Writes the 2^m x 2^m matrix (interleaved) into out (capacity >= 128 doubles),
 * *m_out = m. */
int oracle_gate_matrix(const oracle_gate* g, int* m_out, double* out);

/* ---- Tier A (n <= 12): dense 2^n x 2^n matrices ------------------------- */
/* Definition builder: G[r][c] = [r,c agree off T] * (ctrl(r) ? M[loc r][loc c] : delta). */
int oracle_dense_definition(int n, const oracle_gate* g, double* G);
/* Paper builder from Fig. 5 primitives: kron / eye / onehot / slice, Eq. 1 for
 * adjacent-or-single targets and Eq. 5 (recursively for 3 targets) otherwise;
 * controls as (I - Pi_C) + Pi_C G. */
int oracle_dense_kron(int n, const oracle_gate* g, double* G);
/* Eq. 4 route for a 2-target gate: SWAP chains bring t1 next to t0, apply the
 * adjacent gate, swap back (2N SWAPs for gap N). */
int oracle_dense_swap_route(int n, const oracle_gate* g, double* G);
/* out[r] = sum_{c ascending} G[r][c] * in[c]  (mvdot). */
void oracle_dense_matvec(int n, const double* G, const double* in, double* out);
/* C = A * B for square dim x dim complex matrices (ascending inner sum). */
void oracle_dense_matmul(int64_t dim, const double* A, const double* B, double* C);
/* C = kron(A, B) (Fig. 5 kron). A is ra x ca, B is rb x cb. */
void oracle_kron(int64_t ra, int64_t ca, const double* A, int64_t rb, int64_t cb,
                 const double* B, double* C);

/* ---- Tier B (any n): naive index loop, in place -------------------------- */
int oracle_apply_gate(int n, const oracle_gate* g, double* state);
int oracle_run_circuit(int n, const oracle_gate* gates, size_t n_gates, double* state);
/* Tier B restricted to a sparse set of amplitudes: idx[0..cnt) sorted ascending,
 * amps interleaved, updated in place.  Every present index whose gate group is
 * active must have its whole group present (else -1). */
int oracle_apply_gate_sparse(int n, const oracle_gate* g, size_t cnt,
                             const uint64_t* idx, double* amps);
/* Same loop with an OpenMP parallel-for over k (the P:465-467 pattern); used only
 * to time the oracle on the host cores. */
int oracle_apply_gate_omp(int n, const oracle_gate* g, double* state);
int oracle_omp_max_threads(void);
void oracle_omp_set_threads(int threads);  /* omp_set_num_threads (tests) */

/* ---- Measurement -------------------------------------------------- */
/* probs[v] = sum_{k: bits_Q(k) = v} |a_k|^2, pairwise (recursive halving) over k
 * in ascending order per bin; bit s of v = bit qubits[s] of k.  nq = 0 -> norm^2. */
int oracle_probs(int n, const double* state, const int* qubits, int nq, double* probs);

/* Sampling (reading R15): c[v] = p[0] + ... + p[v] (ascending, p from
 * oracle_probs); shot i = smallest v with u[i] * c[last] < c[v]. */
int oracle_measure_sample(int n, const double* state, const int* qubits, int nq,
                          const double* u, size_t shots, uint64_t* out);
/* Projective measurement with outcome `outcome`: amplitudes whose measured bits
 * differ become 0, the rest are multiplied by 1/sqrt(P(outcome)).
 * *p_out = P(outcome).  -1 if P(outcome) == 0. */
int oracle_measure_collapse(int n, double* state, const int* qubits, int nq, uint64_t outcome,
                            double* p_out);

/* ---- Counter-based input generator (same formula as workloads/) ----------- */
/* amplitudes start..start+count-1 of the SplitMix64 random state, interleaved. */
void oracle_fill_random(uint64_t seed, uint64_t start, uint64_t count, double* out);

#ifdef __cplusplus
}
#endif
#endif
