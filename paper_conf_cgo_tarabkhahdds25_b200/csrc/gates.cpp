// gates.cpp -- the library's gate table and sparsity classification (host side).
//
// Static matrix specialisation (§4.6): the known matrix values pick
// the kernel -- diagonal gates only scale, permutation gates only move
// amplitudes (CNOT/SWAP "eliminate unnecessary calculations"), dense
// gates do a 2^m x 2^m matvec per group (single_qbit).
//
// Matrices: Fig. 1 for X, Y, Z, H, T, I, SWAP; Nielsen & Chuang
// (cited P:120) for S, Rx, Ry, Rz, Phase, U3 (reading R7).  Angles
// use glibc cos/sin of theta/2 in double.  This file is the library's own copy;
// the oracle has a separate one (they share no code).
#include <cmath>
#include <cstring>

#include "lfqs_internal.h"

namespace lfqs {

int kind_arity(int kind) {
  if (kind < 0 || kind >= LFQS_NUM_KINDS) return -1;
  if (kind == LFQS_SWAP || kind == LFQS_UNITARY2) return 2;
  if (kind == LFQS_UNITARY3) return 3;
  return 1;
}

int kind_nparams(int kind) {
  switch (kind) {
    case LFQS_RX: case LFQS_RY: case LFQS_RZ: case LFQS_PHASE: return 1;
    case LFQS_U3: return 3;
    default: return 0;
  }
}

static inline cplx C(double re, double im) { return cplx{re, im}; }

static bool is_one(cplx z) { return z.re == 1.0 && z.im == 0.0; }
static bool is_zero(cplx z) { return z.re == 0.0 && z.im == 0.0; }

Decoded decode_gate(int n, int kind, const int* targets, int n_targets, uint64_t cmask,
                    const double* params, int n_params, const double* matrix) {
  Decoded g;
  const int m = kind_arity(kind);
  require(m > 0, "unknown gate kind " + std::to_string(kind));
  require(n_targets == m, "gate kind " + std::to_string(kind) + " takes " + std::to_string(m) +
                              " target(s), got " + std::to_string(n_targets));
  require(n_params == kind_nparams(kind), "gate kind " + std::to_string(kind) + " takes " +
                                              std::to_string(kind_nparams(kind)) + " param(s)");
  const bool unitary = kind >= LFQS_UNITARY1 && kind <= LFQS_UNITARY3;
  require(!unitary || matrix != nullptr, "UNITARYm needs a matrix");
  uint64_t tmask = 0;
  for (int s = 0; s < m; ++s) {
    require(targets[s] >= 0 && targets[s] < n, "target qubit out of range");
    require(!(tmask >> targets[s] & 1), "duplicate target qubit");
    tmask |= 1ull << targets[s];
    g.targets[s] = targets[s];
  }
  require(n >= 64 || (cmask >> n) == 0, "control qubit out of range");
  require((cmask & tmask) == 0, "a qubit is both target and control");
  g.kind = kind;
  g.m = m;
  g.cmask = cmask;

  cplx* M = g.M;
  const int d = 1 << m;
  for (int i = 0; i < d * d; ++i) M[i] = C(0, 0);
  const double s = M_SQRT1_2;
  const double p0 = n_params > 0 ? params[0] : 0.0;
  const double p1 = n_params > 1 ? params[1] : 0.0;
  const double p2 = n_params > 2 ? params[2] : 0.0;
  const double c = std::cos(p0 / 2.0), sn = std::sin(p0 / 2.0);
  switch (kind) {
    case LFQS_I: M[0] = M[3] = C(1, 0); break;
    case LFQS_X: M[1] = M[2] = C(1, 0); break;
    case LFQS_Y: M[1] = C(0, -1); M[2] = C(0, 1); break;
    case LFQS_Z: M[0] = C(1, 0); M[3] = C(-1, 0); break;
    case LFQS_H: M[0] = M[1] = M[2] = C(s, 0); M[3] = C(-s, 0); g.is_h = true; break;
    case LFQS_S: M[0] = C(1, 0); M[3] = C(0, 1); break;
    case LFQS_SDG: M[0] = C(1, 0); M[3] = C(0, -1); break;
    case LFQS_T: M[0] = C(1, 0); M[3] = C(s, s); break;
    case LFQS_TDG: M[0] = C(1, 0); M[3] = C(s, -s); break;
    case LFQS_RX: M[0] = M[3] = C(c, 0); M[1] = M[2] = C(0, -sn); break;
    case LFQS_RY: M[0] = M[3] = C(c, 0); M[1] = C(-sn, 0); M[2] = C(sn, 0); break;
    case LFQS_RZ: M[0] = C(c, -sn); M[3] = C(c, sn); break;
    case LFQS_PHASE: M[0] = C(1, 0); M[3] = C(std::cos(p0), std::sin(p0)); break;
    case LFQS_U3:
      M[0] = C(c, 0);
      M[1] = C(-(std::cos(p2) * sn), -(std::sin(p2) * sn));
      M[2] = C(std::cos(p1) * sn, std::sin(p1) * sn);
      M[3] = C(std::cos(p1 + p2) * c, std::sin(p1 + p2) * c);
      break;
    case LFQS_SWAP:
      M[0] = M[1 * 4 + 2] = M[2 * 4 + 1] = M[15] = C(1, 0);
      break;
    default:  // UNITARYm
      std::memcpy(M, matrix, sizeof(cplx) * d * d);
      break;
  }

  // Sparsity class.
  switch (kind) {
    case LFQS_I: g.cls = GClass::NOOP; break;
    case LFQS_Z: case LFQS_S: case LFQS_SDG: case LFQS_T: case LFQS_TDG:
    case LFQS_RZ: case LFQS_PHASE: g.cls = GClass::DIAG; break;
    case LFQS_X: g.cls = GClass::PERM_X; break;
    case LFQS_Y: g.cls = GClass::PERM_Y; break;
    case LFQS_SWAP: g.cls = GClass::PERM_SWAP; break;
    default: g.cls = GClass::DENSE; break;
  }
  if (g.cls == GClass::DIAG && m == 1 && is_one(M[0]) && is_one(M[3])) g.cls = GClass::NOOP;
  if (g.cls == GClass::DENSE && unitary) {
    // An explicit matrix that is exactly diagonal takes the diagonal path.
    bool diag = true;
    for (int r = 0; r < d; ++r)
      for (int q = 0; q < d; ++q)
        if (r != q && !is_zero(M[r * d + q])) diag = false;
    if (diag) g.cls = GClass::DIAG;
  }
  return g;
}

}  // namespace lfqs
