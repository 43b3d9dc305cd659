// soa_kernels.cu -- gate application on structure-of-arrays states (NEXT-4).
//
// The paper's layout study (§6.6) compares AOS -- one array
// of (re, im) pairs, the default here and the paper's faster layout on CPU
// (1.19x) -- with SOA, "two arrays (of float numbers)" for the real and the
// imaginary parts.  An SOA state (LFQS_STATE_SOA) holds the real plane
// re[0, 2^n) followed by the imaginary plane im[0, 2^n) in one allocation.
//
// One kernel serves every gate class: thread items expand a free index into the
// group's base index by bit insertion, gather the
// group's 2^m amplitudes from both planes (8- or 4-byte accesses, coalesced
// across the warp for targets >= 1), apply the class update and scatter back:
//   * DIAG: a[k] *= d[loc(k)] with the pinned RN product (R8), only
//     entries != 1 -- value-exact against the oracle like the AOS kernels;
//   * PERM / DENSE: w = M v with FMA, ascending column order (exact for
//     permutation matrices: products with 0 and 1 are exact).
#include <cuda_runtime.h>

#include <cstring>

#include "cx.cuh"
#include "lfqs_internal.h"

namespace lfqs {
namespace {

constexpr int kThreads = 256;

struct SoaGate {
  InsertPlan ip;       // zeros at targets and controls, ones at controls
  uint64_t off[8];     // offset of local index j: sum of its target bits
  double2 m[64];       // DENSE: L x L row-major; DIAG: the L diagonal entries
};

template <class S, int L, bool DIAG>
__global__ void __launch_bounds__(kThreads) k_soa(S* __restrict__ re, S* __restrict__ im,
                                                  uint64_t n_groups, const __grid_constant__ SoaGate g) {
  using C = cx<S>;
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t gi = (uint64_t)blockIdx.x * kThreads + threadIdx.x; gi < n_groups; gi += stride) {
    uint64_t k = gi;
    for (int i = 0; i < g.ip.np; ++i) {
      const int p = g.ip.pos[i];
      const uint64_t lo = k & ((1ull << p) - 1);
      k = ((k - lo) << 1) | lo;
    }
    k |= g.ip.ones;
    C v[L];
#pragma unroll
    for (int j = 0; j < L; ++j) v[j] = mk<S>(__ldcs(re + k + g.off[j]), __ldcs(im + k + g.off[j]));
    if (DIAG) {
#pragma unroll
      for (int j = 0; j < L; ++j) {
        const double2 d = g.m[j];
        if (d.x == 1.0 && d.y == 0.0) continue;
        const C z = cmul_rn(mk<S>((S)d.x, (S)d.y), v[j]);
        __stcs(re + k + g.off[j], z.x);
        __stcs(im + k + g.off[j], z.y);
      }
    } else {
#pragma unroll
      for (int j = 0; j < L; ++j) {
        C acc = mk<S>(0, 0);
#pragma unroll
        for (int i = 0; i < L; ++i) cfma(acc, mk<S>((S)g.m[j * L + i].x, (S)g.m[j * L + i].y), v[i]);
        __stcs(re + k + g.off[j], acc.x);
        __stcs(im + k + g.off[j], acc.y);
      }
    }
  }
}

template <class S, int L, bool DIAG>
void run_soa(const LaunchCtx& ctx, uint64_t n_groups, const SoaGate& g) {
  S* re = reinterpret_cast<S*>(ctx.amps);
  S* im = re + (1ull << ctx.n_local);
  uint64_t nb = (n_groups + kThreads - 1) / kThreads;
  if (nb > 148ull * 32) nb = 148ull * 32;
  if (nb == 0) nb = 1;
  k_soa<S, L, DIAG><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(re, im, n_groups, g);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

template <class S>
void launch_soa_t(const LaunchCtx& ctx, const Decoded& d) {
  if (d.cls == GClass::NOOP) return;
  SoaGate g;
  std::memset(&g, 0, sizeof g);
  uint64_t zmask = d.cmask;
  for (int s = 0; s < d.m; ++s) zmask |= 1ull << d.targets[s];
  for (int q = 0; q < 64; ++q)
    if ((zmask >> q) & 1) g.ip.pos[g.ip.np++] = q;
  g.ip.ones = d.cmask;
  const int L = 1 << d.m;
  for (int j = 0; j < L; ++j) {
    uint64_t o = 0;
    for (int s = 0; s < d.m; ++s)
      if ((j >> (d.m - 1 - s)) & 1) o |= 1ull << d.targets[s];
    g.off[j] = o;
  }
  const bool diag = d.cls == GClass::DIAG;
  if (diag) {
    for (int j = 0; j < L; ++j) g.m[j] = make_double2(d.M[j * L + j].re, d.M[j * L + j].im);
  } else {
    for (int j = 0; j < L * L; ++j) g.m[j] = make_double2(d.M[j].re, d.M[j].im);
  }
  const uint64_t n_groups = 1ull << (ctx.n_local - g.ip.np);
  switch (L) {
    case 2: diag ? run_soa<S, 2, true>(ctx, n_groups, g) : run_soa<S, 2, false>(ctx, n_groups, g); break;
    case 4: diag ? run_soa<S, 4, true>(ctx, n_groups, g) : run_soa<S, 4, false>(ctx, n_groups, g); break;
    default: diag ? run_soa<S, 8, true>(ctx, n_groups, g) : run_soa<S, 8, false>(ctx, n_groups, g); break;
  }
}

}  // namespace

void launch_gate_soa(const LaunchCtx& ctx, const Decoded& g) {
  if (ctx.c64)
    launch_soa_t<float>(ctx, g);
  else
    launch_soa_t<double>(ctx, g);
}

}  // namespace lfqs
