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
  InsertPlan ip;       // zeros at group bits and controls, ones at controls
  uint64_t off[8];     // offset of local index j: sum of its group bits
  double2 m[64];       // DENSE: L x L row-major; DIAG: the L diagonal entries
  int store_all;       // DIAG: rewrite unchanged entries too (whole 32-B sectors)
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
        if (d.x == 1.0 && d.y == 0.0) {
          if (g.store_all) {
            __stcs(re + k + g.off[j], v[j].x);
            __stcs(im + k + g.off[j], v[j].y);
          }
          continue;
        }
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

// Two adjacent groups per item when bit 0 is neither a group bit nor fixed: the
// base indices k, k + 1 share every other bit, so each plane access is one
// 2-element vector (16 B for complex128 planes), contiguous across the warp.
template <class S> struct V2;
template <> struct V2<double> { using T = double2; };
template <> struct V2<float> { using T = float2; };

template <class S, int L, bool DIAG>
__global__ void __launch_bounds__(kThreads) k_soa2(S* __restrict__ re, S* __restrict__ im,
                                                   uint64_t n_items, const __grid_constant__ SoaGate g) {
  using C = cx<S>;
  using VT = typename V2<S>::T;
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t it = (uint64_t)blockIdx.x * kThreads + threadIdx.x; it < n_items; it += stride) {
    uint64_t k = 2 * it;
    for (int i = 0; i < g.ip.np; ++i) {
      const int p = g.ip.pos[i];
      const uint64_t lo = k & ((1ull << p) - 1);
      k = ((k - lo) << 1) | lo;
    }
    k |= g.ip.ones;
    C v[2][L];
#pragma unroll
    for (int j = 0; j < L; ++j) {
      const VT r = __ldcs(reinterpret_cast<const VT*>(re + k + g.off[j]));
      const VT i = __ldcs(reinterpret_cast<const VT*>(im + k + g.off[j]));
      v[0][j] = mk<S>(r.x, i.x);
      v[1][j] = mk<S>(r.y, i.y);
    }
    C w[2][L];
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
      for (int j = 0; j < L; ++j) {
        if (DIAG) {
          const double2 d = g.m[j];
          w[h][j] = (d.x == 1.0 && d.y == 0.0) ? v[h][j] : cmul_rn(mk<S>((S)d.x, (S)d.y), v[h][j]);
        } else {
          C acc = mk<S>(0, 0);
#pragma unroll
          for (int i = 0; i < L; ++i)
            cfma(acc, mk<S>((S)g.m[j * L + i].x, (S)g.m[j * L + i].y), v[h][i]);
          w[h][j] = acc;
        }
      }
#pragma unroll
    for (int j = 0; j < L; ++j) {
      if (DIAG && g.m[j].x == 1.0 && g.m[j].y == 0.0) continue;
      VT r, i;
      r.x = w[0][j].x;
      r.y = w[1][j].x;
      i.x = w[0][j].y;
      i.y = w[1][j].y;
      __stcs(reinterpret_cast<VT*>(re + k + g.off[j]), r);
      __stcs(reinterpret_cast<VT*>(im + k + g.off[j]), i);
    }
  }
}

template <class S, int L, bool DIAG>
void run_soa(const LaunchCtx& ctx, uint64_t n_groups, const SoaGate& g) {
  if (g.ip.np > 0 && g.ip.pos[0] > 0 && n_groups >= 2) {  // bit 0 free: paired vector accesses
    S* re = reinterpret_cast<S*>(ctx.amps);
    S* im = re + (1ull << ctx.n_local);
    uint64_t nb = (n_groups / 2 + kThreads - 1) / kThreads;
    if (nb > 148ull * 32) nb = 148ull * 32;
    k_soa2<S, L, DIAG><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(re, im, n_groups / 2, g);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
    return;
  }
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
  const bool diag = d.cls == GClass::DIAG;
  const int m = d.m, Lg = 1 << m;
  uint64_t tmask = 0;
  for (int s = 0; s < m; ++s) tmask |= 1ull << d.targets[s];
  // Sector rule (as in the AOS kernels): the 8-byte planes put 4
  // consecutive amplitudes in one 32-B sector, so diagonal groups touching bits
  // 0/1 rewrite every entry instead of leaving holes (read-modify-writes).
  // (Moving controls on bits 0/1 into the group, as the AOS path does, measured
  // slower here: the 4 strided 8-byte accesses per plane cost more than the holes.)
  const uint64_t wctl = 0;
  int gbits[3], ng = 0;
  for (int s = 0; s < m; ++s) gbits[ng++] = d.targets[s];  // local index MSB first
  for (int q = 0; q < 2; ++q)
    if ((wctl >> q) & 1) gbits[ng++] = q;
  const uint64_t ctl = d.cmask & ~wctl;
  const int L = 1 << ng;
  // Expanded matrix over the group: gate where the widened controls are 1.
  auto entry = [&](int row, int col) -> double2 {
    const int ncw = ng - m;
    const int rc = row & ((1 << ncw) - 1), cc = col & ((1 << ncw) - 1);
    const int rt = row >> ncw, ct = col >> ncw;
    if (rc != cc) return make_double2(0.0, 0.0);
    if (rc != (1 << ncw) - 1) return make_double2(rt == ct ? 1.0 : 0.0, 0.0);
    return make_double2(d.M[rt * Lg + ct].re, d.M[rt * Lg + ct].im);
  };
  uint64_t zmask = ctl, ones = ctl;
  const bool low = ((tmask | d.cmask) & 3ull) != 0;
  if (diag && !low) {
    // One-entry diagonals (Z, S, T, Phase, CZ, CPhase, MC-Z) touch only the
    // amplitudes whose factor is not 1: fold the targets into the fixed bits.
    int active = -1, na = 0;
    for (int j = 0; j < Lg; ++j)
      if (!(d.M[j * Lg + j].re == 1.0 && d.M[j * Lg + j].im == 0.0)) {
        ++na;
        active = j;
      }
    if (na == 1) {
      for (int s = 0; s < m; ++s)
        if ((active >> (m - 1 - s)) & 1) ones |= 1ull << d.targets[s];
      zmask |= tmask;
      for (int q = 0; q < 64; ++q)
        if ((zmask >> q) & 1) g.ip.pos[g.ip.np++] = q;
      g.ip.ones = ones;
      g.off[0] = 0;
      g.m[0] = make_double2(d.M[active * Lg + active].re, d.M[active * Lg + active].im);
      run_soa<S, 1, true>(ctx, 1ull << (ctx.n_local - g.ip.np), g);
      return;
    }
  }
  for (int s = 0; s < ng; ++s) zmask |= 1ull << gbits[s];
  for (int q = 0; q < 64; ++q)
    if ((zmask >> q) & 1) g.ip.pos[g.ip.np++] = q;
  g.ip.ones = ones;
  for (int j = 0; j < L; ++j) {
    uint64_t o = 0;
    for (int s = 0; s < ng; ++s)
      if ((j >> (ng - 1 - s)) & 1) o |= 1ull << gbits[s];
    g.off[j] = o;
  }
  g.store_all = low ? 1 : 0;
  if (diag) {
    for (int j = 0; j < L; ++j) g.m[j] = entry(j, j);
  } else {
    for (int r = 0; r < L; ++r)
      for (int c = 0; c < L; ++c) g.m[r * L + c] = entry(r, c);
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
