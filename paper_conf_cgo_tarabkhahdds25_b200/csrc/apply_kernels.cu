// apply_kernels.cu -- sm_100a gate-application kernels.
//
// One pass over the changed part of the state per gate: the 2^n x 2^n matrix
// I_L (x) M (x) I_R (Eq. 1) / Eq. 5 is never formed (vector
// fusion); each thread expands a free index into amplitude indices by
// bit insertion (Fig. 3b, Fig. 14: id1 = rR + 2 rL Rs,
// id2 = id1 + Rs; Fig. 8's Ls/Gs/Rs loops P:299-306 for two targets) and
// applies the gate's class-specialised update in place.
//
// B200 design: HBM-bound streaming, so
//   * one-amplitude (16 B) or two-adjacent-amplitude (32 B, LDG/STG.256) vector
//     accesses with evict-first policy; two adjacent groups per thread when
//     qubit 0 is free (k_group_x2);
//   * several independent groups per thread (>= 64 B in flight per lane);
//   * whole 32-B sectors whenever qubit 0 is a control / fixed diagonal bit /
//     SWAP target (a 16-B write costs a sector read-modify-write);
//   * targets below 5 optionally via warp shuffles (k_lowq);
//   * diagonal gates touch only amplitudes whose factor is not 1;
//   * the diagonal multiply is RN, no FMA, so diagonal results are value-exact
//     against the oracle (R8).
// Every kernel is templated on the scalar S: double (complex128, default) or
// float (complex64, NEXT-4).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <type_traits>

#include "cx.cuh"
#include "lfqs_internal.h"

namespace lfqs {
namespace {

constexpr int kThreads = 256;

// Free index -> amplitude index (insert zero bits at ascending positions, OR ones).
template <int NPMAX>
__device__ __forceinline__ uint64_t expand(const InsertPlan& ip, uint64_t g) {
#pragma unroll
  for (int i = 0; i < NPMAX; ++i) {
    if (i < ip.np) {
      const int p = ip.pos[i];
      const uint64_t lo = g & ((1ull << p) - 1);
      g = ((g - lo) << 1) | lo;
    }
  }
  return g | ip.ones;
}

// ---------------------------------------------------------------------------
// Group operators: v[0..L) = amplitudes at k + off[j] (j = local index).
// ---------------------------------------------------------------------------
template <class S>
struct OpSwap2 {  // X / CNOT / Toffoli / SWAP: moves only (bit-exact)
  __device__ __forceinline__ void operator()(cx<S> (&v)[2], uint64_t) const {
    const cx<S> t = v[0];
    v[0] = v[1];
    v[1] = t;
  }
};
template <class S>
struct OpSwapMid {  // SWAP(0, t) on the group (00, 01, 10, 11): exchange 01 <-> 10
  __device__ __forceinline__ void operator()(cx<S> (&v)[4], uint64_t) const {
    const cx<S> t = v[1];
    v[1] = v[2];
    v[2] = t;
  }
};
template <class S>
struct OpY {  // Y = [[0,-i],[i,0]]: v0' = -i v1, v1' = i v0 (moves + sign, exact)
  __device__ __forceinline__ void operator()(cx<S> (&v)[2], uint64_t) const {
    const cx<S> a0 = v[0], a1 = v[1];
    v[0] = mk<S>(a1.y, -a1.x);
    v[1] = mk<S>(-a0.y, a0.x);
  }
};
template <class S>
struct OpH {  // hadgate, Fig. 12c / Fig. 14: sq2r*(s1+s2), sq2r*(s1-s2)
  S s;
  __device__ __forceinline__ void operator()(cx<S> (&v)[2], uint64_t) const {
    const cx<S> a0 = v[0], a1 = v[1];
    v[0] = mk<S>(s * (a0.x + a1.x), s * (a0.y + a1.y));
    v[1] = mk<S>(s * (a0.x - a1.x), s * (a0.y - a1.y));
  }
};
template <class S, int L>
struct OpDense {  // single_qbit (Fig. 12b) generalised: v' = M v
  cx<S> M[L * L];
  __device__ __forceinline__ void operator()(cx<S> (&v)[L], uint64_t) const {
    cx<S> w[L];
#pragma unroll
    for (int j = 0; j < L; ++j) {
      cx<S> acc = mk<S>(0, 0);
#pragma unroll
      for (int i = 0; i < L; ++i) cfma(acc, M[j * L + i], v[i]);
      w[j] = acc;
    }
#pragma unroll
    for (int j = 0; j < L; ++j) v[j] = w[j];
  }
};
// Diagonal, one touched entry per group (Z, S, T, Phase, CZ, CPhase, MC-Z).
template <class S>
struct OpNeg {
  __device__ __forceinline__ void operator()(cx<S> (&v)[1], uint64_t) const {
    v[0] = mk<S>(-v[0].x, -v[0].y);
  }
};
template <class S>
struct OpMulI {  // * (0, 1): (-im, re)
  __device__ __forceinline__ void operator()(cx<S> (&v)[1], uint64_t) const {
    v[0] = mk<S>(-v[0].y, v[0].x);
  }
};
template <class S>
struct OpMulNI {  // * (0, -1): (im, -re)
  __device__ __forceinline__ void operator()(cx<S> (&v)[1], uint64_t) const {
    v[0] = mk<S>(v[0].y, -v[0].x);
  }
};
template <class S>
struct OpMul {  // * d
  cx<S> d;
  __device__ __forceinline__ void operator()(cx<S> (&v)[1], uint64_t) const {
    v[0] = cmul_rn(d, v[0]);
  }
};
// Diagonal over a whole group: v[j] *= d[j] (Rz, general diagonals; no selects).
template <class S, int L>
struct OpDiagGroup {
  cx<S> d[L];
  uint32_t touch;  // bit j set: d[j] != 1
  __device__ __forceinline__ void operator()(cx<S> (&v)[L], uint64_t) const {
#pragma unroll
    for (int j = 0; j < L; ++j)
      if (touch >> j & 1) v[j] = cmul_rn(d[j], v[j]);
  }
};
// A one-amplitude op applied to element `which` of an adjacent pair (bit 0 fixed by
// a control or diagonal pattern): the pair moves as one 32-byte sector so no
// sub-sector (16 B) writes reach L2/DRAM.
template <class S, class Op1>
struct OpAtPair {
  Op1 op;
  int which;
  __device__ __forceinline__ void operator()(cx<S> (&v)[2], uint64_t k) const {
    cx<S> t[1];
    if (which) {
      t[0] = v[1];
      op(t, k);
      v[1] = t[0];
    } else {
      t[0] = v[0];
      op(t, k);
      v[0] = t[0];
    }
  }
};
// A pair op with a control on qubit 0: group (k, k+1, k+2^t, k+2^t+1), the op acts
// on (v1, v3); all four move as two 32-byte sectors.
template <class S, class Op2>
struct OpCtrl0 {
  Op2 op;
  __device__ __forceinline__ void operator()(cx<S> (&v)[4], uint64_t k) const {
    cx<S> p[2] = {v[1], v[3]};
    op(p, k | 1);
    v[1] = p[0];
    v[3] = p[1];
  }
};

template <int L>
struct Offs {
  uint64_t o[L];
};

// ---------------------------------------------------------------------------
// Generic group kernel: each thread handles U groups; each group reads and
// writes L amplitudes at k + off[j].  P256: off[2i+1] == off[2i] + 1, so the
// pair moves as one access.
// ---------------------------------------------------------------------------
//
// pmask / ppat (line-shaped reads): fixed bits at positions 1-2 that run_group took out of
// the insertion plan; every group is loaded (whole 128-B lines, coalesced) but only groups
// with (k & pmask) == ppat are updated and stored (probe: tools/probe_sparse.cu).
template <class S, int L, int U, bool P256, int NPMAX, class Op>
__global__ void __launch_bounds__(kThreads) k_group(cx<S>* __restrict__ a, uint64_t n_groups,
                                                    const InsertPlan ip, const Offs<L> off,
                                                    const Op op, uint64_t pmask, uint64_t ppat) {
  const uint64_t g0 = (uint64_t)blockIdx.x * (kThreads * U) + threadIdx.x;
  cx<S> v[U][L];
  uint64_t kk[U];
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const uint64_t g = g0 + (uint64_t)u * kThreads;
    kk[u] = expand<NPMAX>(ip, g < n_groups ? g : 0);
    if (g < n_groups) {
      if constexpr (P256) {
#pragma unroll
        for (int j = 0; j < L; j += 2) ld2(a + kk[u] + off.o[j], v[u][j], v[u][j + 1]);
      } else {
#pragma unroll
        for (int j = 0; j < L; ++j) v[u][j] = ld1(a + kk[u] + off.o[j]);
      }
    }
  }
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const uint64_t g = g0 + (uint64_t)u * kThreads;
    if (g < n_groups && (kk[u] & pmask) == ppat) {
      op(v[u], kk[u]);
      if constexpr (P256) {
#pragma unroll
        for (int j = 0; j < L; j += 2) st2(a + kk[u] + off.o[j], v[u][j], v[u][j + 1]);
      } else {
#pragma unroll
        for (int j = 0; j < L; ++j) st1(a + kk[u] + off.o[j], v[u][j]);
      }
    }
  }
}

// Two adjacent groups per item when qubit 0 is free (not a target or control):
// groups at k and k+1 share every sector, so each access is one two-amplitude
// LDG/STG and the instruction count per byte halves.
template <class S, int L, int U, int NPMAX, class Op>
__global__ void __launch_bounds__(kThreads) k_group_x2(cx<S>* __restrict__ a, uint64_t n_items,
                                                       const InsertPlan ip, const Offs<L> off,
                                                       const Op op, uint64_t pmask, uint64_t ppat) {
  const uint64_t i0 = (uint64_t)blockIdx.x * (kThreads * U) + threadIdx.x;
  cx<S> v[U][L], w[U][L];
  uint64_t kk[U];
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const uint64_t i = i0 + (uint64_t)u * kThreads;
    kk[u] = expand<NPMAX>(ip, (i < n_items ? i : 0) << 1);
    if (i < n_items) {
#pragma unroll
      for (int j = 0; j < L; ++j) ld2(a + kk[u] + off.o[j], v[u][j], w[u][j]);
    }
  }
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const uint64_t i = i0 + (uint64_t)u * kThreads;
    if (i < n_items && (kk[u] & pmask) == ppat) {
      op(v[u], kk[u]);
      op(w[u], kk[u] | 1);
#pragma unroll
      for (int j = 0; j < L; ++j) st2(a + kk[u] + off.o[j], v[u][j], w[u][j]);
    }
  }
}

// ---------------------------------------------------------------------------
// Low-target (t < 5) warp-shuffle kernel for 2x2-type gates.  A warp owns a
// chunk of 32*V contiguous amplitudes; lane l holds amplitude l + 32 j of the
// chunk; its partner for target t is lane l ^ (1 << t).
// Controls >= 5 + log2 V are inserted into the chunk index (whole chunks are
// skipped); controls below that are a per-lane store predicate.
// ---------------------------------------------------------------------------
template <class S>
struct LaneSwap {  // X
  __device__ __forceinline__ cx<S> operator()(cx<S>, cx<S> p, int) const { return p; }
};
template <class S>
struct LaneY {  // Y: bit 0 -> -i p ; bit 1 -> i p
  __device__ __forceinline__ cx<S> operator()(cx<S>, cx<S> p, int bit) const {
    return bit ? mk<S>(-p.y, p.x) : mk<S>(p.y, -p.x);
  }
};
template <class S>
struct LaneH {
  S s;
  __device__ __forceinline__ cx<S> operator()(cx<S> a, cx<S> p, int bit) const {
    return bit ? mk<S>(s * (p.x - a.x), s * (p.y - a.y)) : mk<S>(s * (a.x + p.x), s * (a.y + p.y));
  }
};
template <class S>
struct LaneDense {  // out = self[bit] * a + other[bit] * p
  cx<S> self_c[2], other_c[2];
  __device__ __forceinline__ cx<S> operator()(cx<S> a, cx<S> p, int bit) const {
    cx<S> acc = mk<S>(0, 0);
    cfma(acc, bit ? self_c[1] : self_c[0], a);
    cfma(acc, bit ? other_c[1] : other_c[0], p);
    return acc;
  }
};

template <class S, int V, class LaneOp>
__global__ void __launch_bounds__(kThreads) k_lowq(cx<S>* __restrict__ a, uint64_t n_chunks,
                                                   const InsertPlan ip_hi, uint64_t low_cmask,
                                                   int t, const LaneOp op) {
  constexpr int kLogV = V == 1 ? 0 : V == 2 ? 1 : V == 4 ? 2 : 3;
  const int lane = threadIdx.x & 31;
  const uint64_t chunk = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
  if (chunk >= n_chunks) return;  // warp-uniform
  const uint64_t base = expand<kMaxInsert>(ip_hi, chunk << (5 + kLogV));
  cx<S> v[V];
#pragma unroll
  for (int j = 0; j < V; ++j) v[j] = ld1(a + base + j * 32 + lane);
  const int bit = (lane >> t) & 1;
#pragma unroll
  for (int j = 0; j < V; ++j) {
    cx<S> p;
    p.x = __shfl_xor_sync(0xffffffffu, v[j].x, 1 << t);
    p.y = __shfl_xor_sync(0xffffffffu, v[j].y, 1 << t);
    const uint64_t k = base + j * 32 + lane;
    if ((k & low_cmask) == low_cmask) st1(a + k, op(v[j], p, bit));
  }
}

// ---------------------------------------------------------------------------
// Dense 4x4 / 8x8 gate whose targets all lie in [1, 5] with qubit 0 free (used by
// default for 4x4 on qubits {1, 2} only; LFQS_OPT_LANE_GROUP = 2 forces it).  The
// generic group kernels give each thread one group; with targets this low a
// group (x2: with its bit-0 neighbours) is a single contiguous 128-256 B run, so
// every warp access touches 32 different lines, one sector each (UNITARY2 on
// qubits (1, 2): 6.3 ms vs 4.9 ms at n = 30).  Here a warp owns 64*V contiguous
// amplitudes and lane l loads pairs p = l + 32 v (amplitudes 2p, 2p+1) -- fully
// coalesced 32-B accesses; the lanes that differ from l only in the target bits
// (lane bit t-1 holds amplitude bit t) hold the other group members, fetched by
// shuffles; each lane computes its own two outputs with the OpDense formula
// (same terms, same order), so results equal the group kernel's bit for bit.
// ---------------------------------------------------------------------------
template <class S, int L>
struct LaneGroupArgs {
  cx<S> M[L * L];
  uint32_t src[L];   // lane bits of local index i (OR-ed onto the lane's non-target bits)
  uint32_t lmask;    // lane bits of the targets
  uint32_t lbit[3];  // lane bit of target s (targets[0] = MSB of the local index)
  uint64_t low_cmask;
};

template <class S, int L, int V>
__global__ void __launch_bounds__(kThreads) k_lanegroup(cx<S>* __restrict__ a, uint64_t n_chunks,
                                                        const InsertPlan ip_hi,
                                                        const LaneGroupArgs<S, L> g) {
  constexpr int m = L == 4 ? 2 : 3;
  constexpr int kLogV = V == 1 ? 0 : V == 2 ? 1 : V == 4 ? 2 : 3;
  const int lane = threadIdx.x & 31;
  const uint64_t chunk = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
  if (chunk >= n_chunks) return;  // warp-uniform
  const uint64_t base = expand<kMaxInsert>(ip_hi, chunk << (6 + kLogV));
  cx<S> v0[V], v1[V];
#pragma unroll
  for (int j = 0; j < V; ++j) ld2(a + base + 2 * (j * 32 + lane), v0[j], v1[j]);
  int jl = 0;
#pragma unroll
  for (int s = 0; s < m; ++s) jl |= ((lane >> g.lbit[s]) & 1) << (m - 1 - s);
  const int rest = lane & ~(int)g.lmask;
#pragma unroll
  for (int j = 0; j < V; ++j) {
    cx<S> acc0 = mk<S>(0, 0), acc1 = mk<S>(0, 0);
#pragma unroll
    for (int i = 0; i < L; ++i) {
      const int src = rest | (int)g.src[i];
      cx<S> p0, p1;
      p0.x = __shfl_sync(0xffffffffu, v0[j].x, src);
      p0.y = __shfl_sync(0xffffffffu, v0[j].y, src);
      p1.x = __shfl_sync(0xffffffffu, v1[j].x, src);
      p1.y = __shfl_sync(0xffffffffu, v1[j].y, src);
      const cx<S> mji = g.M[jl * L + i];
      cfma(acc0, mji, p0);
      cfma(acc1, mji, p1);
    }
    const uint64_t k = base + 2 * (j * 32 + lane);
    if ((k & g.low_cmask) == g.low_cmask) v0[j] = acc0;
    if (((k | 1) & g.low_cmask) == g.low_cmask) v1[j] = acc1;
    st2(a + k, v0[j], v1[j]);
  }
}

// ---------------------------------------------------------------------------
// Exchange swap with a bounded grid (persistent, grid-stride): pairs
// (a[k | 2^l], a[k + partner]) for the free indices k (bit l inserted as 0), two
// adjacent pairs per item when l > 0 (32-B accesses on both sides).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Grid-limited exchange swap (persistent, grid-stride).  period_ns > 0 paces it: the
// grid's j-th round of items starts no earlier than j * period_ns after the CTA started
// (a link-rate emulation, LFQS_OPT_EXCHANGE_RATE_GBS).
template <class S>
__global__ void __launch_bounds__(kThreads) k_xswap(cx<S>* __restrict__ a, uint64_t n_pairs,
                                                     int l, uint64_t partner, InsertPlan ip,
                                                     uint64_t period_ns) {
  // ip inserts 0 at l and the block's fixed bits (never at position 0 when l > 0)
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  const uint64_t bit = 1ull << l;
  const uint64_t n_items = l > 0 ? n_pairs / 2 : n_pairs;
  const uint64_t t0 = period_ns ? globaltimer_ns() : 0;
  uint64_t round = 0;
  for (uint64_t b0 = (uint64_t)blockIdx.x * kThreads; b0 < n_items; b0 += stride, ++round) {
    if (period_ns) {
      if (threadIdx.x == 0)
        while (globaltimer_ns() < t0 + round * period_ns) {
        }
      __syncthreads();
    }
    const uint64_t i = b0 + threadIdx.x;
    if (i >= n_items) continue;
    if (l > 0) {
      const uint64_t k = expand<6>(ip, i << 1);
      cx<S> x0, x1, y0, y1;
      ld2(a + (k | bit), x0, x1);
      ld2(a + k + partner, y0, y1);
      st2(a + (k | bit), y0, y1);
      st2(a + k + partner, x0, x1);
    } else {
      const uint64_t k = expand<6>(ip, i);
      const cx<S> x = ld1(a + (k | 1)), y = ld1(a + k + partner);
      st1(a + (k | 1), y);
      st1(a + k + partner, x);
    }
  }
}

// ---------------------------------------------------------------------------
// Host launch helpers
// ---------------------------------------------------------------------------
InsertPlan make_plan(uint64_t zero_bits, uint64_t one_bits) {
  InsertPlan ip;
  std::memset(&ip, 0, sizeof ip);
  const uint64_t all = zero_bits | one_bits;
  for (int p = 0; p < 64; ++p)
    if (all >> p & 1) {
      require(ip.np < kMaxInsert, "too many fixed qubits");
      ip.pos[ip.np++] = p;
    }
  ip.ones = one_bits;
  return ip;
}

template <class S>
inline cx<S> CV(cplx z) {
  return mk<S>((S)z.re, (S)z.im);
}

inline uint64_t blocks_for(uint64_t items, uint64_t per_block) {
  return (items + per_block - 1) / per_block;
}

template <class S, int L, int U, bool P256, class Op>
void run_group(const LaunchCtx& ctx, uint64_t n_groups, const InsertPlan& ip_in,
               const Offs<L>& off, const Op& op) {
  if (n_groups == 0) return;
  auto* a = reinterpret_cast<cx<S>*>(ctx.amps);
  // Line-shaped reads (LFQS_OPT_LINE_READS): a fixed bit (control or one-entry diagonal
  // pattern) at position 1 or 2 leaves 1 of every 2 or 4 sectors of each 128-B line
  // touched, yet DRAM reads whole lines whatever is requested (tools/probe_sparse.cu:
  // reading 1 sector in 4 takes as long as reading all).  Such bits are taken out of the
  // insertion plan and become a store predicate: the warps stream whole lines, coalesced,
  // and write back only the touched groups.  Same per-amplitude arithmetic.
  InsertPlan ip = ip_in;
  uint64_t pmask = 0, ppat = 0;
  if (ctx.opt->line_reads) {
    uint64_t tb = 0, all = 0;
    for (int j = 0; j < L; ++j) tb |= off.o[j];
    for (int i = 0; i < ip_in.np; ++i) all |= 1ull << ip_in.pos[i];
    const uint64_t F = all & 6ull & ~tb;
    if (F) {
      ip = make_plan(all & ~F, ip_in.ones & ~F);
      pmask = F;
      ppat = ip_in.ones & F;
      n_groups <<= __builtin_popcountll(F);
    }
  }
  bool even = true;
  for (int j = 0; j < L; ++j) even &= (off.o[j] & 1) == 0;
  if constexpr (!P256 && L <= 4) {
    if (ctx.opt->wide256 && even && n_groups >= 2 && (ip.np == 0 || ip.pos[0] >= 1)) {
      const uint64_t n_items = n_groups / 2;
      auto go = [&](auto ux) {
        constexpr int UX = decltype(ux)::value;
        const uint64_t nb = blocks_for(n_items, (uint64_t)kThreads * UX);
        require(nb < (1ull << 31), "grid too large");
        if (ip.np <= 4)
          k_group_x2<S, L, UX, 4, Op>
              <<<(unsigned)nb, kThreads, 0, ctx.stream>>>(a, n_items, ip, off, op, pmask, ppat);
        else
          k_group_x2<S, L, UX, kMaxInsert, Op>
              <<<(unsigned)nb, kThreads, 0, ctx.stream>>>(a, n_items, ip, off, op, pmask, ppat);
      };
      // Groups per thread (tuning knob LFQS_OPT_ITEMS_PER_THREAD for pair gates).
      const int ipt = ctx.opt->items_per_thread;
      if (L == 2 && ipt == 1)
        go(std::integral_constant<int, 1>{});
      else if (L == 2 && ipt == 4)
        go(std::integral_constant<int, 4>{});
      else
        go(std::integral_constant<int, L == 1 ? 4 : (L == 2 ? 2 : 1)>{});
      LFQS_CUDA_CHECK(cudaGetLastError());
      ++*ctx.launch_counter;
      return;
    }
  }
  const uint64_t nb = blocks_for(n_groups, (uint64_t)kThreads * U);
  require(nb < (1ull << 31), "grid too large");
  if (ip.np <= 4)
    k_group<S, L, U, P256, 4, Op>
        <<<(unsigned)nb, kThreads, 0, ctx.stream>>>(a, n_groups, ip, off, op, pmask, ppat);
  else
    k_group<S, L, U, P256, kMaxInsert, Op>
        <<<(unsigned)nb, kThreads, 0, ctx.stream>>>(a, n_groups, ip, off, op, pmask, ppat);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

template <class S, class LaneOp>
void run_lowq(const LaunchCtx& ctx, int t, uint64_t cmask, const LaneOp& op) {
  constexpr int V = 4, kLogV = 2;
  constexpr int CB = 5 + kLogV;
  const uint64_t hi_c = cmask & ~((1ull << CB) - 1), lo_c = cmask & ((1ull << CB) - 1);
  const InsertPlan ip = make_plan(0, hi_c);
  const int n_hi = __builtin_popcountll(hi_c);
  const uint64_t n_chunks = 1ull << (ctx.n_local - CB - n_hi);
  const uint64_t nb = blocks_for(n_chunks, kThreads / 32);
  require(nb < (1ull << 31), "grid too large");
  k_lowq<S, V, LaneOp><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(
      reinterpret_cast<cx<S>*>(ctx.amps), n_chunks, ip, lo_c, t, op);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

// 2-amplitude (pair) gate on target t with controls: X, Y, dense 2x2.
template <class S, class Op, class LaneOp>
void launch_pair(const LaunchCtx& ctx, const Decoded& g, const Op& op, const LaneOp& lane_op) {
  const int t = g.targets[0];
  const int nc = __builtin_popcountll(g.cmask);
  if (g.cmask & 1) {
    // Control on qubit 0: widen to (k, k+1, k+2^t, k+2^t+1) so the untouched
    // neighbours are rewritten and no 16-byte (sub-sector) writes occur.
    const InsertPlan ip = make_plan((1ull << t) | 1ull, g.cmask & ~1ull);
    Offs<4> off{{0ull, 1ull, 1ull << t, (1ull << t) | 1ull}};
    run_group<S, 4, 2, true>(ctx, 1ull << (ctx.n_local - 1 - nc), ip, off, OpCtrl0<S, Op>{op});
    return;
  }
  constexpr int kCB = 7;
  if (ctx.opt->lowq_shuffle && t < 5 && ctx.n_local >= kCB + __builtin_popcountll(g.cmask >> kCB)) {
    run_lowq<S>(ctx, t, g.cmask, lane_op);
    return;
  }
  const uint64_t n_groups = 1ull << (ctx.n_local - 1 - nc);
  const InsertPlan ip = make_plan(1ull << t, g.cmask);
  Offs<2> off{{0ull, 1ull << t}};
  if (t == 0)
    run_group<S, 2, 4, true>(ctx, n_groups, ip, off, op);
  else
    run_group<S, 2, 4, false>(ctx, n_groups, ip, off, op);
}

// Local-index offsets: off[j] = sum_s bit(m-1-s of j) << t_s (reading R2).
template <int L>
Offs<L> group_offsets(const int* t, int m) {
  Offs<L> off;
  for (int j = 0; j < L; ++j) {
    uint64_t o = 0;
    for (int s = 0; s < m; ++s) o |= (uint64_t)((j >> (m - 1 - s)) & 1) << t[s];
    off.o[j] = o;
  }
  return off;
}

// Reorder a 2^m matrix so that its targets are listed in a new order `perm`
// (new target s = old target perm[s]); exact (entries only move).
void permute_targets(const Decoded& g, const int* perm, int* t_new, cplx* M_new) {
  const int m = g.m, d = 1 << m;
  for (int s = 0; s < m; ++s) t_new[s] = g.targets[perm[s]];
  auto old_index = [&](int jn) {
    int jo = 0;
    for (int s = 0; s < m; ++s) {
      const int b = (jn >> (m - 1 - s)) & 1;  // bit of new target s
      jo |= b << (m - 1 - perm[s]);
    }
    return jo;
  };
  for (int r = 0; r < d; ++r)
    for (int c = 0; c < d; ++c) M_new[r * d + c] = g.M[old_index(r) * d + old_index(c)];
}

template <class S, int L>
void launch_dense_m(const LaunchCtx& ctx, const Decoded& g) {
  constexpr int m = L == 4 ? 2 : 3;
  // Put qubit 0 (if a target) last, so amplitude pairs (k, k+1) are adjacent
  // and move as one access.
  int perm[3] = {0, 1, 2};
  for (int s = 0; s < m; ++s)
    if (g.targets[s] == 0) std::swap(perm[s], perm[m - 1]);
  int t[3];
  OpDense<S, L> op;
  cplx Mp[64];
  permute_targets(g, perm, t, Mp);
  for (int i = 0; i < L * L; ++i) op.M[i] = CV<S>(Mp[i]);
  uint64_t tmask = 0;
  for (int s = 0; s < m; ++s) tmask |= 1ull << t[s];
  const int nc = __builtin_popcountll(g.cmask);
  const uint64_t n_groups = 1ull << (ctx.n_local - m - nc);
  const InsertPlan ip = make_plan(tmask, g.cmask);
  const Offs<L> off = group_offsets<L>(t, m);
  // Targets {1, 2} (qubit 0 free): the group kernel's item is one contiguous 128-B
  // run per thread (32 lines per warp access): coalesced lane-group kernel instead
  // (k_lanegroup; measured at n = 30: 6.5 -> 4.9 ms).  For other low targets, and
  // for 8x8 gates, its shuffle volume (8 shuffles per partner and pair) makes it
  // slower than the group kernel (profiles/r01_lane_group.md), so they stay there.
  constexpr int kLGV = 4, kLGB = 6 + 2;  // 4 pairs per lane: 256-amplitude chunks
  const uint64_t hi_c = g.cmask & ~((1ull << kLGB) - 1);
  if (ctx.opt->lane_group && (L == 4 ? tmask == 6ull : ctx.opt->lane_group > 1) &&
      !(tmask & 1) && (tmask >> 6) == 0 &&
      ctx.n_local >= kLGB + __builtin_popcountll(hi_c)) {
    LaneGroupArgs<S, L> la;
    for (int i = 0; i < L * L; ++i) la.M[i] = op.M[i];
    la.lmask = (uint32_t)(tmask >> 1);
    for (int s = 0; s < 3; ++s) la.lbit[s] = s < m ? (uint32_t)(t[s] - 1) : 0;
    for (int i = 0; i < L; ++i) {
      uint32_t o = 0;
      for (int s = 0; s < m; ++s) o |= (uint32_t)((i >> (m - 1 - s)) & 1) << (t[s] - 1);
      la.src[i] = o;
    }
    la.low_cmask = g.cmask & ((1ull << kLGB) - 1);
    const uint64_t n_chunks = 1ull << (ctx.n_local - kLGB - __builtin_popcountll(hi_c));
    const uint64_t nb = blocks_for(n_chunks, kThreads / 32);
    require(nb < (1ull << 31), "grid too large");
    k_lanegroup<S, L, kLGV><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(
        reinterpret_cast<cx<S>*>(ctx.amps), n_chunks, make_plan(0, hi_c), la);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
    return;
  }
  if (t[m - 1] == 0)
    run_group<S, L, (L == 4 ? 2 : 1), true>(ctx, n_groups, ip, off, op);
  else
    run_group<S, L, (L == 4 ? 2 : 1), false>(ctx, n_groups, ip, off, op);
}

template <class S, class Op1>
void run_diag_one(const LaunchCtx& ctx, uint64_t n_groups, uint64_t zeros, uint64_t ones,
                  const Op1& op) {
  if ((zeros | ones) & 1) {
    // Qubit 0 is fixed: widen the group to the adjacent pair so every write is a
    // whole sector (a 16-byte write costs a sector read-modify-write).
    const InsertPlan ip = make_plan((zeros & ~1ull) | 1ull, ones & ~1ull);
    run_group<S, 2, 4, true>(ctx, n_groups, ip, Offs<2>{{0, 1}},
                             OpAtPair<S, Op1>{op, (int)(ones & 1)});
  } else {
    run_group<S, 1, 4, false>(ctx, n_groups, make_plan(zeros, ones), Offs<1>{{0}}, op);
  }
}

template <class S, int L>
void run_diag_group(const LaunchCtx& ctx, const Decoded& g) {
  constexpr int m = L == 2 ? 1 : (L == 4 ? 2 : 3);
  int perm[3] = {0, 1, 2};
  for (int s = 0; s < m; ++s)
    if (g.targets[s] == 0) std::swap(perm[s], perm[m - 1]);
  int t[3];
  cplx Mp[64];
  permute_targets(g, perm, t, Mp);
  OpDiagGroup<S, L> op;
  op.touch = 0;
  for (int j = 0; j < L; ++j) {
    op.d[j] = CV<S>(Mp[j * L + j]);
    if (!(Mp[j * L + j].re == 1.0 && Mp[j * L + j].im == 0.0)) op.touch |= 1u << j;
  }
  uint64_t tmask = 0;
  for (int s = 0; s < m; ++s) tmask |= 1ull << t[s];
  const int nc = __builtin_popcountll(g.cmask);
  const uint64_t n_groups = 1ull << (ctx.n_local - m - nc);
  const InsertPlan ip = make_plan(tmask, g.cmask);
  const Offs<L> off = group_offsets<L>(t, m);
  if (t[m - 1] == 0)
    run_group<S, L, (L == 8 ? 1 : 2), true>(ctx, n_groups, ip, off, op);
  else
    run_group<S, L, (L == 8 ? 1 : 2), false>(ctx, n_groups, ip, off, op);
}

template <class S>
void launch_diag(const LaunchCtx& ctx, const Decoded& g) {
  const int m = g.m, d = 1 << m;
  // Entries != 1 (the only amplitudes that change).
  int n_active = 0, active = -1;
  for (int j = 0; j < d; ++j) {
    const cplx z = g.M[j * d + j];
    if (!(z.re == 1.0 && z.im == 0.0)) {
      ++n_active;
      active = j;
    }
  }
  if (n_active == 0) return;
  const int nc = __builtin_popcountll(g.cmask);
  uint64_t tmask = 0;
  for (int s = 0; s < m; ++s) tmask |= 1ull << g.targets[s];
  if (n_active == 1) {
    // Touch only amplitudes with target bits = active pattern and controls = 1.
    uint64_t pattern = 0;
    for (int s = 0; s < m; ++s) pattern |= (uint64_t)((active >> (m - 1 - s)) & 1) << g.targets[s];
    const uint64_t zeros = tmask & ~pattern, ones = g.cmask | pattern;
    const uint64_t n_groups = 1ull << (ctx.n_local - m - nc);
    const cplx z = g.M[active * d + active];
    if (z.re == -1.0 && z.im == 0.0)
      run_diag_one<S>(ctx, n_groups, zeros, ones, OpNeg<S>{});
    else if (z.re == 0.0 && z.im == 1.0)
      run_diag_one<S>(ctx, n_groups, zeros, ones, OpMulI<S>{});
    else if (z.re == 0.0 && z.im == -1.0)
      run_diag_one<S>(ctx, n_groups, zeros, ones, OpMulNI<S>{});
    else
      run_diag_one<S>(ctx, n_groups, zeros, ones, OpMul<S>{CV<S>(z)});
    return;
  }
  if (m == 1)
    run_diag_group<S, 2>(ctx, g);
  else if (m == 2)
    run_diag_group<S, 4>(ctx, g);
  else
    run_diag_group<S, 8>(ctx, g);
}

template <class S>
void launch_gate_t(const LaunchCtx& ctx, const Decoded& g) {
  switch (g.cls) {
    case GClass::NOOP:
      return;
    case GClass::DIAG:
      launch_diag<S>(ctx, g);
      return;
    case GClass::PERM_X:
      launch_pair<S>(ctx, g, OpSwap2<S>{}, LaneSwap<S>{});
      return;
    case GClass::PERM_Y:
      launch_pair<S>(ctx, g, OpY<S>{}, LaneY<S>{});
      return;
    case GClass::PERM_SWAP: {
      const int t0 = g.targets[0], t1 = g.targets[1];
      const int nc = __builtin_popcountll(g.cmask);
      const InsertPlan ip = make_plan((1ull << t0) | (1ull << t1), g.cmask);
      if ((t0 == 0 || t1 == 0) && !(g.cmask & 1)) {
        // SWAP(0, t): move whole sectors (k, k+1), (k+2^t, k+2^t+1) and exchange
        // the middle two, instead of 16-byte writes into half-used sectors.
        const uint64_t t = 1ull << (t0 == 0 ? t1 : t0);
        Offs<4> off{{0ull, 1ull, t, t | 1ull}};
        run_group<S, 4, 2, true>(ctx, 1ull << (ctx.n_local - 2 - nc), ip, off, OpSwapMid<S>{});
        return;
      }
      Offs<2> off{{1ull << t0, 1ull << t1}};
      run_group<S, 2, 4, false>(ctx, 1ull << (ctx.n_local - 2 - nc), ip, off, OpSwap2<S>{});
      return;
    }
    case GClass::DENSE:
      if (g.m == 1) {
        if (g.is_h) {
          const S s = (S)g.M[0].re;
          launch_pair<S>(ctx, g, OpH<S>{s}, LaneH<S>{s});
        } else {
          OpDense<S, 2> op;
          for (int i = 0; i < 4; ++i) op.M[i] = CV<S>(g.M[i]);
          LaneDense<S> lop;
          lop.self_c[0] = CV<S>(g.M[0]);   // u00
          lop.self_c[1] = CV<S>(g.M[3]);   // u11
          lop.other_c[0] = CV<S>(g.M[1]);  // u01
          lop.other_c[1] = CV<S>(g.M[2]);  // u10
          launch_pair<S>(ctx, g, op, lop);
        }
      } else if (g.m == 2) {
        launch_dense_m<S, 4>(ctx, g);
      } else {
        launch_dense_m<S, 8>(ctx, g);
      }
      return;
  }
}

}  // namespace

// Virtual-partition exchange: swap the l=1 half of this shard with the l=0 half
// of the shard `partner_offset_amps` amplitudes further on (same pass structure
// as a SWAP gate), over the amplitudes whose bits fix_zero are 0 and fix_one
// are 1 (a block of an overlapped exchange; the P2P exchange also fixes one bit to split
// the pairs between the two ranks, p2p.cu).  The partner may be any address (a peer
// GPU's shard mapped by CUDA IPC): the offset wraps mod 2^64.
void launch_half_swap(const LaunchCtx& ctx, int l, uint64_t partner_offset_amps, int ctas,
                      uint64_t fix_zero, uint64_t fix_one) {
  const uint64_t fixed = fix_zero | fix_one;
  require(!(fixed >> l & 1) && !(fix_zero & fix_one) && __builtin_popcountll(fixed) <= 4 &&
              (fixed >> ctx.n_local) == 0 && (l == 0 || !(fixed & 1)),
          "internal: bad exchange block");
  const InsertPlan ip = make_plan((1ull << l) | fix_zero, fix_one);
  Offs<2> off{{1ull << l, partner_offset_amps}};
  const uint64_t n_pairs = 1ull << (ctx.n_local - 1 - __builtin_popcountll(fixed));
  const int rate = ctx.opt->exchange_rate_gbs;
  if (ctas > 0 || rate > 0) {
    // Grid-limited (persistent, grid-stride) variant: an exchange overlapped with local
    // passes needs only the SMs that saturate the link (NVLink 5: ~900 GB/s per direction,
    // an eighth of HBM), leaving the rest to the concurrent compute stream.  With a rate
    // (bytes per direction per ns = GB/s) each round of the grid is paced to it.
    if (ctas <= 0) ctas = 64;
    const uint64_t per_item = (uint64_t)(ctx.c64 ? 8 : 16) * (l > 0 ? 2 : 1);
    const uint64_t period =
        rate > 0 ? ((uint64_t)ctas * kThreads * per_item + rate - 1) / (uint64_t)rate : 0;
    if (ctx.c64)
      k_xswap<float><<<ctas, kThreads, 0, ctx.stream>>>(reinterpret_cast<cx<float>*>(ctx.amps),
                                                         n_pairs, l, partner_offset_amps, ip, period);
    else
      k_xswap<double><<<ctas, kThreads, 0, ctx.stream>>>(reinterpret_cast<cx<double>*>(ctx.amps),
                                                          n_pairs, l, partner_offset_amps, ip, period);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
    return;
  }
  if (ctx.c64)
    run_group<float, 2, 4, false>(ctx, n_pairs, ip, off, OpSwap2<float>{});
  else
    run_group<double, 2, 4, false>(ctx, n_pairs, ip, off, OpSwap2<double>{});
}

void launch_gate(const LaunchCtx& ctx, const Decoded& g) {
  if (ctx.soa) {
    launch_gate_soa(ctx, g);
    return;
  }
  if (ctx.c64)
    launch_gate_t<float>(ctx, g);
  else
    launch_gate_t<double>(ctx, g);
}

}  // namespace lfqs
