// fused_kernels.cu -- staging of several gates in one HBM pass.
//
// The paper applies every gate as its own pass and exposes every intermediate
// state; the optimised kernel of each gate is one pass over S (vector
// fusion).  On B200 a pass over a 16-128 GiB state costs 5-35 ms of
// HBM time while the arithmetic of one gate costs far less, so gates that only
// mix amplitudes inside a tile of 2^K amplitudes are applied in ONE pass
// (LFQS_FUSE_LOW):
//   * a tile is qubits [0, lc) (one contiguous chunk of 2^lc amplitudes) plus
//     up to 8 further qubits claimed by the fused gates' targets (NEXT-1
//     "general cache-blocked fusion"); diagonal gates need no tile qubit (bits
//     outside the tile come from the tile index); controls outside the tile are
//     per-tile predicates;
//   * tiles move by TMA bulk copies (cp.async.bulk + mbarrier; one copy per
//     chunk, issued in parallel by the 32 lanes of warp 0), or by direct
//     coalesced loads/stores (LFQS_OPT_FUSE_TMA_MAX_CHUNKS);
//   * the gate program is a __grid_constant__ kernel parameter (<= 32 KB:
//     headers + a coefficient pool), read through the constant cache;
//   * amplitudes live in registers: thread `tid` of 256 holds tile elements
//     i = r * 256 + tid, r < 2^(K-8).  Diagonal gates, and 1-target gates on
//     register bits (8..K-1) or lane bits (0..4, via shfl.xor), are applied in
//     registers; 1-target gates on warp bits (5..7) and 2/3-target gates go
//     through the shared-memory tile;
//   * scheduling (run_fused_schedule) takes later gates into a pass when they
//     commute *exactly* with the gates they skip.
// Permutation and diagonal gates use exactly the unfused formulas (moves;
// RN complex multiply without FMA, skipped where the factor is exactly 1), so
// fused == unfused value-exactly for them; dense gates agree within rounding.
// Kernels are templated on the amplitude scalar S (double: complex128; float:
// complex64, NEXT-4); the program's coefficients are stored in double.
#include <cuda_runtime.h>

#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <string>
#include <type_traits>
#include <vector>

#include "cx.cuh"
#include "fused_prog.h"
#include "jit.h"
#include "planner.h"
#include "lfqs_internal.h"

namespace lfqs {

namespace {


__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ uint32_t ins0(uint32_t p, int t) {
  return ((p >> t) << (t + 1)) | (p & ((1u << t) - 1));
}
template <class C>
__device__ __forceinline__ bool is_one(C d) {
  return d.x == 1 && d.y == 0;
}
template <class S>
__device__ __forceinline__ cx<S> cvs(double2 z) {  // program coefficient -> amplitude type
  return mk<S>((S)z.x, (S)z.y);
}

// ---- 2x2 functors (type dispatched once per op) ------------------------------
template <class S>
struct FX_ {
  __device__ __forceinline__ void pair(cx<S>& a0, cx<S>& a1) const {
    const cx<S> t = a0;
    a0 = a1;
    a1 = t;
  }
  __device__ __forceinline__ cx<S> lane(cx<S>, cx<S> p, int) const { return p; }
};
template <class S>
struct FY_ {
  __device__ __forceinline__ void pair(cx<S>& a0, cx<S>& a1) const {
    const cx<S> x0 = a0, x1 = a1;
    a0 = mk<S>(x1.y, -x1.x);
    a1 = mk<S>(-x0.y, x0.x);
  }
  __device__ __forceinline__ cx<S> lane(cx<S>, cx<S> p, int bit) const {
    return bit ? mk<S>(-p.y, p.x) : mk<S>(p.y, -p.x);
  }
};
template <class S>
struct FH_ {
  S s;
  __device__ __forceinline__ void pair(cx<S>& a0, cx<S>& a1) const {
    const cx<S> x0 = a0, x1 = a1;
    a0 = mk<S>(s * (x0.x + x1.x), s * (x0.y + x1.y));
    a1 = mk<S>(s * (x0.x - x1.x), s * (x0.y - x1.y));
  }
  // bit ? s (p - a) : s (a + p), written as s (p + (+-a)) -- the same values.
  __device__ __forceinline__ cx<S> lane(cx<S> a, cx<S> p, int bit) const {
    const S ax = bit ? -a.x : a.x, ay = bit ? -a.y : a.y;
    return mk<S>(s * (p.x + ax), s * (p.y + ay));
  }
};
template <class S>
struct FU_ {
  cx<S> c0, c1, c2, c3;
  __device__ __forceinline__ void pair(cx<S>& a0, cx<S>& a1) const {
    cx<S> b0 = mk<S>(0, 0), b1 = b0;
    cfma(b0, c0, a0);
    cfma(b0, c1, a1);
    cfma(b1, c2, a0);
    cfma(b1, c3, a1);
    a0 = b0;
    a1 = b1;
  }
  // Own amplitude first, partner second, in both lanes: only the coefficients
  // depend on the lane bit (the compiled passes select them once per op).
  // The lane's own coefficients moved to (c0, c1): lane(a, p, 0) of the result
  // equals lane(a, p, bit) -- selected once per op, so the loop keeps 2 of 4 live.
  static constexpr bool kSel = true;
  __device__ __forceinline__ FU_ sel(int bit) const {
    return bit ? FU_{c3, c2, c3, c2} : FU_{c0, c1, c0, c1};
  }
  __device__ __forceinline__ cx<S> lane(cx<S> a, cx<S> p, int bit) const {
    cx<S> acc = mk<S>(0, 0);
    cfma(acc, bit ? c3 : c0, a);
    cfma(acc, bit ? c2 : c1, p);
    return acc;
  }
};
template <class S>
struct FR_ {  // real 2x2 [[m00, m01], [m10, m11]]
  S m00, m01, m10, m11;
  __device__ __forceinline__ void pair(cx<S>& a0, cx<S>& a1) const {
    const cx<S> x0 = a0, x1 = a1;
    a0 = mk<S>(fma_(m01, x1.x, m00 * x0.x), fma_(m01, x1.y, m00 * x0.y));
    a1 = mk<S>(fma_(m11, x1.x, m10 * x0.x), fma_(m11, x1.y, m10 * x0.y));
  }
  static constexpr bool kSel = true;
  __device__ __forceinline__ FR_ sel(int bit) const {
    return bit ? FR_{m11, m10, m11, m10} : FR_{m00, m01, m00, m01};
  }
  __device__ __forceinline__ cx<S> lane(cx<S> a, cx<S> p, int bit) const {
    const S A = bit ? m11 : m00, B = bit ? m10 : m01;  // own, partner coefficient
    return mk<S>(fma_(B, p.x, A * a.x), fma_(B, p.y, A * a.y));
  }
};
template <class S>
struct FI_ {  // [[d0, i e01], [i e10, d1]] with real d0, d1, e01, e10
  S d0, e01, e10, d1;
  __device__ __forceinline__ void pair(cx<S>& a0, cx<S>& a1) const {
    const cx<S> x0 = a0, x1 = a1;  // i e x = (-e x.y, e x.x)
    a0 = mk<S>(fma_(-e01, x1.y, d0 * x0.x), fma_(e01, x1.x, d0 * x0.y));
    a1 = mk<S>(fma_(d1, x1.x, -e10 * x0.y), fma_(d1, x1.y, e10 * x0.x));
  }
  static constexpr bool kSel = true;
  __device__ __forceinline__ FI_ sel(int bit) const {
    return bit ? FI_{d1, e10, e10, d1} : FI_{d0, e01, e01, d0};
  }
  __device__ __forceinline__ cx<S> lane(cx<S> a, cx<S> p, int bit) const {
    const S D = bit ? d1 : d0, E = bit ? e10 : e01;  // own diagonal, partner (imaginary) entry
    return mk<S>(fma_(-E, p.y, D * a.x), fma_(E, p.x, D * a.y));
  }
};

// ---- shared-memory path ----------------------------------------------------------
template <class S, class F>
__device__ __forceinline__ void smem_pairs(cx<S>* tile, const F& f, int t, uint32_t mlo,
                                           uint32_t plo, uint32_t T) {
  for (uint32_t p = threadIdx.x; p < (T >> 1); p += kFThreads) {
    const uint32_t i0 = ins0(p, t), i1 = i0 | (1u << t);
    if ((i0 & mlo) != plo) continue;
    cx<S> a0 = tile[i0], a1 = tile[i1];
    f.pair(a0, a1);
    tile[i0] = a0;
    tile[i1] = a1;
  }
}

template <class S, int L>
__device__ __forceinline__ void dense_group(cx<S>* tile, const uint32_t (&idx)[L],
                                            const double2* c) {
  cx<S> v[L], w[L];
#pragma unroll
  for (int j = 0; j < L; ++j) v[j] = tile[idx[j]];
#pragma unroll
  for (int j = 0; j < L; ++j) {
    cx<S> acc = mk<S>(0, 0);
#pragma unroll
    for (int i = 0; i < L; ++i) cfma(acc, cvs<S>(c[j * L + i]), v[i]);
    w[j] = acc;
  }
#pragma unroll
  for (int j = 0; j < L; ++j) tile[idx[j]] = w[j];
}

template <class S>
__device__ void smem_op(cx<S>* tile, const FHdr& h, const double2* c, uint32_t T) {
  const uint32_t mlo = h.mlo, plo = h.plo;
  switch (h.type) {
    case F_X: smem_pairs<S>(tile, FX_<S>{}, h.t0, mlo, plo, T); return;
    case F_Y: smem_pairs<S>(tile, FY_<S>{}, h.t0, mlo, plo, T); return;
    case F_H: smem_pairs<S>(tile, FH_<S>{(S)c[0].x}, h.t0, mlo, plo, T); return;
    case F_UR:
      smem_pairs<S>(tile, FR_<S>{(S)c[0].x, (S)c[1].x, (S)c[2].x, (S)c[3].x}, h.t0, mlo, plo, T);
      return;
    case F_UI:
      smem_pairs<S>(tile, FI_<S>{(S)c[0].x, (S)c[1].y, (S)c[2].y, (S)c[3].x}, h.t0, mlo, plo, T);
      return;
    case F_U2:
      smem_pairs<S>(tile, FU_<S>{cvs<S>(c[0]), cvs<S>(c[1]), cvs<S>(c[2]), cvs<S>(c[3])}, h.t0, mlo,
                    plo, T);
      return;
    case F_SWAP: {
      const int lo = h.t0 < h.t1 ? h.t0 : h.t1, hi = h.t0 < h.t1 ? h.t1 : h.t0;
      for (uint32_t p = threadIdx.x; p < (T >> 2); p += kFThreads) {
        const uint32_t i = ins0(ins0(p, lo), hi);
        if ((i & mlo) != plo) continue;
        const uint32_t x = i | (1u << lo), y = i | (1u << hi);
        const cx<S> vx = tile[x];
        tile[x] = tile[y];
        tile[y] = vx;
      }
      return;
    }
    case F_U4: {
      const int t0 = h.t0, t1 = h.t1;
      const int lo = t0 < t1 ? t0 : t1, hi = t0 < t1 ? t1 : t0;
      for (uint32_t p = threadIdx.x; p < (T >> 2); p += kFThreads) {
        const uint32_t i = ins0(ins0(p, lo), hi);
        if ((i & mlo) != plo) continue;
        const uint32_t idx[4] = {i, i | (1u << t1), i | (1u << t0), i | (1u << t0) | (1u << t1)};
        dense_group<S, 4>(tile, idx, c);
      }
      return;
    }
    default: {  // F_U8
      const int s0 = h.t0, s1 = h.t1, s2 = h.t2;
      int a0 = s0 < s1 ? s0 : s1, a1 = s0 < s1 ? s1 : s0, a2 = s2;
      if (a2 < a1) { const int x = a1; a1 = a2; a2 = x; }
      if (a1 < a0) { const int x = a0; a0 = a1; a1 = x; }
      for (uint32_t p = threadIdx.x; p < (T >> 3); p += kFThreads) {
        const uint32_t i = ins0(ins0(ins0(p, a0), a1), a2);
        if ((i & mlo) != plo) continue;
        uint32_t idx[8];
#pragma unroll
        for (int j = 0; j < 8; ++j)
          idx[j] = i | (((j >> 2) & 1u) << s0) | (((j >> 1) & 1u) << s1) | ((j & 1u) << s2);
        dense_group<S, 8>(tile, idx, c);
      }
      return;
    }
  }
}

// ---- register path ---------------------------------------------------------------
template <int RB, int R, class C, class F>
__device__ __forceinline__ void reg_pairs(C (&v)[R], const F& f, uint32_t mlo, uint32_t plo,
                                          uint32_t tid) {
  if constexpr ((1 << RB) < R) {
    // Predicate split: thread bits once, register bits per r (uniform across the block).
    const bool bt = (tid & mlo & (kFThreads - 1)) == (plo & (kFThreads - 1));
    const uint32_t mr = mlo >> 8, pr = plo >> 8;
    if (!bt) return;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (r >> RB & 1) continue;
      if (((uint32_t)r & mr) != pr) continue;
      f.pair(v[r], v[r | (1 << RB)]);
    }
  }
}

template <class F, class = void>
struct lane_sel : std::false_type {};
template <class F>
struct lane_sel<F, std::void_t<decltype(F::kSel)>> : std::true_type {};

template <int R, class C, class F>
__device__ __forceinline__ void reg_lane(C (&v)[R], const F& f, int bit, int t0, uint32_t mlo,
                                         uint32_t plo, uint32_t tid) {
  const bool bt = (tid & mlo & (kFThreads - 1)) == (plo & (kFThreads - 1));
  const uint32_t mr = mlo >> 8, pr = plo >> 8;
  if (mlo == 0) {  // uncontrolled: every lane, every register
#pragma unroll
    for (int r = 0; r < R; ++r) {
      C p;
      p.x = __shfl_xor_sync(0xffffffffu, v[r].x, 1 << t0);
      p.y = __shfl_xor_sync(0xffffffffu, v[r].y, 1 << t0);
      v[r] = f.lane(v[r], p, bit);
    }
    return;
  }
#pragma unroll
  for (int r = 0; r < R; ++r) {
    if (((uint32_t)r & mr) != pr) continue;
    C p;
    p.x = __shfl_xor_sync(0xffffffffu, v[r].x, 1 << t0);
    p.y = __shfl_xor_sync(0xffffffffu, v[r].y, 1 << t0);
    if (bt) v[r] = f.lane(v[r], p, bit);
  }
}

template <int R, class C, class F>
__device__ __forceinline__ void reg_1q(C (&v)[R], const F& f, int t0, uint32_t mlo, uint32_t plo,
                                       uint32_t tid) {
  if (t0 >= 8) {
    switch (t0 - 8) {
      case 0: reg_pairs<0, R>(v, f, mlo, plo, tid); break;
      case 1: reg_pairs<1, R>(v, f, mlo, plo, tid); break;
      case 2: reg_pairs<2, R>(v, f, mlo, plo, tid); break;
      default: reg_pairs<3, R>(v, f, mlo, plo, tid); break;
    }
    return;
  }
  // Lane bit (t0 < 5): partner lane tid ^ 2^t0.  Register-bit part of the
  // predicate is uniform (skips whole registers); the thread part selects lanes.
  const int bit = (tid >> t0) & 1;
  if constexpr (lane_sel<F>::value)
    reg_lane(v, f.sel(bit), 0, t0, mlo, plo, tid);
  else
    reg_lane(v, f, bit, t0, mlo, plo, tid);
}

// F_DIAG1 on the registers r with (r & MR) == PR (MR, PR: register bits 8..11 of
// the predicate).  One instantiation per pattern with at most two register bits
// (all QFT / CPhase / CZ / T shapes); more bits take the generic loop.
template <int MR, int PR, int R, class C>
__device__ __forceinline__ void diag1_regs(C (&v)[R], const C d) {
#pragma unroll
  for (int r = 0; r < R; ++r)
    if ((r & MR) == PR) v[r] = cmul_rn(d, v[r]);
}

template <int R, class C>
__device__ __forceinline__ void diag1_dispatch(C (&v)[R], const C d, uint32_t code) {
#define LFQS_D1(MR, PR) \
  case ((MR) << 4) | (PR): diag1_regs<MR, PR, R>(v, d); return;
  switch (code) {
    LFQS_D1(0, 0)
    LFQS_D1(1, 0) LFQS_D1(1, 1) LFQS_D1(2, 0) LFQS_D1(2, 2)
    LFQS_D1(4, 0) LFQS_D1(4, 4) LFQS_D1(8, 0) LFQS_D1(8, 8)
    LFQS_D1(3, 0) LFQS_D1(3, 1) LFQS_D1(3, 2) LFQS_D1(3, 3)
    LFQS_D1(5, 0) LFQS_D1(5, 1) LFQS_D1(5, 4) LFQS_D1(5, 5)
    LFQS_D1(6, 0) LFQS_D1(6, 2) LFQS_D1(6, 4) LFQS_D1(6, 6)
    LFQS_D1(9, 0) LFQS_D1(9, 1) LFQS_D1(9, 8) LFQS_D1(9, 9)
    LFQS_D1(10, 0) LFQS_D1(10, 2) LFQS_D1(10, 8) LFQS_D1(10, 10)
    LFQS_D1(12, 0) LFQS_D1(12, 4) LFQS_D1(12, 8) LFQS_D1(12, 12)
    default: break;
  }
#undef LFQS_D1
  const uint32_t mr = code >> 4, pr = code & 15;
#pragma unroll
  for (int r = 0; r < R; ++r)
    if (((uint32_t)r & mr) == pr) v[r] = cmul_rn(d, v[r]);
}

// Factor of a DIAG1 / DIAGN op at tile element i of the tile at `base` (1 when
// its predicate fails).  Used to build phase tables.
template <class S>
__device__ __forceinline__ cx<S> diag_factor(const FHdr& g, const double2* pc, uint64_t base,
                                             uint32_t i) {
  if ((base & g.mhi) != g.phi || (i & g.mlo) != g.plo) return mk<S>(1, 0);
  const double2* c = pc + g.coef;
  if (g.type == F_DIAG1) return cvs<S>(c[0]);
  const int m = g.m;
  const int ts[3] = {g.t0, g.t1, g.t2};
  uint32_t j = 0;
#pragma unroll
  for (int s = 0; s < 3; ++s)
    if (s < m) {
      const uint32_t b = ts[s] >= 64 ? (uint32_t)((base >> (ts[s] - 64)) & 1) : (i >> ts[s]) & 1u;
      j |= b << (m - 1 - s);
    }
  return cvs<S>(c[j]);
}

// A phase-table member that holds for every entry of its table (jit.cpp hoisted_member).
__device__ __forceinline__ bool dtab_hoisted(const FHdr& g, uint32_t cm) {
  return g.type == F_DIAG1 && g.mlo == cm;
}

// Global amplitude index of tile element i (chunk = i >> lc, offset = low lc bits).
__device__ __forceinline__ uint64_t tile_addr(const FTile& tg, uint64_t base, uint32_t i) {
  uint64_t off = base | (i & ((1u << tg.lc) - 1));
  const uint32_t ch = i >> tg.lc;
  for (int k = 0; k < tg.nh; ++k) off |= (uint64_t)((ch >> k) & 1) << tg.hpos[k];
  return off;
}

// complex64 tiles are half the bytes: 4 CTAs per SM (64 registers) instead of 2
// (profiles/r01_c64_occupancy.md).
template <int K, bool DIRECT, class S>
__global__ void __launch_bounds__(kFThreads, sizeof(S) == 4 ? 4 : 2) k_fused(cx<S>* __restrict__ a,
                                                        uint64_t tile_ins,
                                                        const __grid_constant__ FProg prog) {
  using C = cx<S>;
  constexpr uint32_t T = 1u << K;
  constexpr int R = T / kFThreads;  // amplitudes per thread
  extern __shared__ __align__(128) unsigned char smem_raw[];
  C* tile = reinterpret_cast<C*>(smem_raw);
  __shared__ __align__(8) uint64_t bar;
  __shared__ C dtab[256];  // phase table of the current F_DTAB op
  const uint32_t tid = threadIdx.x;
  const FTile& tg = prog.tile;
  const int lc = tg.lc, nh = tg.nh;
  // Tile base: the tile index with zeros inserted at every tile qubit.  tile_ins (a
  // block of the state, for overlapped exchanges): up to three fixed bits inserted into
  // the tile index first (tile_insertions()).
  uint64_t t = blockIdx.x;
#pragma unroll
  for (int i = 0; i < 3; ++i) {
    const uint32_t b = (uint32_t)(tile_ins >> (8 * i)) & 0x7f;
    const int p = b & 63;
    const uint64_t lo = t & ((1ull << p) - 1);
    t = ((t - lo) << 1) | lo | ((uint64_t)(b >> 6) << p);
  }
  uint64_t base = t << lc;
  for (int i = 0; i < nh; ++i) {
    const int p = tg.hpos[i];
    const uint64_t lo = base & ((1ull << p) - 1);
    base = ((base - lo) << 1) | lo;
  }
  const uint32_t bytes = T * (uint32_t)sizeof(C), chunk_bytes = (uint32_t)sizeof(C) << lc;
  const uint32_t bar_a = smem_u32(&bar), tile_a = smem_u32(tile);
  C v[R];
  const int nops = prog.nops;
  if (DIRECT) {
    // Direct register loads (each warp reads 32 consecutive amplitudes of one
    // chunk per instruction, coalesced).
#pragma unroll
    for (int r = 0; r < R; ++r) v[r] = ld1(a + tile_addr(tg, base, (uint32_t)r * kFThreads + tid));
  } else {
    if (tid < 32) {
      // Lane 0 arms the barrier with the whole tile; the 32 lanes of warp 0 then
      // issue the chunk copies in parallel (a bulk copy costs ~50 SM cycles of
      // TMA service time whatever its size).
      if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar_a));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar_a),
                     "r"(bytes)
                     : "memory");
      }
      __syncwarp();
      for (uint32_t ch = tid; ch < (1u << nh); ch += 32) {
        uint64_t off = base;
        for (int i = 0; i < nh; ++i) off |= (uint64_t)((ch >> i) & 1) << tg.hpos[i];
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
                "r"(tile_a + ch * chunk_bytes),
            "l"(a + off), "r"(chunk_bytes), "r"(bar_a)
            : "memory");
      }
    }
    __syncthreads();  // barrier initialised before anyone waits on it
    {
      uint32_t done = 0;
      while (!done) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(bar_a)
            : "memory");
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) v[r] = tile[r * kFThreads + tid];
  }
  bool in_regs = true;  // else the authoritative copy is the smem tile

  for (int o = 0; o < nops; ++o) {
    const FHdr& h = prog.h[o];
    if ((base & h.mhi) != h.phi) continue;  // tile-level predicate (uniform)
    const int type = h.type;
    const uint32_t mlo = h.mlo, plo = h.plo;
    if (type == F_DTAB) {  // LFQS_FUSE_PHASE: one lookup + multiply for the m member ops
      const int nm = h.m;
      const uint32_t U = mlo, cm = plo & 0xffffu, cp = plo >> 16;
      const int nb = __popc(U);
      __syncthreads();  // the previous table's readers (and tile writers) are done
      if (tid < (1u << nb)) {
        // Entry tid: tile pattern with tid's bits deposited at U's positions.
        uint32_t ie = cp, u = U;
        for (int b = 0; b < nb; ++b) {
          const int pos = __ffs(u) - 1;
          u &= u - 1;
          ie |= ((tid >> b) & 1u) << pos;
        }
        // Members that hold for every entry (one-entry diagonals whose tile-bit predicate
        // is the common one: decided by the tile index alone) are a per-tile factor C; with
        // >= 2 of them the entry is C * (the other members' product), each product in
        // program order -- the pass compiler computes C once per tile (jit.cpp
        // dtab_factor), the same values.
        int nh = 0;
        for (int j = 1; j <= nm; ++j) nh += dtab_hoisted(prog.h[o + j], cm);
        C t = mk<S>(1, 0), cf = mk<S>(1, 0);
        for (int j = 1; j <= nm; ++j) {
          const C d = diag_factor<S>(prog.h[o + j], prog.c, base, ie);
          if (is_one(d)) continue;
          if (nh >= 2 && dtab_hoisted(prog.h[o + j], cm))
            cf = cmul_fma(d, cf);
          else
            t = cmul_fma(d, t);
        }
        if (nh >= 2) t = cmul_fma(cf, t);
        dtab[tid] = t;
      }
      if (!in_regs) {
#pragma unroll
        for (int r = 0; r < R; ++r) v[r] = tile[r * kFThreads + tid];
        in_regs = true;
      }
      __syncthreads();
      if ((tid & cm & (kFThreads - 1)) == (cp & (kFThreads - 1))) {
        // e(i) = pext(i, U): thread bits once, register bits as per-bit weights.
        uint32_t et = 0, u = U & (kFThreads - 1);
        for (int k = 0; u; ++k) {
          const int pos = __ffs(u) - 1;
          u &= u - 1;
          et |= ((tid >> pos) & 1u) << k;
        }
        uint32_t w[4];
        int k = __popc(U & (kFThreads - 1));
#pragma unroll
        for (int b = 0; b < 4; ++b) {
          w[b] = (U >> (8 + b) & 1) ? 1u << k : 0u;
          k += (U >> (8 + b)) & 1;
        }
        const uint32_t crm = cm >> 8, crp = cp >> 8;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (((uint32_t)r & crm) != crp) continue;
          uint32_t e = et;
#pragma unroll
          for (int b = 0; b < 4; ++b)
            if ((r >> b) & 1) e += w[b];
          v[r] = cmul_fma(dtab[e], v[r]);
        }
      }
      o += nm;
      continue;
    }
    if (type == F_DIAG1) {  // one diagonal entry d != 1 (the dominant op of phase-heavy programs)
      if (!in_regs) {
        __syncthreads();
#pragma unroll
        for (int r = 0; r < R; ++r) v[r] = tile[r * kFThreads + tid];
        in_regs = true;
      }
      // Split the predicate: thread bits (lanes that fail skip) and register
      // bits, dispatched to a compile-time register set so that no DP
      // instruction is issued for a register the predicate excludes.
      if ((tid & mlo & (kFThreads - 1)) == (plo & (kFThreads - 1)))
        diag1_dispatch<R>(v, cvs<S>(prog.c[h.coef]), ((mlo >> 8) << 4) | (plo >> 8));
      continue;
    }
    const int t0 = h.t0;
    const double2* c = prog.c + h.coef;
    const bool regpath = type <= F_DIAGN || (type <= F_U2 && (t0 < 5 || t0 >= 8));
    if (regpath && !in_regs) {
      __syncthreads();
#pragma unroll
      for (int r = 0; r < R; ++r) v[r] = tile[r * kFThreads + tid];
      in_regs = true;
    } else if (!regpath && in_regs) {
#pragma unroll
      for (int r = 0; r < R; ++r) tile[r * kFThreads + tid] = v[r];
      in_regs = false;
      __syncthreads();
    } else if (!regpath) {
      __syncthreads();
    }
    if (!regpath) {
      smem_op<S>(tile, h, c, T);
      continue;
    }
    switch (type) {
      case F_DIAGN: {  // factor d[j], j from the target bits (>= 64: outside the tile)
        const int m = h.m;
        if (m == 1) {  // Rz-like: two entries selected by one bit
          const C d0 = cvs<S>(c[0]), d1 = cvs<S>(c[1]);
          if (t0 >= 64) {
            const C d = ((base >> (t0 - 64)) & 1) ? d1 : d0;
#pragma unroll
            for (int r = 0; r < R; ++r) {
              const uint32_t i = (uint32_t)r * kFThreads + tid;
              if ((i & mlo) == plo) v[r] = cmul_rn(d, v[r]);
            }
          } else {
#pragma unroll
            for (int r = 0; r < R; ++r) {
              const uint32_t i = (uint32_t)r * kFThreads + tid;
              if ((i & mlo) == plo) v[r] = cmul_rn(((i >> t0) & 1) ? d1 : d0, v[r]);
            }
          }
          break;
        }
        const int ts[3] = {h.t0, h.t1, h.t2};
        uint32_t jh = 0, jmask = 0;
#pragma unroll
        for (int s = 0; s < 3; ++s)
          if (s < m) {
            if (ts[s] >= 64)  // a qubit outside the tile: its bit comes from the tile base
              jh |= (uint32_t)((base >> (ts[s] - 64)) & 1) << (m - 1 - s);
            else
              jmask |= 1u << (m - 1 - s);
          }
        C dd[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) dd[j] = j < (1 << m) ? cvs<S>(c[j]) : mk<S>(1, 0);
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const uint32_t i = (uint32_t)r * kFThreads + tid;
          if ((i & mlo) != plo) continue;
          uint32_t j = jh;
#pragma unroll
          for (int s = 0; s < 3; ++s)
            if (s < m && (jmask >> (m - 1 - s) & 1)) j |= ((i >> ts[s]) & 1u) << (m - 1 - s);
          C d = dd[0];
#pragma unroll
          for (int q = 1; q < 8; ++q)
            if ((uint32_t)q == j) d = dd[q];
          if (!is_one(d)) v[r] = cmul_rn(d, v[r]);
        }
        break;
      }
      case F_X: reg_1q<R>(v, FX_<S>{}, t0, mlo, plo, tid); break;
      case F_Y: reg_1q<R>(v, FY_<S>{}, t0, mlo, plo, tid); break;
      case F_H: reg_1q<R>(v, FH_<S>{(S)c[0].x}, t0, mlo, plo, tid); break;
      case F_UR:
        reg_1q<R>(v, FR_<S>{(S)c[0].x, (S)c[1].x, (S)c[2].x, (S)c[3].x}, t0, mlo, plo, tid);
        break;
      case F_UI:
        reg_1q<R>(v, FI_<S>{(S)c[0].x, (S)c[1].y, (S)c[2].y, (S)c[3].x}, t0, mlo, plo, tid);
        break;
      default:
        reg_1q<R>(v, FU_<S>{cvs<S>(c[0]), cvs<S>(c[1]), cvs<S>(c[2]), cvs<S>(c[3])}, t0, mlo, plo,
                  tid);
        break;
    }
  }

  if (DIRECT) {
    if (!in_regs) {
      __syncthreads();
#pragma unroll
      for (int r = 0; r < R; ++r) v[r] = tile[r * kFThreads + tid];
    }
#pragma unroll
    for (int r = 0; r < R; ++r) st1(a + tile_addr(tg, base, (uint32_t)r * kFThreads + tid), v[r]);
    return;
  }
  if (in_regs) {
#pragma unroll
    for (int r = 0; r < R; ++r) tile[r * kFThreads + tid] = v[r];
  }
  // Make the generic-proxy smem writes visible to the async proxy, then the
  // lanes of warp 0 issue the bulk stores.
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (tid < 32) {
    for (uint32_t ch = tid; ch < (1u << nh); ch += 32) {
      uint64_t off = base;
      for (int i = 0; i < nh; ++i) off |= (uint64_t)((ch >> i) & 1) << tg.hpos[i];
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(a + off),
                   "r"(tile_a + ch * chunk_bytes), "r"(chunk_bytes)
                   : "memory");
    }
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    // Only the shared-memory source must outlive the copy; completion of the
    // global writes is ordered by the end of the grid (as in TMA-store epilogues).
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
  }
}

inline double2 D2(cplx z) { return make_double2(z.re, z.im); }

// Coefficient budget of one gate, an upper bound on what encode() appends for it after
// build_program's merges: any 1-target gate may end up merged into (or absorb) a dense
// 1-target neighbour, which is encoded as a full U2 (4 coefficients), so every 1-target
// gate is budgeted at 4 whatever its class.
int coef_count(const Decoded& g) {
  const int d = 1 << g.m;
  if (g.m == 1) return 4;
  if (g.m == 2) return 16;  // a 2-target gate may absorb 1-target gates (merge_2q): dense
  switch (g.cls) {
    case GClass::DIAG: return d;  // upper bound (DIAG1 uses 1)
    case GClass::PERM_X: case GClass::PERM_Y: case GClass::PERM_SWAP: return 0;
    default: return d * d;
  }
}

// tb[q] = tile bit of qubit q, or -1 when q is not a tile qubit.
struct TileMap {
  int tb[64];
};

// Appends gate g to the program (program space was checked by the caller).
void encode(const Decoded& g, const TileMap& tm, FProg& P) {
  if (g.cls == GClass::NOOP) return;
  require(P.nops < kMaxOps && P.ncoef + coef_count(g) <= kMaxCoef,
          "internal: fused program over its op / coefficient budget");
  FHdr& h = P.h[P.nops];
  std::memset(&h, 0, sizeof h);
  uint64_t mlo = 0, plo = 0, mhi = 0, phi = 0;
  // A fixed bit of qubit q with value b: a per-amplitude condition on its tile
  // bit, or a per-tile condition on the global bit when q is not in the tile.
  auto fix = [&](int q, int b) {
    if (tm.tb[q] >= 0) {
      mlo |= 1ull << tm.tb[q];
      plo |= (uint64_t)b << tm.tb[q];
    } else {
      mhi |= 1ull << q;
      phi |= (uint64_t)b << q;
    }
  };
  for (int q = 0; q < 64; ++q)
    if (g.cmask >> q & 1) fix(q, 1);
  auto tbit = [&](int s) { return tm.tb[g.targets[s]] >= 0 ? tm.tb[g.targets[s]] : 64 + g.targets[s]; };
  h.m = (uint8_t)g.m;
  h.t0 = (uint8_t)tbit(0);
  h.t1 = (uint8_t)(g.m > 1 ? tbit(1) : 0);
  h.t2 = (uint8_t)(g.m > 2 ? tbit(2) : 0);
  h.coef = (uint16_t)P.ncoef;
  const int d = 1 << g.m;
  switch (g.cls) {
    case GClass::DIAG: {
      int n_active = 0, active = 0;
      for (int j = 0; j < d; ++j) {
        const cplx z = g.M[j * d + j];
        if (!(z.re == 1.0 && z.im == 0.0)) {
          ++n_active;
          active = j;
        }
      }
      if (n_active == 0) return;
      if (n_active == 1) {
        h.type = F_DIAG1;
        for (int s = 0; s < g.m; ++s) fix(g.targets[s], (active >> (g.m - 1 - s)) & 1);
        P.c[P.ncoef++] = D2(g.M[active * d + active]);
      } else {
        h.type = F_DIAGN;
        for (int j = 0; j < d; ++j) P.c[P.ncoef++] = D2(g.M[j * d + j]);
      }
      break;
    }
    case GClass::PERM_X: h.type = F_X; break;
    case GClass::PERM_Y: h.type = F_Y; break;
    case GClass::PERM_SWAP: h.type = F_SWAP; break;
    default:
      if (g.m == 1) {
        h.type = g.is_h ? F_H : F_U2;
        if (!g.is_h) {
          const cplx* M = g.M;
          if (M[0].im == 0.0 && M[1].im == 0.0 && M[2].im == 0.0 && M[3].im == 0.0)
            h.type = F_UR;
          else if (M[0].im == 0.0 && M[3].im == 0.0 && M[1].re == 0.0 && M[2].re == 0.0)
            h.type = F_UI;
        }
      } else {
        h.type = g.m == 2 ? F_U4 : F_U8;
      }
      if (g.is_h) {
        P.c[P.ncoef++] = D2(g.M[0]);
      } else {
        for (int i = 0; i < d * d; ++i) P.c[P.ncoef++] = D2(g.M[i]);
      }
      break;
  }
  h.mlo = (uint32_t)mlo;
  h.plo = (uint32_t)plo;
  h.mhi = mhi;
  h.phi = phi;
  ++P.nops;
}

template <int K, bool DIRECT, class S>
void launch_kd(const LaunchCtx& ctx, const FProg& P, uint64_t tile_ins) {
  const size_t smem = sizeof(cx<S>) << K;
  ensure_smem_attr((const void*)k_fused<K, DIRECT, S>, (int)smem);
  const uint64_t tiles = 1ull << (ctx.n_local - K);
  k_fused<K, DIRECT, S><<<(unsigned)tiles, kFThreads, smem, ctx.stream>>>(
      reinterpret_cast<cx<S>*>(ctx.amps), tile_ins, P);
}
// TMA bulk copies for tiles of at most fuse_tma_max_chunks chunks (default: all),
// direct register loads otherwise.
template <int K>
void launch_k(const LaunchCtx& ctx, const FProg& P, uint64_t tile_ins) {
  const bool direct = (1 << P.tile.nh) > ctx.opt->fuse_tma_max_chunks;
  if (ctx.c64) {
    if (direct)
      launch_kd<K, true, float>(ctx, P, tile_ins);
    else
      launch_kd<K, false, float>(ctx, P, tile_ins);
  } else {
    if (direct)
      launch_kd<K, true, double>(ctx, P, tile_ins);
    else
      launch_kd<K, false, double>(ctx, P, tile_ins);
  }
}

struct TileCfg {
  int K, L, slots;
};

bool tile_cfg(const LaunchCtx& ctx, int tile_qubits, TileCfg* c) {
  int K = tile_qubits < ctx.n_local ? tile_qubits : ctx.n_local;
  if (K > kMaxK) K = kMaxK;
  if (K < kMinK) return false;
  int L = ctx.opt->fuse_low_qubits > 0 ? ctx.opt->fuse_low_qubits : 7;  // 0: auto (7 here)
  if (L > K) L = K;
  if (L < K - kMaxHigh) L = K - kMaxHigh;
  c->K = K;
  c->L = L;
  c->slots = K - L;
  return true;
}

// Qubits a non-diagonal gate needs in the tile that it does not have yet.
uint64_t tile_need(const Decoded& g, uint64_t in_tile) {
  if (g.cls == GClass::DIAG) return 0;
  uint64_t need = 0;
  for (int s = 0; s < g.m; ++s)
    if (!(in_tile >> g.targets[s] & 1)) need |= 1ull << g.targets[s];
  return need;
}

uint64_t qubit_mask(const Decoded& g) {
  uint64_t m = g.cmask;
  for (int s = 0; s < g.m; ++s) m |= 1ull << g.targets[s];
  return m;
}

bool is_diag_op(const FHdr& h) { return h.type == F_DIAG1 || h.type == F_DIAGN; }

// Tile bits an encoded diagonal op reads: its predicate bits and, for DIAGN,
// its in-tile target bits.
uint32_t diag_support(const FHdr& h) {
  uint32_t u = h.mlo;
  if (h.type == F_DIAGN) {
    const int ts[3] = {h.t0, h.t1, h.t2};
    for (int s = 0; s < h.m; ++s)
      if (ts[s] < 64) u |= 1u << ts[s];
  }
  return u;
}

// LFQS_FUSE_PHASE: every maximal run of consecutive diagonal ops in the program
// (diagonal matrices commute, so their product is order-free up to rounding) is
// cut greedily, in program order, into groups whose table bits -- the union of
// the members' tile bits minus the bits every member fixes to the same value
// (the common predicate) -- number <= 8; a group of >= kMinTable members is
// preceded by an F_DTAB header and evaluated as one table per tile.
constexpr int kMinTable = 3;
constexpr int kTableBits = 8;
// A diagonal op whose factor depends on the tile (out-of-tile fixed bits or targets).
bool tile_dependent(const FHdr& h) {
  if (h.mhi != 0) return true;
  if (h.type == F_DIAGN) {
    const int ts[3] = {h.t0, h.t1, h.t2};
    for (int s = 0; s < h.m; ++s)
      if (ts[s] >= 64) return true;
  }
  return false;
}

// split: each run is first stable-partitioned into tile-invariant and tile-dependent
// members (LFQS_OPT_FUSE_PHASE_SPLIT).  A tile-dependent member (e.g. a QFT CPhase whose
// control lies outside the tile) adds no table bits, but every table entry evaluates it;
// grouped apart, such members usually share their in-tile bits as a common predicate and
// form a table of very few entries, so the per-tile build does ~1/256 of the work.
// Hadamard scales folded (LFQS_OPT_FUSE_H_SCALE, default 1).  Every amplitude of a tile
// passes through each unpredicated Hadamard exactly once, so the k factors 1/sqrt(2) of a
// pass's k >= 2 unpredicated F_H ops are one uniform scalar (1/sqrt(2))^k: the last of them
// carries it (2^(-k/2) exactly for even k) and the others compute the unscaled butterfly
// (a + b, a - b) -- coefficient 1, an exact product the pass compiler drops.  Linear ops
// commute with a scalar, so the pass computes the same state up to rounding (dense
// tolerance class; H is dense): 2 FP64 multiplies per amplitude per folded Hadamard fewer
// (QFT / Grover / QPE passes).  Interpreter and pass compiler run the same program.
// Global phase of a dense 1-target matrix (static matrix specialisation, up to a
// phase): U = z R, |z| = 1, with R real (kind 1: F_UR) or with a real diagonal and an
// imaginary off-diagonal (kind 2: F_UI) -- 4 FP64 operations per amplitude instead of 8.
// The parts dropped from R must be below 1e-15 of the largest entry (e.g. sqrt(X) =
// e^{i pi/4} Rx(pi/2), sqrt(Y) = e^{i pi/4} Ry(pi/2)).  Returns 0 when U has no such form.
int phase_real_form(const cplx* M, cplx* R, cplx* z) {
  double best = 0.0;
  for (int i = 0; i < 4; ++i) best = std::max(best, std::hypot(M[i].re, M[i].im));
  if (best == 0.0) return 0;
  const double tol = 1e-15 * best;
  for (int i = 0; i < 4; ++i) {
    if (std::hypot(M[i].re, M[i].im) < 0.25 * best) continue;
    for (int rot = 0; rot < 2; ++rot) {
      const double a = std::atan2(M[i].im, M[i].re) + (rot ? M_PI / 2 : 0.0);
      const double zr = std::cos(a), zi = std::sin(a);
      cplx T[4];
      for (int k = 0; k < 4; ++k)  // conj(z) * M
        T[k] = cplx{M[k].re * zr + M[k].im * zi, M[k].im * zr - M[k].re * zi};
      bool real = true, ui = true;
      for (int k = 0; k < 4; ++k) {
        real &= std::fabs(T[k].im) <= tol;
        ui &= (k == 0 || k == 3) ? std::fabs(T[k].im) <= tol : std::fabs(T[k].re) <= tol;
      }
      if (!real && !ui) continue;
      for (int k = 0; k < 4; ++k) {
        R[k] = T[k];
        if (real || k == 0 || k == 3)
          R[k].im = 0.0;
        else
          R[k].re = 0.0;
      }
      *z = cplx{zr, zi};
      return real ? 1 : 2;
    }
  }
  // kind 3: a real diagonal after the phase, any off-diagonal (sqrt W = e^{i pi/4} R): stays
  // F_U2, the pass compiler drops the diagonal's zero imaginary parts (12 FP64 operations per
  // pair instead of 16)
  for (int i = 0; i < 4; i += 3) {
    if (std::hypot(M[i].re, M[i].im) < 0.25 * best) continue;
    const double a = std::atan2(M[i].im, M[i].re);
    const double zr = std::cos(a), zi = std::sin(a);
    cplx T[4];
    for (int k = 0; k < 4; ++k)
      T[k] = cplx{M[k].re * zr + M[k].im * zi, M[k].im * zr - M[k].re * zi};
    if (std::fabs(T[0].im) > tol || std::fabs(T[3].im) > tol) continue;
    for (int k = 0; k < 4; ++k) R[k] = T[k];
    R[0].im = R[3].im = 0.0;
    *z = cplx{zr, zi};
    return 3;
  }
  return 0;
}

// Global phases taken out of a pass's dense 1-target gates (LFQS_OPT_FUSE_PHASE_EXTRACT,
// default 1).  Every unpredicated F_U2 op that is z R with R of a 4-operation form
// (phase_real_form) becomes that form, and the product of the z's -- a uniform scalar,
// which commutes with every linear op of the pass -- is multiplied into one remaining
// unpredicated F_U2 op's coefficients (a gate without such a form, else the last
// convertible one stays F_U2 and carries it).  4 FP64 operations per amplitude fewer per
// converted gate; rounding changes only (dense tolerance class).  Interpreter and pass
// compiler run the same program.
void extract_phases(FProg& P) {
  std::vector<int> conv;
  int carrier = -1;
  for (int o = 0; o < P.nops; ++o) {
    const FHdr& h = P.h[o];
    if (h.type != F_U2 || h.mlo || h.mhi) continue;
    cplx M[4], R[4], z;
    for (int k = 0; k < 4; ++k) M[k] = cplx{P.c[h.coef + k].x, P.c[h.coef + k].y};
    const int kind = phase_real_form(M, R, &z);
    // kind 3 pays only if the diagonal had imaginary parts to drop
    if (kind == 1 || kind == 2 || (kind == 3 && (M[0].im != 0.0 || M[3].im != 0.0)))
      conv.push_back(o);
    else
      carrier = o;
  }
  if (conv.empty()) return;
  if (carrier < 0) {
    if (conv.size() < 2) return;
    carrier = conv.back();
    conv.pop_back();
  }
  cplx Z{1.0, 0.0};
  for (int o : conv) {
    FHdr& h = P.h[o];
    cplx M[4], R[4], z;
    for (int k = 0; k < 4; ++k) M[k] = cplx{P.c[h.coef + k].x, P.c[h.coef + k].y};
    const int kind = phase_real_form(M, R, &z);
    h.type = kind == 1 ? F_UR : kind == 2 ? F_UI : F_U2;
    for (int k = 0; k < 4; ++k) P.c[h.coef + k] = D2(R[k]);
    Z = cplx{Z.re * z.re - Z.im * z.im, Z.re * z.im + Z.im * z.re};
  }
  const FHdr& hc = P.h[carrier];
  for (int k = 0; k < 4; ++k) {
    const double2 c = P.c[hc.coef + k];
    P.c[hc.coef + k] = make_double2(Z.re * c.x - Z.im * c.y, Z.re * c.y + Z.im * c.x);
  }
}

void fold_h_scales(FProg& P) {
  int k = 0, last = -1;
  for (int o = 0; o < P.nops; ++o) {
    const FHdr& h = P.h[o];
    if (h.type == F_H && h.mlo == 0 && h.mhi == 0) {
      ++k;
      last = o;
    }
  }
  if (k < 2) return;
  const double s = (k & 1) ? std::ldexp(M_SQRT1_2, -(k - 1) / 2) : std::ldexp(1.0, -k / 2);
  for (int o = 0; o < P.nops; ++o) {
    const FHdr& h = P.h[o];
    if (h.type == F_H && h.mlo == 0 && h.mhi == 0) P.c[h.coef] = double2{o == last ? s : 1.0, 0.0};
  }
}

void merge_phase_runs(FProg& P, bool split) {
  static thread_local FHdr out[kMaxOps];
  static thread_local FHdr run[kMaxOps];
  int no = 0, o = 0;
  const int n = P.nops;
  int spare = kMaxOps - n;  // room for F_DTAB headers
  while (o < n) {
    if (!is_diag_op(P.h[o])) {
      out[no++] = P.h[o++];
      continue;
    }
    int e = o;
    while (e < n && is_diag_op(P.h[e])) ++e;
    int nr = 0;
    if (split) {
      for (int k = o; k < e; ++k)
        if (!tile_dependent(P.h[k])) run[nr++] = P.h[k];
    }
    const int ninv = nr;
    for (int k = o; k < e; ++k)
      if (!split || tile_dependent(P.h[k])) run[nr++] = P.h[k];
    // groups never straddle the invariant / dependent boundary
    for (int part = 0; part < 2; ++part) {
      const int b0 = part == 0 ? 0 : ninv, b1 = part == 0 ? ninv : nr;
      for (int i = b0; i < b1;) {
        uint32_t cm = run[i].mlo, cp = run[i].plo & cm, sup = diag_support(run[i]);
        int j = i + 1;
        for (; j < b1 && j - i < 255; ++j) {
          const FHdr& g = run[j];
          const uint32_t cm2 = cm & g.mlo & ~(cp ^ g.plo);
          const uint32_t sup2 = sup | diag_support(g);
          if (__builtin_popcount(sup2 & ~cm2) > kTableBits) break;
          cm = cm2;
          cp &= cm2;
          sup = sup2;
        }
        if (j - i >= kMinTable && spare > 0) {
          FHdr t;
          std::memset(&t, 0, sizeof t);
          t.type = F_DTAB;
          t.m = (uint8_t)(j - i);
          t.mlo = sup & ~cm;
          t.plo = cm | (cp << 16);
          out[no++] = t;
          --spare;
        }
        for (int k = i; k < j; ++k) out[no++] = run[k];
        i = j;
      }
    }
    o = e;
  }
  std::memcpy(P.h, out, sizeof(FHdr) * no);
  P.nops = no;
}

// ---- 2-target merges (LFQS_OPT_FUSE_MERGE_2Q) ---------------------------------------
// A dense 1-target gate next to a 2-target gate on a superset of its qubit (nothing in
// between touches it, so they are adjacent in the commuting order, Eq. 3) is folded
// into the 4x4 matrix on the host, and two 2-target gates on the same pair are multiplied,
// when the product costs fewer FP64 operations per amplitude than the gates did separately
// (cost_of).  Sycamore-like cycles (a
// dense 1-target gate on each qubit, then fSim on pairs) lose about a quarter of their FP64
// work; the heavy passes are FP64-bound (profiles/r02_heavy_passes.md).  Rounding changes
// only (dense tolerance class); permutation / diagonal-only pairs never merge.
// FP64 operations per amplitude of a d x d gate matrix as the kernels evaluate it: each
// coefficient costs 2 per nonzero real / imaginary part (x2 for the amplitude's two
// components), a coefficient +-1 or +-i is a move / negation (1), zeros cost nothing; a
// permutation class gate is pure moves (0).
int cost_of(const cplx* M, int d, GClass cls);
// A dense 1-target gate as a pass runs it: without controls, its phase-real form when it has
// one (extract_phases; the phase goes to a carrier op at no cost).
int cost_1q(const Decoded& u, bool extract) {
  cplx R[4], z;
  if (extract && u.cmask == 0 && u.cls == GClass::DENSE && phase_real_form(u.M, R, &z))
    return cost_of(R, 2, GClass::DENSE);
  return cost_of(u.M, 2, u.cls);
}

int cost_of(const cplx* M, int d, GClass cls) {
  if (cls == GClass::PERM_X || cls == GClass::PERM_Y || cls == GClass::PERM_SWAP) return 0;
  int c = 0;
  for (int i = 0; i < d * d; ++i) {
    const double re = M[i].re, im = M[i].im;
    if (re == 0.0 && im == 0.0) continue;
    if ((im == 0.0 && (re == 1.0 || re == -1.0)) || (re == 0.0 && (im == 1.0 || im == -1.0)))
      c += 1;
    else
      c += 2 * (re != 0.0) + 2 * (im != 0.0);
  }
  return c * 4 / d;  // x4: per amplitude in units of 1/4 (integer arithmetic)
}
void mat4_mul(const cplx* A, const cplx* B, cplx* C) {  // C = A B (row-major 4x4)
  for (int r = 0; r < 4; ++r)
    for (int c = 0; c < 4; ++c) {
      double re = 0.0, im = 0.0;
      for (int k = 0; k < 4; ++k) {
        const cplx x = A[r * 4 + k], y = B[k * 4 + c];
        re += x.re * y.re - x.im * y.im;
        im += x.re * y.im + x.im * y.re;
      }
      C[r * 4 + c] = cplx{re, im};
    }
}
// U on local bit `msb` ? 1 : 0 of a 4x4 (targets[0] = local bit 1): U (x) I or I (x) U.
void embed2(const cplx* U, bool msb, cplx* E) {
  for (int r = 0; r < 4; ++r)
    for (int c = 0; c < 4; ++c) {
      const int ur = msb ? r >> 1 : r & 1, uc = msb ? c >> 1 : c & 1;
      const int or_ = msb ? r & 1 : r >> 1, oc = msb ? c & 1 : c >> 1;
      E[r * 4 + c] = or_ == oc ? U[ur * 2 + uc] : cplx{0.0, 0.0};
    }
}
// M with its two local bits exchanged (the same gate with targets listed the other way).
void swap_bits4(const cplx* M, cplx* O) {
  auto p = [](int j) { return ((j & 1) << 1) | (j >> 1); };
  for (int r = 0; r < 4; ++r)
    for (int c = 0; c < 4; ++c) O[p(r) * 4 + p(c)] = M[r * 4 + c];
}
void set_dense4(Decoded& a, const cplx* M) {
  for (int i = 0; i < 16; ++i) a.M[i] = M[i];
  a.cls = GClass::DENSE;
  a.is_h = false;
  a.kind = LFQS_UNITARY2;
}

// A 1-target gate with exactly one control as the 2-target gate it is on (control, target):
// |0><0| (x) I + |1><1| (x) U, control = local bit 1 (targets[0]).
Decoded as_two_target(const Decoded& g) {
  Decoded h = g;
  const int c = __builtin_ctzll(g.cmask);
  h.m = 2;
  h.targets[0] = c;
  h.targets[1] = g.targets[0];
  h.targets[2] = 0;
  h.cmask = 0;
  h.is_h = false;
  h.kind = LFQS_UNITARY2;
  for (int i = 0; i < 16; ++i) h.M[i] = cplx{0.0, 0.0};
  h.M[0] = h.M[5] = cplx{1.0, 0.0};
  for (int r = 0; r < 2; ++r)
    for (int q = 0; q < 2; ++q) h.M[(2 + r) * 4 + 2 + q] = g.M[r * 2 + q];
  return h;
}

template <class LastTouching>
bool merge_2q(std::vector<Decoded>& prog, Decoded& g, LastTouching&& last_touching,
              const TileMap& tm, bool extract) {
  // Diagonal gates are left alone: they are nearly free inside a pass (phase tables fold
  // whole runs of them into one lookup) and stay exact.
  if (g.cls == GClass::DIAG) return false;
  if (g.m == 1 && __builtin_popcountll(g.cmask) == 1) {
    // CZ / CNOT / CPhase / CU: merge in its 4x4 form when that pays (e.g. the dense
    // 1-target gates on both its qubits right before it); otherwise it stays as it is.
    Decoded h = as_two_target(g);
    return merge_2q(prog, h, last_touching, tm, extract);
  }
  // A merged gate is dense: both of its targets must be tile qubits (diagonal gates may
  // act on qubits outside the tile, read from the tile index, a dense one may not).
  auto in_tile2 = [&](const Decoded& x) {
    return x.m == 2 && tm.tb[x.targets[0]] >= 0 && tm.tb[x.targets[1]] >= 0;
  };
  const uint64_t gq = qubit_mask(g);
  if (g.m == 1 && g.cls == GClass::DENSE) {
    // g after a 2-target gate a on (a0, a1) that g's target belongs to
    const long k = last_touching(gq);
    if (k < 0) return false;
    Decoded& a = prog[k];
    const int t = g.targets[0];
    if (a.m != 2 || a.cmask != g.cmask || (a.targets[0] != t && a.targets[1] != t) ||
        !in_tile2(a) || a.cls == GClass::DIAG)
      return false;
    cplx E[16], P[16];
    embed2(g.M, a.targets[0] == g.targets[0], E);
    mat4_mul(E, a.M, P);
    if (cost_of(P, 4, GClass::DENSE) >= cost_of(a.M, 4, a.cls) + cost_1q(g, extract))
      return false;
    set_dense4(a, P);
    return true;
  }
  if (g.m != 2 || g.cls == GClass::NOOP || !in_tile2(g)) return false;
  // two 2-target gates on the same pair
  const long k = last_touching(gq);
  if (k >= 0) {
    Decoded& a = prog[k];
    if (a.m == 2 && a.cmask == g.cmask && qubit_mask(a) == gq && a.cls != GClass::DIAG &&
        (a.cls == GClass::DENSE || g.cls == GClass::DENSE)) {
      cplx G[16], P[16];
      if (a.targets[0] == g.targets[0])
        for (int i = 0; i < 16; ++i) G[i] = g.M[i];
      else
        swap_bits4(g.M, G);
      mat4_mul(G, a.M, P);
      if (cost_of(P, 4, GClass::DENSE) < cost_of(a.M, 4, a.cls) + cost_of(G, 4, g.cls)) {
        set_dense4(a, P);
        return true;
      }
    }
  }
  // dense 1-target gates on g's targets right before it (nothing in between touches
  // their qubits): g . (U0 (x) U1)
  long ks[2] = {-1, -1};
  int cost_sep = cost_of(g.M, 4, g.cls);
  cplx P[16];
  for (int i = 0; i < 16; ++i) P[i] = g.M[i];
  for (int s2 = 0; s2 < 2; ++s2) {
    const uint64_t q = (1ull << g.targets[s2]) | g.cmask;
    const long j = last_touching(q);
    if (j < 0) continue;
    const Decoded& u = prog[j];
    if (u.m != 1 || u.cls != GClass::DENSE || u.cmask != g.cmask || u.targets[0] != g.targets[s2])
      continue;
    cplx E[16], T[16];
    embed2(u.M, s2 == 0, E);
    mat4_mul(P, E, T);
    for (int i = 0; i < 16; ++i) P[i] = T[i];
    cost_sep += cost_1q(u, extract);
    ks[s2] = j;
  }
  if (ks[0] < 0 && ks[1] < 0) return false;
  if (cost_of(P, 4, GClass::DENSE) >= cost_sep) return false;
  for (long j : ks)
    if (j >= 0) prog[j].cls = GClass::NOOP;  // absorbed into g
  set_dense4(g, P);
  prog.push_back(g);
  return true;
}

// Builds the tile geometry for qubit set in_tile (filled up to K qubits), merges
// same-qubit 1-target runs containing a dense gate, and encodes the program.
void build_program(const LaunchCtx& ctx, const TileCfg& cfg, uint64_t in_tile,
                   const std::vector<const Decoded*>& list, FProg& P) {
  const int K = cfg.K;
  for (int q = 0; q < ctx.n_local && __builtin_popcountll(in_tile) < K; ++q) in_tile |= 1ull << q;
  TileMap tm;
  P.nops = 0;
  P.ncoef = 0;
  int b = 0, lc = 0;
  std::memset(&P.tile, 0, sizeof P.tile);  // unused hpos entries too (JIT cache key)
  for (int q = 0; q < 64; ++q) {
    tm.tb[q] = -1;
    if (q < ctx.n_local && (in_tile >> q & 1)) {
      tm.tb[q] = b;
      if (b == q) {
        lc = q + 1;
      } else {
        P.tile.hpos[P.tile.nh++] = (uint8_t)q;
      }
      ++b;
    }
  }
  P.tile.lc = lc;
  require(b == K && lc + P.tile.nh == K, "internal: bad fused tile");
  // Merge runs of 1-target gates on the same qubit with the same controls when at
  // least one is dense (matrix product on the host; dense results are compared
  // within rounding, permutation/diagonal-only runs are never merged).  With
  // LFQS_OPT_FUSE_MERGE_COMMUTING the run may be interleaved with gates on other
  // qubits: g merges into the last earlier gate that touches any of its qubits
  // when that gate is a 1-target gate on the same target with the same controls --
  // every gate in between acts on disjoint qubits and commutes with g exactly
  // (Eq. 3), so e.g. the H layer and X layer of a Grover diffusion become
  // one dense layer.
  std::vector<Decoded> prog;
  prog.reserve(list.size());
  // index of the last live gate of prog touching any qubit in mask (within 256), or -1
  auto last_touching = [&](uint64_t mask) -> long {
    for (size_t k = prog.size(); k-- > 0 && prog.size() - k <= 256;)
      if (prog[k].cls != GClass::NOOP && (qubit_mask(prog[k]) & mask)) return (long)k;
    return -1;
  };
  for (const Decoded* gp : list) {
    if (gp->cls == GClass::NOOP) continue;
    Decoded g = *gp;
    if (ctx.opt->fuse_merge_2q && merge_2q(prog, g, last_touching, tm, ctx.opt->fuse_phase_extract))
      continue;
    if (!prog.empty()) {
      size_t ai = prog.size() - 1;
      if (ctx.opt->fuse_merge_commuting && g.m == 1) {
        const long k = last_touching(qubit_mask(g));
        if (k >= 0) ai = (size_t)k;
      }
      Decoded& a = prog[ai];
      if (a.cls != GClass::NOOP && a.m == 1 && g.m == 1 && a.targets[0] == g.targets[0] &&
          a.cmask == g.cmask &&
          (a.cls == GClass::DENSE || g.cls == GClass::DENSE)) {
        cplx Cm[4];
        for (int r = 0; r < 2; ++r)
          for (int c = 0; c < 2; ++c) {
            const cplx x = g.M[r * 2 + 0], y = a.M[0 * 2 + c], u = g.M[r * 2 + 1],
                       w = a.M[1 * 2 + c];
            Cm[r * 2 + c] = cplx{x.re * y.re - x.im * y.im + (u.re * w.re - u.im * w.im),
                                 x.re * y.im + x.im * y.re + (u.re * w.im + u.im * w.re)};
          }
        for (int k = 0; k < 4; ++k) a.M[k] = Cm[k];
        a.cls = GClass::DENSE;
        a.is_h = false;
        a.kind = LFQS_UNITARY1;
        continue;
      }
    }
    prog.push_back(g);
  }
  for (const Decoded& g : prog) encode(g, tm, P);
  if (ctx.opt->fuse_phase_extract) extract_phases(P);
  if (ctx.opt->fuse_h_scale) fold_h_scales(P);
  if (ctx.phase_tables) merge_phase_runs(P, ctx.opt->fuse_phase_split);
}

// Launches an encoded pass: the compiled kernel of its program (LFQS_FUSE_JIT)
// or the interpreting kernel k_fused<K>.
// The launch covers 2^(ctx.n_local - K) tiles; tile_ins (tile_insertions()) fixes up to
// three more bits of the tile index (a block of the state, for overlapped exchanges).
void launch_built(const LaunchCtx& ctx, int K, const FProg& P, const std::string* key = nullptr,
                  uint64_t tile_ins = kNoTileIns) {
  if (ctx.jit && (1 << P.tile.nh) <= ctx.opt->fuse_tma_max_chunks) {
    const int jc = jit_config(ctx, K, &P);
    jit_launch(ctx, P, K, key ? *key : jit_key(P, K, ctx.c64, jc), jc, tile_ins);
    ++*ctx.launch_counter;
    return;
  }
  switch (K) {
    case 8: launch_k<8>(ctx, P, tile_ins); break;
    case 9: launch_k<9>(ctx, P, tile_ins); break;
    case 10: launch_k<10>(ctx, P, tile_ins); break;
    case 11: launch_k<11>(ctx, P, tile_ins); break;
    default: launch_k<12>(ctx, P, tile_ins); break;
  }
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

void launch_program(const LaunchCtx& ctx, const TileCfg& cfg, uint64_t in_tile,
                    const std::vector<const Decoded*>& list) {
  static thread_local FProg P;  // ~32 KB, reused (copied into the launch)
  build_program(ctx, cfg, in_tile, list, P);
  launch_built(ctx, cfg.K, P);
}

}  // namespace

// Greedy segmentation of a gate prefix (NEXT-1 "general cache-blocked fusion"):
// the tile holds qubits [0, L) (contiguous, for coalesced 2^L-amplitude chunks)
// plus up to K - L further qubits claimed, in gate order, by the targets of
// non-diagonal gates; diagonal gates need no slot.  Free slots are filled with
// the lowest remaining qubits (larger contiguous chunks).
bool run_fused_circuit(const LaunchCtx& ctx, const std::vector<Decoded>& gates, size_t begin,
                       size_t end, int tile_qubits, size_t* consumed) {
  *consumed = 0;
  TileCfg cfg;
  if (!tile_cfg(ctx, tile_qubits, &cfg)) return false;
  uint64_t in_tile = (1ull << cfg.L) - 1;
  int used = 0, nops = 0, ncoef = 0;
  const int max_ops = ctx.phase_tables ? kMaxOps - 16 : kMaxOps;  // room for F_DTAB headers
  std::vector<const Decoded*> list;
  size_t i = begin;
  for (; i < end; ++i) {
    const Decoded& g = gates[i];
    if (g.cls == GClass::NOOP) continue;
    if (nops >= max_ops || ncoef + coef_count(g) > kMaxCoef) break;
    const uint64_t need = tile_need(g, in_tile);
    const int nn = __builtin_popcountll(need);
    if (used + nn > cfg.slots) break;
    in_tile |= need;
    used += nn;
    ++nops;
    ncoef += coef_count(g);
    list.push_back(&g);
  }
  if (nops < 2) return false;  // a single gate runs faster in its class kernel
  launch_program(ctx, cfg, in_tile, list);
  *consumed = i - begin;
  return true;
}

// Commutation-aware scheduling: each pass walks the remaining gates in order and
// takes every gate that fits the tile and commutes *exactly* with all gates it
// skips: disjoint qubits, and never two diagonal gates (whose multiplications on
// a shared amplitude would round differently in the other order).  Permutation /
// diagonal results therefore stay bit-identical to gate-by-gate application;
// dense gates reorder only across disjoint qubits (rounding-level differences).
//
// plan_fused_schedule builds the passes (and, for LFQS_FUSE_JIT, compiles them) without
// launching anything; launch_fused_pass runs one of them on any block of the state whose
// qubits include every qubit the pass touches (the executor runs boundary passes of an
// overlapped exchange part by part, state.cu).
// ---- bit-permutation pass (LFQS_OPT_FUSE_PERM) -------------------------------------------
// A run of SWAP gates composes into a permutation pi of the index bits (SWAP
// moves amplitudes only).  When pi is an involution (disjoint transpositions: QFT's final
// bit reversal), the tile bits S = {0..L-1} u pi({0..L-1}) are closed under it, and so is
// the rest: tile t (the free bits) maps to tile sigma(t), with sigma(sigma(t)) = t.  One CTA
// per tile pair loads both tiles (coalesced runs of 2^L amplitudes), then writes each
// destination element from the shared-memory copy of its source: every amplitude read
// and written once -- one HBM pass for the whole SWAP run instead of one per few SWAPs.
// Moves only: bit-identical to the SWAP gates.

template <class S, int EPT>
__global__ void __launch_bounds__(256) k_bitperm(cx<S>* __restrict__ a,
                                                 const __grid_constant__ PermArgs A) {
  extern __shared__ __align__(16) unsigned char perm_smem[];
  cx<S>* sm = reinterpret_cast<cx<S>*>(perm_smem);
  constexpr uint32_t T = 256u * EPT;  // 2^ns elements per tile
  // shared-memory slot of element e: one 16-B pad per 32 elements, so that the gather by
  // permuted index (lanes 32 elements apart for a bit reversal) hits distinct banks
  constexpr uint32_t TP = T + T / 32;
  auto slot = [](uint32_t e) { return e + (e >> 5); };
  const uint64_t t = blockIdx.x;
  uint64_t pt = 0, bt = 0, bp = 0;
  if (A.f0 >= 0 && A.rev) {  // QFT's bit reversal: contiguous tile-index bits, reversed
    pt = __brevll(t) >> (64 - A.nf);
    if (pt < t) return;  // the partner's CTA moves this pair
    bt = t << A.f0;
    bp = pt << A.f0;
  } else {
    for (int k = 0; k < A.nf; ++k) {
      const uint64_t b = (t >> k) & 1;
      pt |= b << A.fdst[k];
      bt |= b << A.fbit[k];
    }
    if (pt < t) return;  // the partner's CTA moves this pair
    for (int k = 0; k < A.nf; ++k) bp |= ((pt >> k) & 1) << A.fbit[k];
  }
  auto dep = [&](uint32_t e) {
    if (A.s_lo >= 0)  // two runs of tile bits: [0, s_lo) and [s_h0, ...)
      return (uint64_t)(e & ((1u << A.s_lo) - 1)) | ((uint64_t)(e >> A.s_lo) << A.s_h0);
    uint64_t o = 0;
#pragma unroll
    for (int k = 0; k < 16; ++k)
      if (k < A.ns) o |= (uint64_t)((e >> k) & 1) << A.sbit[k];
    return o;
  };
  const bool pair = pt != t;
  // element e = r * 256 + tid: its offset and its source element are ORs of a per-thread
  // part (tid's bits) and a per-r part (the same for every thread) -- the bit loops run once
  auto srcmap = [&](uint32_t e) {
    if (A.srev) return __brev(e) >> (32 - A.ns);
    uint32_t src = 0;
#pragma unroll
    for (int k = 0; k < 16; ++k)
      if (k < A.ns) src |= ((e >> A.sdst[k]) & 1u) << k;
    return src;
  };
  const uint64_t dt = dep(threadIdx.x);
  const uint32_t st = srcmap(threadIdx.x);
  uint64_t dr[EPT];
  uint32_t sr[EPT];
#pragma unroll
  for (int r = 0; r < EPT; ++r) {
    dr[r] = dep(r * 256u);
    sr[r] = srcmap(r * 256u);
  }
  // every load of both tiles in flight before the first shared-memory store
  cx<S> v[2 * EPT];
#pragma unroll
  for (int r = 0; r < EPT; ++r) {
    const uint64_t o = dt | dr[r];
    v[r] = ld1(a + (bt | o));
    if (pair) v[EPT + r] = ld1(a + (bp | o));
  }
#pragma unroll
  for (int r = 0; r < EPT; ++r) {
    sm[slot(r * 256u + threadIdx.x)] = v[r];
    if (pair) sm[TP + slot(r * 256u + threadIdx.x)] = v[EPT + r];
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < EPT; ++r) {
    // destination element e holds the source element whose bit k is e's bit sdst[k]
    const uint32_t src = st | sr[r];
    const uint64_t o = dt | dr[r];
    st1(a + (bp | o), sm[slot(src)]);
    if (pair) st1(a + (bt | o), sm[TP + slot(src)]);
  }
}

template <class S>
void launch_bitperm_t(const LaunchCtx& ctx, const PermArgs& A, unsigned tiles) {
  const size_t smem = (size_t)2 * sizeof(cx<S>) * ((1u << A.ns) + (1u << A.ns) / 32);
  auto* p = reinterpret_cast<cx<S>*>(ctx.amps);
  auto go = [&](auto kern) {
    ensure_smem_attr((const void*)kern, (int)smem);
    kern<<<tiles, 256, smem, ctx.stream>>>(p, A);
  };
  switch (A.ns) {
    case 8: go(k_bitperm<S, 1>); break;
    case 9: go(k_bitperm<S, 2>); break;
    case 10: go(k_bitperm<S, 4>); break;
    case 11: go(k_bitperm<S, 8>); break;
    default: go(k_bitperm<S, 16>); break;
  }
}

void launch_bitperm(const LaunchCtx& ctx, const PermArgs& A) {
  const uint64_t tiles = 1ull << A.nf;
  require(tiles < (1ull << 31) && A.ns >= 8 && A.ns <= 12,
          "internal: bad bit-permutation pass geometry");
  if (ctx.c64)
    launch_bitperm_t<float>(ctx, A, (unsigned)tiles);
  else
    launch_bitperm_t<double>(ctx, A, (unsigned)tiles);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

bool is_plain_swap(const Decoded& g) {
  return g.cls == GClass::PERM_SWAP && g.cmask == 0 && g.m == 2;
}

// The SWAPs of gates[b, e) (NOOPs skipped) as one permutation pass.  False when the
// composition is not an involution or the shard is too small for closed tiles.
bool plan_swap_run(const LaunchCtx& ctx, const std::vector<Decoded>& gates, size_t b, size_t e,
                   PermArgs* pa, uint64_t* moved) {
  const int nl = ctx.n_local;
  const size_t i = b;
  int pi[64];  // pi[q]: the position the data bit at q ends at
  for (int q = 0; q < 64; ++q) pi[q] = q;
  // tile bits: auto (1) = 10 (complex128: 2 x 16 KiB tiles; 12 bits' 2 x 64 KiB allow one
  // CTA per SM: 5.97 -> 10.2 ms for the n = 30 bit reversal; complex64 n = 31: 5.66 vs 8.18)
  const int max_bits = ctx.opt->fuse_perm == 1 ? 10 : ctx.opt->fuse_perm;
  for (size_t k = i; k < e; ++k) {
    const Decoded& g = gates[k];
    if (g.cls == GClass::NOOP) continue;
    const int x = g.targets[0], y = g.targets[1];
    for (int q = 0; q < nl; ++q) pi[q] = pi[q] == x ? y : pi[q] == y ? x : pi[q];
  }
  for (int q = 0; q < nl; ++q)
    if (pi[pi[q]] != q) return false;
  uint64_t S = 0;
  for (int L = 1; L <= nl; ++L) {  // the most low bits whose closure fits
    uint64_t s2 = 0;
    for (int q = 0; q < L; ++q) s2 |= (1ull << q) | (1ull << pi[q]);
    if (__builtin_popcountll(s2) > max_bits) break;
    S = s2;
  }
  if ((S & 31) != 31 || __builtin_popcountll(S) < 8 || nl - __builtin_popcountll(S) < 1)
    return false;
  PermArgs A;
  int sidx[64], fidx[64];
  for (int q = 0; q < nl; ++q) {
    if (S >> q & 1) {
      sidx[q] = A.ns;
      A.sbit[A.ns++] = (uint8_t)q;
    } else {
      fidx[q] = A.nf;
      A.fbit[A.nf++] = (uint8_t)q;
    }
  }
  for (int k = 0; k < A.ns; ++k) A.sdst[k] = (uint8_t)sidx[pi[A.sbit[k]]];
  for (int k = 0; k < A.nf; ++k) A.fdst[k] = (uint8_t)fidx[pi[A.fbit[k]]];
  bool contig = A.nf > 0, rev = A.nf > 0;
  for (int k = 0; k < A.nf; ++k) {
    contig &= A.fbit[k] == A.fbit[0] + k;
    rev &= A.fdst[k] == A.nf - 1 - k;
  }
  if (contig) A.f0 = A.fbit[0];
  A.rev = rev;
  int lo = 0;
  while (lo < A.ns && A.sbit[lo] == lo) ++lo;
  bool two_runs = true, srev = true;
  for (int k = lo; k < A.ns; ++k) two_runs &= A.sbit[k] == A.sbit[lo] + (k - lo);
  for (int k = 0; k < A.ns; ++k) srev &= A.sdst[k] == A.ns - 1 - k;
  if (two_runs) {
    A.s_lo = lo;
    A.s_h0 = lo < A.ns ? A.sbit[lo] : 0;
  }
  A.srev = srev;
  uint64_t mv = 0;
  for (int q = 0; q < nl; ++q)
    if (pi[q] != q) mv |= 1ull << q;
  *pa = A;
  *moved = mv;
  return true;
}

void plan_fused_core(const LaunchCtx& ctx_in, const std::vector<Decoded>& gates,
                     int tile_qubits, std::vector<FusedPass>& out);

// A trailing run of >= 3 uncontrolled SWAPs whose composition is an involution (QFT's final
// bit reversal) becomes a bit-permutation pass after the fused passes of the gates before
// it, when that saves passes (LFQS_OPT_FUSE_PERM).
void plan_fused_schedule(const LaunchCtx& ctx_in, const std::vector<Decoded>& gates,
                         int tile_qubits, std::vector<FusedPass>& out) {
  out.clear();
  struct Run {
    size_t b, e;
    std::shared_ptr<PermArgs> pa;
    uint64_t moved;
  };
  std::vector<Run> runs;
  if (ctx_in.opt->fuse_perm != 0 && !ctx_in.soa) {
    for (size_t k = 0; k < gates.size();) {
      if (!is_plain_swap(gates[k])) {
        ++k;
        continue;
      }
      size_t e = k;
      int count = 0;
      while (e < gates.size() && (is_plain_swap(gates[e]) || gates[e].cls == GClass::NOOP)) {
        count += is_plain_swap(gates[e]);
        ++e;
      }
      // trailing runs only: a run inside a circuit splits its fused runs, and the passes
      // around it got heavier than the SWAPs saved (QPE(30) with its inverse QFT's leading
      // bit reversal as a pass: 12 -> 9 passes but 67.7 -> 78.0 ms)
      size_t t = e;
      while (t < gates.size() && gates[t].cls == GClass::NOOP) ++t;
      PermArgs pa;
      uint64_t mv = 0;
      if (count >= 3 && t == gates.size() && plan_swap_run(ctx_in, gates, k, e, &pa, &mv))
        runs.push_back(Run{k, e, std::make_shared<PermArgs>(pa), mv});
      k = e;
    }
  }
  Options o = *ctx_in.opt;
  o.fuse_perm = 0;
  LaunchCtx sub = ctx_in;
  sub.opt = &o;
  if (!runs.empty() && !ctx_in.plan_only) {
    // keep the permutation passes only if they save passes: SWAPs next to diagonal-only
    // work (an inverse QFT's leading bit reversal after QPE's controlled phases) already
    // ride in passes that have tile slots to spare (host-only pass counts)
    auto count = [&](bool with) {
      uint64_t c = 0;
      LaunchCtx pc = with ? ctx_in : sub;
      pc.plan_only = true;
      pc.launch_counter = &c;
      std::vector<FusedPass> tmp;
      plan_fused_schedule(pc, gates, tile_qubits, tmp);
      return c;
    };
    if (count(true) >= count(false)) runs.clear();
  }
  if (runs.empty()) {
    plan_fused_core(ctx_in, gates, tile_qubits, out);
    return;
  }
  // the automatic low-qubit choice compares whole-run pass counts, permutation passes
  // included (QFT(30): 6 vs 5 passes -> L = 7, 36.7 ms, not L = 6's 38.7 ms)
  o.auto_extra_passes = (int)runs.size();
  auto segment = [&](size_t b, size_t e) {
    if (b >= e) return;
    std::vector<Decoded> part(gates.begin() + b, gates.begin() + e);
    std::vector<FusedPass> tmp;
    plan_fused_core(sub, part, tile_qubits, tmp);
    for (FusedPass& ps : tmp) {
      if (!ps.prog && !ps.perm) ps.gate += (int)b;
      out.push_back(std::move(ps));
    }
  };
  size_t at = 0;
  for (const Run& r : runs) {
    segment(at, r.b);
    if (ctx_in.plan_only) {
      ++*ctx_in.launch_counter;
    } else {
      FusedPass ps;
      ps.perm = r.pa;
      ps.qmask = ps.nd_mask = r.moved;
      out.push_back(std::move(ps));
    }
    at = r.e;
  }
  segment(at, gates.size());
}

void plan_fused_core(const LaunchCtx& ctx_in, const std::vector<Decoded>& gates,
                     int tile_qubits, std::vector<FusedPass>& out) {
  out.clear();
  // LFQS_OPT_FUSE_LOW_QUBITS = 0 (auto): plan the passes (host only) with 7, 6 and 5
  // contiguous low qubits per tile and take 6 only when it saves >= 20 % of the passes --
  // a 1-KiB-chunk tile costs ~10 % more per pass (twice the TMA copies) but claims one
  // more qubit (measured at n = 30: QFT 65 -> 60 ms, Grover 113 -> 109, GHZ 26 -> 24 with
  // 6; random layered, VQE, Sycamore-like and QPE faster with 7).
  Options auto_opt;
  LaunchCtx ctx = ctx_in;
  if (ctx_in.opt->fuse_low_qubits == 0 && !ctx_in.plan_only) {
    auto count = [&](int L) {
      Options o = *ctx_in.opt;
      o.fuse_low_qubits = L;
      uint64_t c = 0;
      LaunchCtx pc = ctx_in;
      pc.opt = &o;
      pc.plan_only = true;
      pc.launch_counter = &c;
      std::vector<FusedPass> tmp;
      plan_fused_core(pc, gates, tile_qubits, tmp);
      return c;
    };
    const uint64_t p7 = count(7), p6 = count(6);
    auto_opt = *ctx_in.opt;
    const uint64_t x = (uint64_t)ctx_in.opt->auto_extra_passes;
    auto_opt.fuse_low_qubits = ((p6 + x) * 5 <= (p7 + x) * 4) ? 6 : 7;
    // moves and Hadamards only (GHZ): passes are pure HBM streams, so 6 low qubits pay as
    // soon as they save more than the ~10 % a 1-KiB-chunk pass costs extra (GHZ(33): 6 -> 5
    // passes, 225 -> 204 ms); phase tables and dense gates keep the 20 % rule
    bool light = true;
    for (const Decoded& g : gates)
      light &= g.cls == GClass::NOOP || g.cls == GClass::PERM_X || g.cls == GClass::PERM_Y ||
               g.cls == GClass::PERM_SWAP || g.is_h;
    if (light && (p6 + x) * 11 < (p7 + x) * 10) auto_opt.fuse_low_qubits = 6;
    // 5 low qubits (512-B chunks, 128 bulk copies per tile: +46 % per pass for Grover(33))
    // only when that cuts the passes to <= 65 %: many light passes at large n (Grover(33):
    // 26 -> 16 passes, 1052 -> 947 ms); FP64-heavy circuits lose (random layered(33): 46 ->
    // 35 passes but 2514 -> 2764 ms), and their pass counts fall less
    const uint64_t pb = (auto_opt.fuse_low_qubits == 6 ? p6 : p7) + x, p5 = count(5) + x;
    if (p5 * 20 <= pb * 13) auto_opt.fuse_low_qubits = 5;
    ctx.opt = &auto_opt;
  }
  TileCfg cfg;
  std::vector<int> rest;
  for (size_t i = 0; i < gates.size(); ++i)
    if (gates[i].cls != GClass::NOOP) rest.push_back((int)i);
  auto nd_of = [&](const Decoded& g) {
    uint64_t m = 0;
    if (g.cls != GClass::DIAG)
      for (int t = 0; t < g.m; ++t) m |= 1ull << g.targets[t];
    return m;
  };
  auto single = [&](int gi) {
    FusedPass ps;
    ps.gate = gi;
    ps.qmask = qubit_mask(gates[gi]);
    ps.nd_mask = nd_of(gates[gi]);
    out.push_back(std::move(ps));
  };
  if (!tile_cfg(ctx, tile_qubits, &cfg)) {
    if (ctx.plan_only) {
      *ctx.launch_counter += rest.size();
      return;
    }
    for (int i : rest) single(i);
    return;
  }
  const bool jit_ok = ctx.jit && (1 << (cfg.K - cfg.L)) <= ctx.opt->fuse_tma_max_chunks;
  constexpr size_t kWindow = 4096;  // gates scanned per pass
  const int max_ops = ctx.phase_tables ? kMaxOps - 16 : kMaxOps;  // room for F_DTAB headers
  std::vector<char> taken(gates.size(), 0);
  size_t head = 0;  // rest[0, head) are done
  while (head < rest.size()) {
    uint64_t in_tile = (1ull << cfg.L) - 1, blocked_q = 0, blocked_nd = 0;
    bool blocked_diag = false;
    int used = 0, nops = 0, ncoef = 0;
    std::vector<const Decoded*> list;
    std::vector<int> picked;
    size_t scanned = 0;
    for (size_t p = head; p < rest.size() && scanned < kWindow; ++p) {
      const int gi = rest[p];
      if (taken[gi]) continue;
      ++scanned;
      const Decoded& g = gates[gi];
      const bool diag = g.cls == GClass::DIAG;
      const uint64_t qm = qubit_mask(g);
      // Exact mode: a diagonal may not pass a skipped diagonal (rounding order of
      // the phase products); LFQS_FUSE_PHASE: it may (tables round anyway), so
      // only skipped non-diagonal gates block it.
      bool ok = ctx.phase_tables && diag ? (qm & blocked_nd) == 0
                                         : (qm & blocked_q) == 0 && !(diag && blocked_diag);
      if (ok && nops < max_ops && ncoef + coef_count(g) <= kMaxCoef) {
        const uint64_t need = tile_need(g, in_tile);
        const int nn = __builtin_popcountll(need);
        if (used + nn <= cfg.slots) {
          in_tile |= need;
          used += nn;
          ++nops;
          ncoef += coef_count(g);
          list.push_back(&g);
          picked.push_back(gi);
          continue;
        }
      }
      blocked_q |= qm;  // later gates touching these qubits must wait
      if (!diag) blocked_nd |= qm;
      blocked_diag |= diag;
    }
    if (ctx.plan_only) {  // pass count only (auto tile geometry)
      ++*ctx.launch_counter;
      if (nops < 2) {
        while (taken[rest[head]]) ++head;
        taken[rest[head]] = 1;
      } else {
        for (int gi : picked) taken[gi] = 1;
      }
    } else if (nops < 2) {
      // Nothing to fuse with the first remaining gate: its class kernel.
      while (taken[rest[head]]) ++head;
      single(rest[head]);
      taken[rest[head]] = 1;
    } else {
      FusedPass ps;
      ps.prog.reset(new FProg);
      ps.K = cfg.K;
      build_program(ctx, cfg, in_tile, list, *ps.prog);
      for (int gi : picked) {
        ps.qmask |= qubit_mask(gates[gi]);
        ps.nd_mask |= nd_of(gates[gi]);
      }
      if (jit_ok) ps.key = jit_key(*ps.prog, cfg.K, ctx.c64, jit_config(ctx, cfg.K, ps.prog.get()));
      out.push_back(std::move(ps));
      for (int gi : picked) taken[gi] = 1;
    }
    while (head < rest.size() && taken[rest[head]]) ++head;
  }
  if (ctx.plan_only || !jit_ok) return;
  std::map<int, std::vector<std::pair<std::string, const FProg*>>> items;  // per generator config
  for (const FusedPass& ps : out)
    if (ps.prog) items[jit_config(ctx, cfg.K, ps.prog.get())].emplace_back(ps.key, ps.prog.get());
  for (const auto& it : items) jit_compile(it.second, cfg.K, ctx.c64, it.first);
}

void launch_fused_pass(const LaunchCtx& ctx, const std::vector<Decoded>& gates,
                       const FusedPass& ps) {
  if (ps.perm)
    launch_bitperm(ctx, *ps.perm);
  else if (ps.prog)
    launch_built(ctx, ps.K, *ps.prog, ps.key.empty() ? nullptr : &ps.key);
  else
    launch_gate(ctx, gates[ps.gate]);
}

// Block v of the chunk qubits (lfqs_internal.h): fused passes fix the chunk bits in the
// tile index (tile-index insertions), so the pass runs over the block's tiles only; a
// single gate runs on the contiguous block of the top chunk qubits, its controls and
// diagonal entries on them resolved on the host as the planner does for a rank's global
// bits (Planner::rank_local with the block index in the role of the rank).
bool pass_blockwise(const FusedPass& ps, uint64_t chunk, int n_local) {
  const int c = __builtin_popcountll(chunk);
  if (c == 0 || c > 3 || ps.perm || (ps.nd_mask & chunk) || (chunk >> n_local)) return false;
  if (!ps.prog) return chunk == (((1ull << c) - 1) << (n_local - c));
  if (ps.K > n_local - c) return false;
  const FTile& tg = ps.prog->tile;
  uint64_t in_tile = (1ull << tg.lc) - 1;
  for (int i = 0; i < tg.nh; ++i) in_tile |= 1ull << tg.hpos[i];
  return (chunk & in_tile) == 0;
}

namespace {
uint64_t tile_insertions(const FTile& tg, uint64_t chunk, uint64_t v) {
  uint64_t ins = kNoTileIns;
  int i = 0;
  for (int q = 0; q < 64; ++q) {
    if (!(chunk >> q & 1)) continue;
    int below = 0;  // tile qubits below q
    for (int h = 0; h < tg.nh; ++h) below += tg.hpos[h] < q;
    const int tp = q - tg.lc - below;  // q's position in the tile index
    require(q >= tg.lc && tp >= 0 && tp < 63 && i < 3, "internal: chunk qubit inside the tile");
    ins &= ~(0xffull << (8 * i));
    ins |= (uint64_t)(tp | (int)((v >> i) & 1) << 6) << (8 * i);
    ++i;
  }
  return ins;
}
}  // namespace

void launch_fused_pass_part(const LaunchCtx& ctx, const std::vector<Decoded>& gates,
                            const FusedPass& ps, uint64_t chunk, uint64_t v) {
  require(pass_blockwise(ps, chunk, ctx.n_local), "internal: pass not confined to the block");
  const int c = __builtin_popcountll(chunk);
  const int n_sub = ctx.n_local - c;
  if (ps.prog) {
    LaunchCtx x = ctx;  // same base pointer; the block's tiles only
    x.n_local = n_sub;
    launch_built(x, ps.K, *ps.prog, ps.key.empty() ? nullptr : &ps.key,
                 tile_insertions(ps.prog->tile, chunk, v));
    return;
  }
  Planner blk(ctx.n_local, 1 << c);
  Decoded lg;
  if (!blk.rank_local(gates[ps.gate], (int)v, 0, &lg) || lg.cls == GClass::NOOP) return;
  LaunchCtx x = ctx;
  x.amps = static_cast<unsigned char*>(ctx.amps) + (v << n_sub) * (ctx.c64 ? 8 : 16);
  x.n_local = n_sub;
  launch_gate(x, lg);
}

void run_fused_schedule(const LaunchCtx& ctx, const std::vector<Decoded>& gates,
                        int tile_qubits) {
  std::vector<FusedPass> passes;
  plan_fused_schedule(ctx, gates, tile_qubits, passes);
  if (ctx.plan_only) return;
  if (ctx.dry_run) {  // host-only (lfqs_jit_precompile): planned and compiled, not launched
    *ctx.launch_counter += passes.size();
    return;
  }
  for (const FusedPass& ps : passes) launch_fused_pass(ctx, gates, ps);
}

}  // namespace lfqs
