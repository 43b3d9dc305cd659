// fused_kernels.cu -- staging of consecutive gates in one HBM pass.
//
// The paper applies every gate as its own pass and exposes every intermediate
// state; the optimised kernel of each gate is one pass over S (vector
// fusion).  On B200 a pass over a 16-128 GiB state costs 5-35 ms of
// HBM time while the arithmetic of one gate costs far less, so a run of
// consecutive gates that only mix amplitudes inside a 2^K tile is applied in
// ONE pass (LFQS_FUSE_LOW):
//   * the tile (2^K contiguous amplitudes, K <= 12 -> 64 KiB) is staged into
//     shared memory with one TMA bulk copy (cp.async.bulk + mbarrier) and
//     written back with one bulk store;
//   * amplitudes then live in registers: thread `tid` of 256 holds tile
//     elements i = r * 256 + tid, r < 2^(K-8).  Diagonal gates, and 1-target
//     gates on register bits (8..K-1) or lane bits (0..4, via shfl.xor), are
//     applied in registers; 1-target gates on warp bits (5..7) and 2/3-target
//     gates go through the shared-memory tile;
//   * a gate fuses when all its targets are < K (controls anywhere: controls
//     >= K are a per-tile predicate) or when it is diagonal (any qubits: target
//     bits >= K come from the tile index).
// Permutation and diagonal gates use exactly the unfused formulas (moves;
// RN complex multiply without FMA, skipped where the factor is exactly 1), so
// fused == unfused value-exactly for them; dense gates agree within rounding.
#include <cuda_runtime.h>

#include <cstring>
#include <vector>

#include "lfqs_internal.h"

namespace lfqs {

namespace {

enum FType : int { F_DIAG = 0, F_X, F_Y, F_H, F_U2, F_SWAP, F_U4, F_U8 };

struct FOp {
  int type;
  int m;
  int t[3];        // targets (DIAG: any position; others: < K)
  int pad;
  uint64_t cl;     // controls below K (per amplitude)
  uint64_t ch;     // controls at or above K (per tile)
  double2 c[64];   // matrix row-major, or the diagonal d[j] for DIAG
};

constexpr int kFThreads = 256;
constexpr int kMaxOps = 256;
constexpr int kMinK = 8, kMaxK = 12;

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ double2 cmul_rn(double2 d, double2 a) {
  return make_double2(__dsub_rn(__dmul_rn(d.x, a.x), __dmul_rn(d.y, a.y)),
                      __dadd_rn(__dmul_rn(d.x, a.y), __dmul_rn(d.y, a.x)));
}
__device__ __forceinline__ void cfma(double2& acc, double2 m, double2 v) {
  acc.x = fma(m.x, v.x, acc.x);
  acc.x = fma(-m.y, v.y, acc.x);
  acc.y = fma(m.x, v.y, acc.y);
  acc.y = fma(m.y, v.x, acc.y);
}
__device__ __forceinline__ uint32_t ins0(uint32_t p, int t) {
  return ((p >> t) << (t + 1)) | (p & ((1u << t) - 1));
}
__device__ __forceinline__ bool is_one(double2 d) { return d.x == 1.0 && d.y == 0.0; }

// The 2x2 update of a pair (a0 = bit 0, a1 = bit 1), same formulas as apply_kernels.cu.
__device__ __forceinline__ void pair_update(int type, const FOp& op, double2& a0, double2& a1) {
  const double2 x0 = a0, x1 = a1;
  if (type == F_X) {
    a0 = x1;
    a1 = x0;
  } else if (type == F_Y) {
    a0 = make_double2(x1.y, -x1.x);
    a1 = make_double2(-x0.y, x0.x);
  } else if (type == F_H) {
    const double s = op.c[0].x;
    a0 = make_double2(s * (x0.x + x1.x), s * (x0.y + x1.y));
    a1 = make_double2(s * (x0.x - x1.x), s * (x0.y - x1.y));
  } else {
    double2 b0 = make_double2(0.0, 0.0), b1 = b0;
    cfma(b0, op.c[0], x0);
    cfma(b0, op.c[1], x1);
    cfma(b1, op.c[2], x0);
    cfma(b1, op.c[3], x1);
    a0 = b0;
    a1 = b1;
  }
}

template <int L>
__device__ __forceinline__ void dense_group(double2* tile, const uint32_t (&idx)[L],
                                            const double2* __restrict__ c) {
  double2 v[L], w[L];
#pragma unroll
  for (int j = 0; j < L; ++j) v[j] = tile[idx[j]];
#pragma unroll
  for (int j = 0; j < L; ++j) {
    double2 acc = make_double2(0.0, 0.0);
#pragma unroll
    for (int i = 0; i < L; ++i) cfma(acc, c[j * L + i], v[i]);
    w[j] = acc;
  }
#pragma unroll
  for (int j = 0; j < L; ++j) tile[idx[j]] = w[j];
}

// Non-register op on the shared-memory tile (T = 2^K amplitudes).
__device__ void smem_op(double2* tile, const FOp& op, uint32_t T) {
  const uint32_t cl = (uint32_t)op.cl;
  const int type = op.type;
  if (type <= F_U2) {
    const int t = op.t[0];
    for (uint32_t p = threadIdx.x; p < (T >> 1); p += kFThreads) {
      const uint32_t i0 = ins0(p, t), i1 = i0 | (1u << t);
      if ((i0 & cl) != cl) continue;
      double2 a0 = tile[i0], a1 = tile[i1];
      pair_update(type, op, a0, a1);
      tile[i0] = a0;
      tile[i1] = a1;
    }
  } else if (type == F_SWAP) {
    const int lo = op.t[0] < op.t[1] ? op.t[0] : op.t[1];
    const int hi = op.t[0] < op.t[1] ? op.t[1] : op.t[0];
    for (uint32_t p = threadIdx.x; p < (T >> 2); p += kFThreads) {
      const uint32_t i = ins0(ins0(p, lo), hi);
      if ((i & cl) != cl) continue;
      const uint32_t x = i | (1u << lo), y = i | (1u << hi);
      const double2 vx = tile[x];
      tile[x] = tile[y];
      tile[y] = vx;
    }
  } else if (type == F_U4) {
    const int t0 = op.t[0], t1 = op.t[1];
    const int lo = t0 < t1 ? t0 : t1, hi = t0 < t1 ? t1 : t0;
    for (uint32_t p = threadIdx.x; p < (T >> 2); p += kFThreads) {
      const uint32_t i = ins0(ins0(p, lo), hi);
      if ((i & cl) != cl) continue;
      const uint32_t idx[4] = {i, i | (1u << t1), i | (1u << t0), i | (1u << t0) | (1u << t1)};
      dense_group<4>(tile, idx, op.c);
    }
  } else {  // F_U8
    const int s0 = op.t[0], s1 = op.t[1], s2 = op.t[2];
    int a0 = s0 < s1 ? s0 : s1, a1 = s0 < s1 ? s1 : s0, a2 = s2;
    if (a2 < a1) { const int x = a1; a1 = a2; a2 = x; }
    if (a1 < a0) { const int x = a0; a0 = a1; a1 = x; }
    for (uint32_t p = threadIdx.x; p < (T >> 3); p += kFThreads) {
      const uint32_t i = ins0(ins0(ins0(p, a0), a1), a2);
      if ((i & cl) != cl) continue;
      uint32_t idx[8];
#pragma unroll
      for (int j = 0; j < 8; ++j)
        idx[j] = i | (((j >> 2) & 1u) << s0) | (((j >> 1) & 1u) << s1) | ((j & 1u) << s2);
      dense_group<8>(tile, idx, op.c);
    }
  }
}

// Register-path functors: the gate type is dispatched once per op, outside the
// unrolled per-register loops (keeps register pressure low).
struct RX_ {
  __device__ __forceinline__ void pair(double2& a0, double2& a1) const {
    const double2 t = a0;
    a0 = a1;
    a1 = t;
  }
  __device__ __forceinline__ double2 lane(double2, double2 p, int) const { return p; }
};
struct RY_ {
  __device__ __forceinline__ void pair(double2& a0, double2& a1) const {
    const double2 x0 = a0, x1 = a1;
    a0 = make_double2(x1.y, -x1.x);
    a1 = make_double2(-x0.y, x0.x);
  }
  __device__ __forceinline__ double2 lane(double2, double2 p, int bit) const {
    return bit ? make_double2(-p.y, p.x) : make_double2(p.y, -p.x);
  }
};
struct RH_ {
  double s;
  __device__ __forceinline__ void pair(double2& a0, double2& a1) const {
    const double2 x0 = a0, x1 = a1;
    a0 = make_double2(s * (x0.x + x1.x), s * (x0.y + x1.y));
    a1 = make_double2(s * (x0.x - x1.x), s * (x0.y - x1.y));
  }
  __device__ __forceinline__ double2 lane(double2 a, double2 p, int bit) const {
    return bit ? make_double2(s * (p.x - a.x), s * (p.y - a.y))
               : make_double2(s * (a.x + p.x), s * (a.y + p.y));
  }
};
struct RU_ {
  double2 c0, c1, c2, c3;
  __device__ __forceinline__ void pair(double2& a0, double2& a1) const {
    double2 b0 = make_double2(0.0, 0.0), b1 = b0;
    cfma(b0, c0, a0);
    cfma(b0, c1, a1);
    cfma(b1, c2, a0);
    cfma(b1, c3, a1);
    a0 = b0;
    a1 = b1;
  }
  __device__ __forceinline__ double2 lane(double2 a, double2 p, int bit) const {
    double2 acc = make_double2(0.0, 0.0);
    if (bit) {
      cfma(acc, c2, p);
      cfma(acc, c3, a);
    } else {
      cfma(acc, c0, a);
      cfma(acc, c1, p);
    }
    return acc;
  }
};

template <int RB, int R, class F>
__device__ __forceinline__ void reg_pairs(double2 (&v)[R], const F& f, uint32_t cl, uint32_t tid) {
  if constexpr ((1 << RB) < R) {
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (r >> RB & 1) continue;
      const uint32_t i0 = (uint32_t)r * kFThreads + tid;
      if ((i0 & cl) != cl) continue;
      f.pair(v[r], v[r | (1 << RB)]);
    }
  }
}

template <int R, class F>
__device__ __forceinline__ void reg_op(double2 (&v)[R], const F& f, int t0, uint32_t cl,
                                       uint32_t tid) {
  if (t0 >= 8) {
    switch (t0 - 8) {
      case 0: reg_pairs<0, R>(v, f, cl, tid); break;
      case 1: reg_pairs<1, R>(v, f, cl, tid); break;
      case 2: reg_pairs<2, R>(v, f, cl, tid); break;
      default: reg_pairs<3, R>(v, f, cl, tid); break;
    }
    return;
  }
  // Lane bit (t0 < 5): partner lane tid ^ 2^t0.
  const int bit = (tid >> t0) & 1;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    double2 p;
    p.x = __shfl_xor_sync(0xffffffffu, v[r].x, 1 << t0);
    p.y = __shfl_xor_sync(0xffffffffu, v[r].y, 1 << t0);
    const uint32_t i = (uint32_t)r * kFThreads + tid;
    if ((i & cl) == cl) v[r] = f.lane(v[r], p, bit);
  }
}

template <int K>
__global__ void __launch_bounds__(kFThreads, 2) k_fused(double2* __restrict__ a,
                                                        const FOp* __restrict__ prog, int nops) {
  constexpr uint32_t T = 1u << K;
  constexpr int R = T / kFThreads;  // amplitudes per thread
  extern __shared__ __align__(128) double2 tile[];
  __shared__ __align__(8) uint64_t bar;
  const uint32_t tid = threadIdx.x;
  const uint64_t base = (uint64_t)blockIdx.x << K;
  const uint32_t bytes = T * 16u;
  const uint32_t bar_a = smem_u32(&bar), tile_a = smem_u32(tile);
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar_a));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar_a), "r"(bytes)
                 : "memory");
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
            "r"(tile_a),
        "l"(a + base), "r"(bytes), "r"(bar_a)
        : "memory");
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
  double2 v[R];
#pragma unroll
  for (int r = 0; r < R; ++r) v[r] = tile[r * kFThreads + tid];
  bool in_regs = true;  // else the authoritative copy is the smem tile

  for (int o = 0; o < nops; ++o) {
    const FOp& op = prog[o];
    const uint64_t ch = op.ch;
    if ((base & ch) != ch) continue;  // a high control is 0 on this tile (uniform)
    const int type = op.type;
    const uint32_t cl = (uint32_t)op.cl;
    const int t0 = op.t[0];
    const bool regpath = type == F_DIAG ||
                        (type <= F_U2 && (t0 < 5 || t0 >= 8));
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
      smem_op(tile, op, T);
      continue;
    }
    if (type == F_DIAG) {
      // j = local diagonal index; bits of targets >= K come from the tile base.
      const int m = op.m;
      uint32_t jh = 0, jmask = 0;  // uniform part of j and which j-bits are per amplitude
      const int ta = op.t[0], tb = op.t[1], tc = op.t[2];
#pragma unroll
      for (int s = 0; s < 3; ++s) {
        const int t = s == 0 ? ta : (s == 1 ? tb : tc);
        if (s < m) {
          if (t >= K)
            jh |= (uint32_t)((base >> t) & 1) << (m - 1 - s);
          else
            jmask |= 1u << (m - 1 - s);
        }
      }
      if (jmask == 0) {  // factor uniform over the tile (or over amplitudes passing cl)
        const double2 d = op.c[jh];
        if (is_one(d)) continue;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const uint32_t i = (uint32_t)r * kFThreads + tid;
          if ((i & cl) == cl) v[r] = cmul_rn(d, v[r]);
        }
      } else {
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const uint32_t i = (uint32_t)r * kFThreads + tid;
          if ((i & cl) != cl) continue;
          uint32_t j = jh;
#pragma unroll
          for (int s = 0; s < 3; ++s) {
            const int t = s == 0 ? ta : (s == 1 ? tb : tc);
            if (s < m && (jmask >> (m - 1 - s) & 1)) j |= ((i >> t) & 1u) << (m - 1 - s);
          }
          const double2 d = op.c[j];
          if (!is_one(d)) v[r] = cmul_rn(d, v[r]);
        }
      }
    } else if (type == F_X) {
      reg_op<R>(v, RX_{}, t0, cl, tid);
    } else if (type == F_Y) {
      reg_op<R>(v, RY_{}, t0, cl, tid);
    } else if (type == F_H) {
      reg_op<R>(v, RH_{op.c[0].x}, t0, cl, tid);
    } else {
      reg_op<R>(v, RU_{op.c[0], op.c[1], op.c[2], op.c[3]}, t0, cl, tid);
    }
  }

  if (in_regs) {
#pragma unroll
    for (int r = 0; r < R; ++r) tile[r * kFThreads + tid] = v[r];
  }
  // Make the generic-proxy smem writes visible to the async proxy, then one
  // thread issues the bulk store and waits for it.
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (tid == 0) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(a + base),
                 "r"(tile_a), "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

inline double2 D2(cplx z) { return make_double2(z.re, z.im); }

void encode(const Decoded& g, int K, FOp* op) {
  std::memset(op, 0, sizeof(FOp));
  const uint64_t lowmask = (1ull << K) - 1;
  op->cl = g.cmask & lowmask;
  op->ch = g.cmask & ~lowmask;
  op->m = g.m;
  for (int s = 0; s < g.m; ++s) op->t[s] = g.targets[s];
  const int d = 1 << g.m;
  switch (g.cls) {
    case GClass::DIAG:
      op->type = F_DIAG;
      for (int j = 0; j < d; ++j) op->c[j] = D2(g.M[j * d + j]);
      return;
    case GClass::PERM_X: op->type = F_X; return;
    case GClass::PERM_Y: op->type = F_Y; return;
    case GClass::PERM_SWAP: op->type = F_SWAP; return;
    default:
      break;
  }
  if (g.m == 1) {
    op->type = g.is_h ? F_H : F_U2;
    if (g.is_h) op->c[0] = D2(g.M[0]);
  } else {
    op->type = g.m == 2 ? F_U4 : F_U8;
  }
  if (!g.is_h)
    for (int i = 0; i < d * d; ++i) op->c[i] = D2(g.M[i]);
}

template <int K>
void launch_k(const LaunchCtx& ctx, const FOp* d_prog, int nops) {
  const size_t smem = size_t(16) << K;
  ensure_smem_attr((const void*)k_fused<K>, (int)smem);
  const uint64_t tiles = 1ull << (ctx.n_local - K);
  k_fused<K><<<(unsigned)tiles, kFThreads, smem, ctx.stream>>>(
      reinterpret_cast<double2*>(ctx.amps), d_prog, nops);
}

}  // namespace

bool fusable(const Decoded& g, int K, int n_local) {
  (void)n_local;
  if (g.cls == GClass::NOOP || g.cls == GClass::DIAG) return true;
  for (int s = 0; s < g.m; ++s)
    if (g.targets[s] >= K) return false;
  return true;
}

bool run_fused_circuit(const LaunchCtx& ctx, const std::vector<Decoded>& gates, size_t begin,
                       size_t end, int tile_qubits, size_t* consumed) {
  *consumed = 0;
  int K = tile_qubits < ctx.n_local ? tile_qubits : ctx.n_local;
  if (K > kMaxK) K = kMaxK;
  if (K < kMinK) return false;
  size_t i = begin;
  int nops = 0;
  while (i < end && nops < kMaxOps && fusable(gates[i], K, ctx.n_local)) {
    if (gates[i].cls != GClass::NOOP) ++nops;
    ++i;
  }
  if (nops < 2) return false;  // a single gate runs faster in its class kernel
  // Program buffer owned by the state; reuse is stream-ordered (this upload is
  // queued after the previous fused kernel).  The host vector is pageable, so
  // cudaMemcpyAsync stages it before returning and no host sync is needed.
  if (*ctx.fused_prog == nullptr)
    LFQS_CUDA_CHECK(cudaMalloc(ctx.fused_prog, sizeof(FOp) * kMaxOps));
  FOp* d_prog = static_cast<FOp*>(*ctx.fused_prog);
  std::vector<FOp> h(nops);
  int o = 0;
  for (size_t q = begin; q < i; ++q)
    if (gates[q].cls != GClass::NOOP) encode(gates[q], K, &h[o++]);
  LFQS_CUDA_CHECK(cudaMemcpyAsync(d_prog, h.data(), sizeof(FOp) * o, cudaMemcpyHostToDevice,
                                  ctx.stream));
  switch (K) {
    case 8: launch_k<8>(ctx, d_prog, o); break;
    case 9: launch_k<9>(ctx, d_prog, o); break;
    case 10: launch_k<10>(ctx, d_prog, o); break;
    case 11: launch_k<11>(ctx, d_prog, o); break;
    default: launch_k<12>(ctx, d_prog, o); break;
  }
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
  *consumed = i - begin;
  return true;
}

}  // namespace lfqs
