// fused_kernels.cu -- shared-memory staging of consecutive gates.
//
// The paper applies every gate as its own pass and exposes every intermediate
// state; the optimised kernel of each gate is one pass over S (vector
// fusion).  On B200 a pass over a 16-128 GiB state costs 5-35 ms of
// HBM time while the arithmetic of one gate costs < 0.3 ms, so a run of
// consecutive gates that only mix amplitudes inside a 2^k tile is applied in
// ONE pass: the tile is staged into shared memory with a TMA bulk copy
// (cp.async.bulk + mbarrier), every gate of the run is applied there, and the
// tile is written back with one bulk store.  A gate fuses when all its targets
// are < k (controls anywhere: high controls are a per-tile predicate), or when
// it is diagonal (any qubits: high target bits come from the tile index).
// Permutation and diagonal gates use exactly the unfused formulas, so fused ==
// unfused value-exactly for them; dense gates agree within rounding.
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
  int t[3];        // targets (DIAG: any position; others: < k)
  int pad;
  uint64_t cl;     // controls below k (per amplitude)
  uint64_t ch;     // controls at or above k (per tile)
  double2 c[64];   // matrix row-major, or the diagonal d[j] for DIAG
};

constexpr int kFThreads = 256;  // x3 CTAs per SM (64 KiB tiles) to overlap load/compute/store
constexpr int kMaxOps = 256;

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
    for (int i = 0; i < L; ++i) cfma(acc, __ldg(&c[j * L + i]), v[i]);
    w[j] = acc;
  }
#pragma unroll
  for (int j = 0; j < L; ++j) tile[idx[j]] = w[j];
}

__global__ void __launch_bounds__(kFThreads, 3) k_fused(double2* __restrict__ a,
                                                     const FOp* __restrict__ prog, int nops,
                                                     int K) {
  extern __shared__ __align__(128) double2 tile[];
  __shared__ __align__(8) uint64_t bar;
  const uint32_t T = 1u << K;
  const uint64_t base = (uint64_t)blockIdx.x << K;
  const uint32_t bytes = T * 16u;
  const uint32_t bar_a = smem_u32(&bar), tile_a = smem_u32(tile);
  if (threadIdx.x == 0) {
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

  for (int o = 0; o < nops; ++o) {
    const FOp& op = prog[o];
    const uint64_t ch = op.ch;
    if ((base & ch) != ch) continue;  // a high control is 0 on this tile (uniform)
    const uint32_t cl = (uint32_t)op.cl;
    const int type = op.type;
    if (type == F_DIAG) {
      const int m = op.m;
      for (uint32_t i = threadIdx.x; i < T; i += kFThreads) {
        if ((i & cl) != cl) continue;
        const uint64_t k = base | i;
        int j = 0;
        for (int s = 0; s < m; ++s) j = (j << 1) | (int)((k >> op.t[s]) & 1);
        const double2 d = __ldg(&op.c[j]);
        if (d.x == 1.0 && d.y == 0.0) continue;
        tile[i] = cmul_rn(d, tile[i]);
      }
    } else if (type <= F_U2) {
      const int t = op.t[0];
      for (uint32_t p = threadIdx.x; p < (T >> 1); p += kFThreads) {
        const uint32_t i0 = ins0(p, t), i1 = i0 | (1u << t);
        if ((i0 & cl) != cl) continue;
        const double2 a0 = tile[i0], a1 = tile[i1];
        double2 b0, b1;
        if (type == F_X) {
          b0 = a1;
          b1 = a0;
        } else if (type == F_Y) {
          b0 = make_double2(a1.y, -a1.x);
          b1 = make_double2(-a0.y, a0.x);
        } else if (type == F_H) {
          const double s = op.c[0].x;
          b0 = make_double2(s * (a0.x + a1.x), s * (a0.y + a1.y));
          b1 = make_double2(s * (a0.x - a1.x), s * (a0.y - a1.y));
        } else {
          b0 = make_double2(0.0, 0.0);
          b1 = b0;
          cfma(b0, __ldg(&op.c[0]), a0);
          cfma(b0, __ldg(&op.c[1]), a1);
          cfma(b1, __ldg(&op.c[2]), a0);
          cfma(b1, __ldg(&op.c[3]), a1);
        }
        tile[i0] = b0;
        tile[i1] = b1;
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
      int s0 = op.t[0], s1 = op.t[1], s2 = op.t[2];
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
    __syncthreads();
  }

  // Write back: make the generic-proxy smem writes visible to the async proxy,
  // then one thread issues the bulk store and waits for it.
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
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
  } else {
    op->type = g.m == 2 ? F_U4 : F_U8;
  }
  for (int i = 0; i < d * d; ++i) op->c[i] = D2(g.M[i]);
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
  const int K = tile_qubits < ctx.n_local ? tile_qubits : ctx.n_local;
  if (K < 5) return false;
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
  const size_t smem = (size_t(16) << K);
  ensure_smem_attr((const void*)k_fused, 16 << 13);
  const uint64_t tiles = 1ull << (ctx.n_local - K);
  k_fused<<<(unsigned)tiles, kFThreads, smem, ctx.stream>>>(reinterpret_cast<double2*>(ctx.amps),
                                                            d_prog, o, K);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
  *consumed = i - begin;
  return true;
}

}  // namespace lfqs
