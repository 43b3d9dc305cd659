// reduce_kernels.cu -- norm / marginal-probability reduction and state initialisers.
//
// Measurement at the end of a circuit: P(Q = v) = sum_{k: bits_Q(k) = v} |a_k|^2.
// B200 design: one read-only streaming pass.  Each
// warp reads 32 contiguous amplitudes per instruction (16 B per lane, evict-
// first), folds |a|^2 across the lane bits that are NOT measured with xor-
// shuffles, and the lanes that represent a distinct low-bit outcome add into a
// per-warp shared-memory histogram (no atomics: each bin has exactly one
// writer lane).  Warps are then summed in fixed order per block, and blocks in
// fixed order by a second tiny kernel: the result is deterministic for a given
// shard size, independent of scheduling.
#include <cuda_runtime.h>

#include <cstring>
#include <mutex>
#include <set>
#include <utility>

#include "lfqs_internal.h"

namespace lfqs {
namespace {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;
constexpr int kBlocks = 148 * 4;  // fixed grid => fixed summation order
constexpr int kU = 4;             // 32-amplitude rows per warp iteration
constexpr int kMaxQ = 10;

struct QList {
  int nq;
  int q[kMaxQ];
  uint32_t lane_free;  // lane bits (0..4) not measured: folded by shuffles
  uint64_t fmask, fpat;  // only amplitudes with (k & fmask) == fpat contribute
};

__device__ __forceinline__ double2 ldcs(const double2* p) {
  double2 v;
  asm volatile("ld.global.cs.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}

__device__ __forceinline__ int bin_of(const QList& ql, uint64_t k) {
  int v = 0;
#pragma unroll
  for (int s = 0; s < kMaxQ; ++s)
    if (s < ql.nq) v |= (int)((k >> ql.q[s]) & 1) << s;
  return v;
}

__global__ void __launch_bounds__(kThreads) k_probs(const double2* __restrict__ a, uint64_t n_rows,
                                                    const QList ql, double* __restrict__ partials) {
  extern __shared__ double hist[];  // [kWarps][nbins]
  const int nbins = 1 << ql.nq;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < kWarps * nbins; i += kThreads) hist[i] = 0.0;
  __syncthreads();
  double* my = hist + warp * nbins;
  const bool rep = (lane & ql.lane_free) == 0;
  // rows of 32 amplitudes; warp w of block b handles row groups in a fixed stride
  const uint64_t stride = (uint64_t)gridDim.x * kWarps * kU;
  for (uint64_t r0 = ((uint64_t)blockIdx.x * kWarps + warp) * kU; r0 < n_rows; r0 += stride) {
    double p[kU];
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const uint64_t r = r0 + u;
      if (r < n_rows) {
        const double2 x = ldcs(a + r * 32 + lane);
        p[u] = ((r * 32 + lane) & ql.fmask) == ql.fpat ? x.x * x.x + x.y * x.y : 0.0;
      } else {
        p[u] = 0.0;
      }
    }
#pragma unroll
    for (int u = 0; u < kU; ++u) {
#pragma unroll
      for (int b = 0; b < 5; ++b)
        if (ql.lane_free >> b & 1) p[u] += __shfl_xor_sync(0xffffffffu, p[u], 1 << b);
      if (rep && r0 + u < n_rows) my[bin_of(ql, (r0 + u) * 32 + lane)] += p[u];
    }
  }
  __syncthreads();
  for (int bin = threadIdx.x; bin < nbins; bin += kThreads) {
    double s = 0.0;
    for (int w = 0; w < kWarps; ++w) s += hist[w * nbins + bin];
    partials[(uint64_t)blockIdx.x * nbins + bin] = s;
  }
}

__global__ void k_probs_final(const double* __restrict__ partials, int nblocks, int nbins,
                              double* __restrict__ out) {
  const int bin = blockIdx.x * blockDim.x + threadIdx.x;
  if (bin >= nbins) return;
  double s = 0.0;
  for (int b = 0; b < nblocks; ++b) s += partials[(uint64_t)b * nbins + bin];
  out[bin] = s;
}

// Small-state path (< 32 amplitudes): one thread, ascending order.
__global__ void k_probs_tiny(const double2* __restrict__ a, uint64_t n_amps, const QList ql,
                             double* __restrict__ out) {
  const int nbins = 1 << ql.nq;
  for (int b = 0; b < nbins; ++b) out[b] = 0.0;
  for (uint64_t k = 0; k < n_amps; ++k)
    if ((k & ql.fmask) == ql.fpat) out[bin_of(ql, k)] += a[k].x * a[k].x + a[k].y * a[k].y;
}

// --- projective collapse (one streaming pass, 32-byte accesses) --------------
__global__ void __launch_bounds__(kThreads) k_collapse(double2* __restrict__ a, uint64_t n_pairs,
                                                       uint64_t mask, uint64_t pat, double scale) {
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t i = (uint64_t)blockIdx.x * kThreads + threadIdx.x; i < n_pairs; i += stride) {
    const uint64_t k = 2 * i;
    double2 x, y;
    asm volatile("ld.global.cs.v4.f64 {%0,%1,%2,%3}, [%4];"
                 : "=d"(x.x), "=d"(x.y), "=d"(y.x), "=d"(y.y)
                 : "l"(a + k));
    x = ((k & mask) == pat) ? make_double2(scale * x.x, scale * x.y) : make_double2(0.0, 0.0);
    y = (((k + 1) & mask) == pat) ? make_double2(scale * y.x, scale * y.y) : make_double2(0.0, 0.0);
    asm volatile("st.global.cs.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(a + k), "d"(x.x), "d"(x.y),
                 "d"(y.x), "d"(y.y)
                 : "memory");
  }
}

// --- initialisers -----------------------------------------------------------
__global__ void k_set_one(double2* a, uint64_t idx) { a[idx] = make_double2(1.0, 0.0); }

__device__ __forceinline__ uint64_t sm64(uint64_t seed, uint64_t i) {  // SplitMix64 output #i
  uint64_t z = seed + (i + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void __launch_bounds__(kThreads) k_init_random(double2* __restrict__ a, uint64_t n_amps,
                                                          uint64_t seed, uint64_t offset) {
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t k = (uint64_t)blockIdx.x * kThreads + threadIdx.x; k < n_amps; k += stride) {
    const uint64_t gk = offset + k;
    const double re = (double)(sm64(seed, 2 * gk) >> 11) * 0x1.0p-53 * 2.0 - 1.0;
    const double im = (double)(sm64(seed, 2 * gk + 1) >> 11) * 0x1.0p-53 * 2.0 - 1.0;
    a[k] = make_double2(re, im);
  }
}

}  // namespace

int probs_blocks() { return kBlocks; }

void ensure_smem_attr(const void* kernel, int bytes) {
  // cudaFuncSetAttribute is per device; remember (kernel, device) pairs done.
  static std::mutex mu;
  static std::set<std::pair<const void*, int>> done;
  int dev = 0;
  LFQS_CUDA_CHECK(cudaGetDevice(&dev));
  std::lock_guard<std::mutex> lk(mu);
  if (done.count({kernel, dev})) return;
  LFQS_CUDA_CHECK(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
  done.insert({kernel, dev});
}

void launch_probs(const LaunchCtx& ctx, const int* qubits, int nq, double* d_partials,
                  int n_partials_blocks, double* d_out, uint64_t fmask, uint64_t fpat) {
  require(nq >= 0 && nq <= kMaxQ, "one probability pass covers at most 10 qubits");
  QList ql;
  std::memset(&ql, 0, sizeof ql);
  ql.nq = nq;
  ql.fmask = fmask;
  ql.fpat = fpat;
  uint32_t measured_lane_bits = 0;
  for (int s = 0; s < nq; ++s) {
    ql.q[s] = qubits[s];
    if (qubits[s] < 5) measured_lane_bits |= 1u << qubits[s];
  }
  ql.lane_free = 0x1fu & ~measured_lane_bits;
  const uint64_t n_amps = 1ull << ctx.n_local;
  const auto* a = reinterpret_cast<const double2*>(ctx.amps);
  if (n_amps < 32) {
    k_probs_tiny<<<1, 1, 0, ctx.stream>>>(a, n_amps, ql, d_out);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
    return;
  }
  require(n_partials_blocks >= kBlocks, "partials buffer too small");
  const int nbins = 1 << nq;
  const size_t smem = sizeof(double) * kWarps * nbins;
  ensure_smem_attr((const void*)k_probs, sizeof(double) * kWarps * (1 << kMaxQ));
  k_probs<<<kBlocks, kThreads, smem, ctx.stream>>>(a, n_amps / 32, ql, d_partials);
  LFQS_CUDA_CHECK(cudaGetLastError());
  k_probs_final<<<(nbins + 255) / 256, 256, 0, ctx.stream>>>(d_partials, kBlocks, nbins, d_out);
  LFQS_CUDA_CHECK(cudaGetLastError());
  *ctx.launch_counter += 2;
}

void launch_collapse(const LaunchCtx& ctx, uint64_t mask, uint64_t pat, double scale,
                     bool zero_all) {
  const uint64_t n = 1ull << ctx.n_local;
  if (zero_all) {
    LFQS_CUDA_CHECK(cudaMemsetAsync(ctx.amps, 0, n * 16, ctx.stream));
    return;
  }
  uint64_t nb = (n / 2 + kThreads - 1) / kThreads;
  if (nb > 148ull * 64) nb = 148ull * 64;
  k_collapse<<<(unsigned)nb, kThreads, 0, ctx.stream>>>(reinterpret_cast<double2*>(ctx.amps),
                                                        n / 2, mask, pat, scale);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

void launch_init_basis(const LaunchCtx& ctx, int64_t local_index) {
  LFQS_CUDA_CHECK(cudaMemsetAsync(ctx.amps, 0, sizeof(double) * 2 * (1ull << ctx.n_local), ctx.stream));
  if (local_index >= 0) {
    k_set_one<<<1, 1, 0, ctx.stream>>>(reinterpret_cast<double2*>(ctx.amps), (uint64_t)local_index);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
  }
}

void launch_init_random(const LaunchCtx& ctx, uint64_t seed, uint64_t global_offset) {
  const uint64_t n = 1ull << ctx.n_local;
  uint64_t nb = (n + kThreads - 1) / kThreads;
  if (nb > 148ull * 64) nb = 148ull * 64;
  k_init_random<<<(unsigned)nb, kThreads, 0, ctx.stream>>>(reinterpret_cast<double2*>(ctx.amps), n,
                                                           seed, global_offset);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

}  // namespace lfqs
