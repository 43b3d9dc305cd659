// reduce_kernels.cu -- norm / marginal-probability reduction, collapse and state initialisers.
//
// Measurement at the end of a circuit: P(Q = v) = sum_{k: bits_Q(k) = v} |a_k|^2.
// B200 design: one read-only streaming pass.  Each
// warp reads 32 contiguous amplitudes per instruction (evict-first), folds
// |a|^2 across the lane bits that are NOT measured with xor-shuffles, and the
// lanes that represent a distinct low-bit outcome add into a per-warp shared-
// memory histogram (no atomics: each bin has exactly one writer lane).  Warps
// are then summed in fixed order per block, and blocks in fixed order by a
// second tiny kernel: the result is deterministic for a given shard size.
// Probabilities are accumulated in double for both amplitude precisions.
#include <cuda_runtime.h>

#include <cstring>
#include <mutex>
#include <set>
#include <utility>

#include "cx.cuh"
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
  uint32_t lane_free;    // lane bits (0..4) not measured: folded by shuffles
  uint64_t fmask, fpat;  // only amplitudes with (k & fmask) == fpat contribute
};

__device__ __forceinline__ int bin_of(const QList& ql, uint64_t k) {
  int v = 0;
#pragma unroll
  for (int s = 0; s < kMaxQ; ++s)
    if (s < ql.nq) v |= (int)((k >> ql.q[s]) & 1) << s;
  return v;
}

// Amplitude accessors: interleaved pairs (AOS) or two planes (SOA, LFQS_STATE_SOA).
// The reductions visit amplitudes in the same order either way, so probabilities
// are bit-identical across layouts.
template <class S>
struct Aos {
  cx<S>* a;
  __device__ __forceinline__ cx<S> get(uint64_t k) const { return ld1(a + k); }
  __device__ __forceinline__ cx<S> get_plain(uint64_t k) const { return a[k]; }
  __device__ __forceinline__ void put(uint64_t k, cx<S> v) const { a[k] = v; }
  __device__ __forceinline__ void get2(uint64_t k, cx<S>& x, cx<S>& y) const { ld2(a + k, x, y); }
  __device__ __forceinline__ void put2(uint64_t k, cx<S> x, cx<S> y) const { st2(a + k, x, y); }
};
template <class S>
struct Soa {
  S* re;
  S* im;
  __device__ __forceinline__ cx<S> get(uint64_t k) const { return mk<S>(__ldcs(re + k), __ldcs(im + k)); }
  __device__ __forceinline__ cx<S> get_plain(uint64_t k) const { return mk<S>(re[k], im[k]); }
  __device__ __forceinline__ void put(uint64_t k, cx<S> v) const {
    re[k] = v.x;
    im[k] = v.y;
  }
  __device__ __forceinline__ void get2(uint64_t k, cx<S>& x, cx<S>& y) const {
    x = get(k);
    y = get(k + 1);
  }
  __device__ __forceinline__ void put2(uint64_t k, cx<S> x, cx<S> y) const {
    put(k, x);
    put(k + 1, y);
  }
};

template <class S>
__device__ __forceinline__ double norm2(cx<S> x) {
  const double re = (double)x.x, im = (double)x.y;
  return re * re + im * im;
}

template <class S, class A>
__global__ void __launch_bounds__(kThreads) k_probs(const A a, uint64_t n_rows,
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
        const cx<S> x = a.get(r * 32 + lane);
        p[u] = ((r * 32 + lane) & ql.fmask) == ql.fpat ? norm2<S>(x) : 0.0;
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
template <class S, class A>
__global__ void k_probs_tiny(const A a, uint64_t n_amps, const QList ql,
                             double* __restrict__ out) {
  const int nbins = 1 << ql.nq;
  for (int b = 0; b < nbins; ++b) out[b] = 0.0;
  for (uint64_t k = 0; k < n_amps; ++k)
    if ((k & ql.fmask) == ql.fpat) out[bin_of(ql, k)] += norm2<S>(a.get_plain(k));
}

// --- projective collapse (one streaming pass, two-amplitude accesses) --------
template <class S, class A>
__global__ void __launch_bounds__(kThreads) k_collapse(const A a, uint64_t n_pairs,
                                                       uint64_t mask, uint64_t pat, S scale) {
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t i = (uint64_t)blockIdx.x * kThreads + threadIdx.x; i < n_pairs; i += stride) {
    const uint64_t k = 2 * i;
    cx<S> x, y;
    a.get2(k, x, y);
    x = ((k & mask) == pat) ? mk<S>(scale * x.x, scale * x.y) : mk<S>(0, 0);
    y = (((k + 1) & mask) == pat) ? mk<S>(scale * y.x, scale * y.y) : mk<S>(0, 0);
    a.put2(k, x, y);
  }
}

// --- initialisers -----------------------------------------------------------
template <class S, class A>
__global__ void k_set_one(const A a, uint64_t idx) {
  a.put(idx, mk<S>(1, 0));
}

__device__ __forceinline__ uint64_t sm64(uint64_t seed, uint64_t i) {  // SplitMix64 output #i
  uint64_t z = seed + (i + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

template <class S, class A>
__global__ void __launch_bounds__(kThreads) k_init_random(const A a, uint64_t n_amps,
                                                          uint64_t seed, uint64_t offset) {
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t k = (uint64_t)blockIdx.x * kThreads + threadIdx.x; k < n_amps; k += stride) {
    const uint64_t gk = offset + k;
    const double re = (double)(sm64(seed, 2 * gk) >> 11) * 0x1.0p-53 * 2.0 - 1.0;
    const double im = (double)(sm64(seed, 2 * gk + 1) >> 11) * 0x1.0p-53 * 2.0 - 1.0;
    a.put(k, mk<S>((S)re, (S)im));
  }
}

template <class S>
Aos<S> aos(const LaunchCtx& ctx) {
  return Aos<S>{reinterpret_cast<cx<S>*>(ctx.amps)};
}
template <class S>
Soa<S> soa_acc(const LaunchCtx& ctx) {
  S* re = reinterpret_cast<S*>(ctx.amps);
  return Soa<S>{re, re + (1ull << ctx.n_local)};
}

template <class S, class A>
void probs_t(const LaunchCtx& ctx, const A a, const QList& ql, double* d_partials, double* d_out) {
  const uint64_t n_amps = 1ull << ctx.n_local;
  if (n_amps < 32) {
    k_probs_tiny<S, A><<<1, 1, 0, ctx.stream>>>(a, n_amps, ql, d_out);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
    return;
  }
  const int nbins = 1 << ql.nq;
  const size_t smem = sizeof(double) * kWarps * nbins;
  ensure_smem_attr((const void*)k_probs<S, A>, sizeof(double) * kWarps * (1 << kMaxQ));
  k_probs<S, A><<<kBlocks, kThreads, smem, ctx.stream>>>(a, n_amps / 32, ql, d_partials);
  LFQS_CUDA_CHECK(cudaGetLastError());
  k_probs_final<<<(nbins + 255) / 256, 256, 0, ctx.stream>>>(d_partials, kBlocks, nbins, d_out);
  LFQS_CUDA_CHECK(cudaGetLastError());
  *ctx.launch_counter += 2;
}

inline size_t amp_bytes(const LaunchCtx& ctx) { return ctx.c64 ? 8 : 16; }

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
  require(n_partials_blocks >= kBlocks, "partials buffer too small");
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
  if (ctx.c64 && ctx.soa)
    probs_t<float>(ctx, soa_acc<float>(ctx), ql, d_partials, d_out);
  else if (ctx.c64)
    probs_t<float>(ctx, aos<float>(ctx), ql, d_partials, d_out);
  else if (ctx.soa)
    probs_t<double>(ctx, soa_acc<double>(ctx), ql, d_partials, d_out);
  else
    probs_t<double>(ctx, aos<double>(ctx), ql, d_partials, d_out);
}

void launch_collapse(const LaunchCtx& ctx, uint64_t mask, uint64_t pat, double scale,
                     bool zero_all) {
  const uint64_t n = 1ull << ctx.n_local;
  if (zero_all) {
    LFQS_CUDA_CHECK(cudaMemsetAsync(ctx.amps, 0, n * amp_bytes(ctx), ctx.stream));
    return;
  }
  uint64_t nb = (n / 2 + kThreads - 1) / kThreads;
  if (nb > 148ull * 64) nb = 148ull * 64;
  if (ctx.c64 && ctx.soa)
    k_collapse<float><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(soa_acc<float>(ctx), n / 2, mask,
                                                                  pat, (float)scale);
  else if (ctx.c64)
    k_collapse<float><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(aos<float>(ctx), n / 2, mask, pat,
                                                                  (float)scale);
  else if (ctx.soa)
    k_collapse<double><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(soa_acc<double>(ctx), n / 2, mask,
                                                                   pat, scale);
  else
    k_collapse<double><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(aos<double>(ctx), n / 2, mask,
                                                                   pat, scale);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

void launch_init_basis(const LaunchCtx& ctx, int64_t local_index) {
  LFQS_CUDA_CHECK(
      cudaMemsetAsync(ctx.amps, 0, amp_bytes(ctx) * (1ull << ctx.n_local), ctx.stream));
  if (local_index >= 0) {
    const uint64_t li = (uint64_t)local_index;
    if (ctx.c64 && ctx.soa)
      k_set_one<float><<<1, 1, 0, ctx.stream>>>(soa_acc<float>(ctx), li);
    else if (ctx.c64)
      k_set_one<float><<<1, 1, 0, ctx.stream>>>(aos<float>(ctx), li);
    else if (ctx.soa)
      k_set_one<double><<<1, 1, 0, ctx.stream>>>(soa_acc<double>(ctx), li);
    else
      k_set_one<double><<<1, 1, 0, ctx.stream>>>(aos<double>(ctx), li);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
  }
}

void launch_init_random(const LaunchCtx& ctx, uint64_t seed, uint64_t global_offset) {
  const uint64_t n = 1ull << ctx.n_local;
  uint64_t nb = (n + kThreads - 1) / kThreads;
  if (nb > 148ull * 64) nb = 148ull * 64;
  if (ctx.c64 && ctx.soa)
    k_init_random<float><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(soa_acc<float>(ctx), n, seed,
                                                                     global_offset);
  else if (ctx.c64)
    k_init_random<float><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(aos<float>(ctx), n, seed,
                                                                     global_offset);
  else if (ctx.soa)
    k_init_random<double><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(soa_acc<double>(ctx), n, seed,
                                                                      global_offset);
  else
    k_init_random<double><<<(unsigned)nb, kThreads, 0, ctx.stream>>>(aos<double>(ctx), n, seed,
                                                                      global_offset);
  LFQS_CUDA_CHECK(cudaGetLastError());
  ++*ctx.launch_counter;
}

}  // namespace lfqs
