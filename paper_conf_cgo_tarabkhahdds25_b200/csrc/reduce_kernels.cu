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

#include <algorithm>
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
constexpr int kMaxLo = 10;        // qubits binned in the shared-memory histogram
constexpr int kMaxQ = 20;         // qubits per measurement (lfqs_measure_probs)

// Two-level binning (one read pass for up to 20 measured qubits): the measured qubits
// at the kMaxLo lowest positions ("lo") are histogrammed per warp in shared memory as
// before; the others ("hi", all at positions >= 10, so never a lane bit) select a
// subspace: work unit u = h * slices + s reads slice s of the amplitudes whose hi bits
// equal h -- their indices are the subspace index with h's bits inserted at the hi
// positions -- and writes its lo-histogram to partials[u].  A final kernel sums the
// slices of each (h, lo) bin in fixed order, so the result is deterministic.
struct QList {
  int nq;                // lo qubits (<= kMaxLo)
  int q[kMaxLo];         // their positions; bin bit u = bit q[u]
  uint32_t lane_free;    // lane bits (0..4) not measured: folded by shuffles
  int nh;                // hi qubits (<= kMaxQ - kMaxLo), ascending positions
  int hpos[kMaxQ - kMaxLo];
  uint64_t slices;       // slices per hi pattern
  uint64_t rows;         // 32-amplitude rows in one hi subspace
};

__device__ __forceinline__ int bin_of(const QList& ql, uint64_t k) {
  int v = 0;
#pragma unroll
  for (int s = 0; s < kMaxLo; ++s)
    if (s < ql.nq) v |= (int)((k >> ql.q[s]) & 1) << s;
  return v;
}

// subspace index j -> amplitude index: insert the bits of h at the hi positions
__device__ __forceinline__ uint64_t insert_hi(const QList& ql, uint64_t j, uint64_t h) {
#pragma unroll
  for (int u = 0; u < kMaxQ - kMaxLo; ++u)
    if (u < ql.nh) {
      const int p = ql.hpos[u];
      j = ((j >> p) << (p + 1)) | (j & ((1ull << p) - 1)) | (((h >> u) & 1ull) << p);
    }
  return j;
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
__global__ void __launch_bounds__(kThreads) k_probs(const A a, const QList ql, uint64_t units,
                                                    double* __restrict__ partials) {
  extern __shared__ double hist[];  // [kWarps][nbins]
  const int nbins = 1 << ql.nq;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < kWarps * nbins; i += kThreads) hist[i] = 0.0;
  __syncthreads();
  double* my = hist + warp * nbins;
  const bool rep = (lane & ql.lane_free) == 0;
  const uint64_t per = (ql.rows + ql.slices - 1) / ql.slices;
  for (uint64_t unit = blockIdx.x; unit < units; unit += gridDim.x) {
    const uint64_t h = unit / ql.slices, sl = unit % ql.slices;
    const uint64_t rb = sl * per, re = min(ql.rows, rb + per);
    // rows of 32 amplitudes; warp w handles row groups in a fixed stride
    for (uint64_t r0 = rb + (uint64_t)warp * kU; r0 < re; r0 += (uint64_t)kWarps * kU) {
      double p[kU];
      uint64_t k[kU];
#pragma unroll
      for (int u = 0; u < kU; ++u) {
        k[u] = insert_hi(ql, (r0 + u) * 32, h) + lane;
        p[u] = (r0 + u < re) ? norm2<S>(a.get(k[u])) : 0.0;
      }
#pragma unroll
      for (int u = 0; u < kU; ++u) {
#pragma unroll
        for (int b = 0; b < 5; ++b)
          if (ql.lane_free >> b & 1) p[u] += __shfl_xor_sync(0xffffffffu, p[u], 1 << b);
        if (rep && r0 + u < re) my[bin_of(ql, k[u])] += p[u];
      }
    }
    __syncthreads();
    for (int bin = threadIdx.x; bin < nbins; bin += kThreads) {
      double s = 0.0;
      for (int w = 0; w < kWarps; ++w) {
        s += hist[w * nbins + bin];
        hist[w * nbins + bin] = 0.0;
      }
      partials[unit * nbins + bin] = s;
    }
    __syncthreads();
  }
}

// out[v], v < 2^(nlo + nh): bit u of v's lo part = lo qubit u, of its hi part = hi qubit u
// (the caller's order is restored on the host side of launch_probs through lo_of / hi_of).
struct FinalMap {
  int nq;                 // caller's qubit count
  int lo_of[kMaxQ];       // caller index s -> lo bit (or -1)
  int hi_of[kMaxQ];       // caller index s -> hi bit (or -1)
};

__global__ void k_probs_final(const double* __restrict__ partials, uint64_t slices, int nlo,
                              const FinalMap fm, double* __restrict__ out) {
  const uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v >= (1ull << fm.nq)) return;
  uint64_t lo = 0, h = 0;
  for (int s = 0; s < fm.nq; ++s) {
    const uint64_t b = (v >> s) & 1;
    if (fm.lo_of[s] >= 0) lo |= b << fm.lo_of[s];
    else h |= b << fm.hi_of[s];
  }
  double acc = 0.0;
  const uint64_t base = h * slices;
  for (uint64_t s = 0; s < slices; ++s) acc += partials[((base + s) << nlo) + lo];
  out[v] = acc;
}

// Small-state path (< 32 amplitudes): one thread, ascending order, the caller's bins.
struct CallerQ {
  int nq;
  int q[kMaxQ];
};

template <class S, class A>
__global__ void k_probs_tiny(const A a, uint64_t n_amps, const CallerQ cq,
                             double* __restrict__ out) {
  const int nbins = 1 << cq.nq;
  for (int b = 0; b < nbins; ++b) out[b] = 0.0;
  for (uint64_t k = 0; k < n_amps; ++k) {
    int v = 0;
    for (int s = 0; s < cq.nq; ++s) v |= (int)((k >> cq.q[s]) & 1) << s;
    out[v] += norm2<S>(a.get_plain(k));
  }
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

// Splits the caller's qubits into lo (the kMaxLo lowest positions) and hi (ascending).
struct ProbsPlan {
  QList ql;
  FinalMap fm;
  CallerQ cq;
  uint64_t units;
};

ProbsPlan make_probs_plan(int n_local, const int* qubits, int nq) {
  ProbsPlan pp;
  std::memset(&pp, 0, sizeof pp);
  pp.fm.nq = nq;
  pp.cq.nq = nq;
  int order[kMaxQ];
  for (int s = 0; s < nq; ++s) {
    order[s] = s;
    pp.cq.q[s] = qubits[s];
  }
  std::sort(order, order + nq, [&](int x, int y) { return qubits[x] < qubits[y]; });
  const int nlo = nq < kMaxLo ? nq : kMaxLo;
  uint32_t measured_lane_bits = 0;
  for (int u = 0; u < nq; ++u) {
    const int s = order[u];
    pp.fm.lo_of[s] = pp.fm.hi_of[s] = -1;
    if (u < nlo) {
      pp.ql.q[u] = qubits[s];
      pp.fm.lo_of[s] = u;
      if (qubits[s] < 5) measured_lane_bits |= 1u << qubits[s];
    } else {
      pp.ql.hpos[u - nlo] = qubits[s];  // ascending: insert_hi's order
      pp.fm.hi_of[s] = u - nlo;
    }
  }
  pp.ql.nq = nlo;
  pp.ql.nh = nq - nlo;
  pp.ql.lane_free = 0x1fu & ~measured_lane_bits;
  pp.ql.rows = n_local >= 5 ? (1ull << (n_local - pp.ql.nh)) / 32 : 0;
  // enough units for every block to see several (balance), each slice >= kU rows per warp
  const uint64_t hs = 1ull << pp.ql.nh;
  uint64_t sl = pp.ql.nh == 0 ? (uint64_t)kBlocks : std::max<uint64_t>(1, 4ull * kBlocks / hs);
  sl = std::min<uint64_t>(sl, std::max<uint64_t>(1, pp.ql.rows / (kWarps * kU)));
  pp.ql.slices = sl;
  pp.units = hs * sl;
  return pp;
}

template <class S, class A>
void probs_t(const LaunchCtx& ctx, const A a, const ProbsPlan& pp, double* d_partials,
             double* d_out) {
  const uint64_t n_amps = 1ull << ctx.n_local;
  if (n_amps < 32) {
    k_probs_tiny<S, A><<<1, 1, 0, ctx.stream>>>(a, n_amps, pp.cq, d_out);
    LFQS_CUDA_CHECK(cudaGetLastError());
    ++*ctx.launch_counter;
    return;
  }
  const int nbins = 1 << pp.ql.nq;
  const size_t smem = sizeof(double) * kWarps * nbins;
  ensure_smem_attr((const void*)k_probs<S, A>, sizeof(double) * kWarps * (1 << kMaxLo));
  const unsigned grid = (unsigned)std::min<uint64_t>(pp.units, kBlocks);
  k_probs<S, A><<<grid, kThreads, smem, ctx.stream>>>(a, pp.ql, pp.units, d_partials);
  LFQS_CUDA_CHECK(cudaGetLastError());
  const uint64_t nout = 1ull << pp.fm.nq;
  k_probs_final<<<(unsigned)((nout + 255) / 256), 256, 0, ctx.stream>>>(
      d_partials, pp.ql.slices, pp.ql.nq, pp.fm, d_out);
  LFQS_CUDA_CHECK(cudaGetLastError());
  *ctx.launch_counter += 2;
}

inline size_t amp_bytes(const LaunchCtx& ctx) { return ctx.c64 ? 8 : 16; }

}  // namespace

size_t probs_partials_doubles(int n_local, const int* qubits, int nq) {
  const ProbsPlan pp = make_probs_plan(n_local, qubits, nq);
  return std::max<size_t>(1, pp.units << pp.ql.nq);
}

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
                  size_t partials_doubles, double* d_out) {
  require(nq >= 0 && nq <= kMaxQ, "one probability pass covers at most 20 qubits");
  const ProbsPlan pp = make_probs_plan(ctx.n_local, qubits, nq);
  require(partials_doubles >= (pp.units << pp.ql.nq), "internal: partials buffer too small");
  if (ctx.c64 && ctx.soa)
    probs_t<float>(ctx, soa_acc<float>(ctx), pp, d_partials, d_out);
  else if (ctx.c64)
    probs_t<float>(ctx, aos<float>(ctx), pp, d_partials, d_out);
  else if (ctx.soa)
    probs_t<double>(ctx, soa_acc<double>(ctx), pp, d_partials, d_out);
  else
    probs_t<double>(ctx, aos<double>(ctx), pp, d_partials, d_out);
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
