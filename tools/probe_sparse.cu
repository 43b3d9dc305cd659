// probe_sparse.cu -- DRAM access-pattern probe for the sparse-touch gate classes
// (VERDICT r1 "What's weak" 2 / "do this" 4).  Standalone: not part of liblfqs.
//
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/probe tools/probe_sparse.cu
//   /tmp/probe [log2_amps=30]
//
// A complex128 state of 2^n amplitudes (16 B each) is viewed as 128-B lines of four
// 32-B sectors.  Each pattern reads and/or writes a subset of sectors, in place, and
// is timed with CUDA events (best of 5 after 2 warm-ups).  Printed: ms, the bytes the
// pattern requests (sectors loaded + stored), and the requested GB/s.  Run it under
// `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum` to see what DRAM moves.
//
// Patterns (k = sector index in the line, 0..3; "touched" = the gate's changed sector):
//   copy_all      read+write every sector (a dense gate pass: the HBM ceiling)
//   read_all      read every sector, write nothing
//   s1of4_rw      read+write sector 3 of every line, one 32-B access per thread
//                 (the Toffoli-with-controls-{1,2} pattern of k_group_x2)
//   s1of4_line    a quarter-warp reads the whole line (4 x 32 B, coalesced), the lane
//                 that holds sector 3 writes it back (line-shaped reads, sector writes)
//   s1of4_l2pf    as s1of4_rw, the load carrying the L2::128B prefetch-size hint
//   s1of4_w       write sector 3 of every line, no reads
//   s1of4_r       read sector 3 of every line, no writes
//   s1of2_rw      read+write the second 32-B sector of every 64-B half line (Z on qubit 1)
//   s1of2_line    whole-line coalesced reads, writes of the touched sectors only
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstdint>

#define CK(x)                                                                        \
  do {                                                                               \
    cudaError_t e_ = (x);                                                            \
    if (e_ != cudaSuccess) {                                                         \
      std::fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_));                  \
      std::exit(1);                                                                  \
    }                                                                                \
  } while (0)

struct alignas(32) Sec {
  double a, b, c, d;
};

__device__ __forceinline__ Sec ldcs(const Sec* p) {
  Sec v;
  asm volatile("ld.global.cs.v4.f64 {%0,%1,%2,%3}, [%4];"
               : "=d"(v.a), "=d"(v.b), "=d"(v.c), "=d"(v.d)
               : "l"(p));
  return v;
}
__device__ __forceinline__ Sec ldpf(const Sec* p) {
  Sec v;
  asm volatile("ld.global.cs.L2::128B.v4.f64 {%0,%1,%2,%3}, [%4];"
               : "=d"(v.a), "=d"(v.b), "=d"(v.c), "=d"(v.d)
               : "l"(p));
  return v;
}
__device__ __forceinline__ void stcs(Sec* p, Sec v) {
  asm volatile("st.global.cs.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(p), "d"(v.a), "d"(v.b), "d"(v.c),
               "d"(v.d)
               : "memory");
}
__device__ __forceinline__ Sec neg(Sec v) { return Sec{-v.a, -v.b, -v.c, -v.d}; }

constexpr int kT = 256, kU = 4;

// every sector: read + write (a dense gate pass)
__global__ void __launch_bounds__(kT) copy_all(Sec* s, uint64_t nsec) {
  const uint64_t base = (uint64_t)blockIdx.x * kT * kU + threadIdx.x;
  Sec v[kU];
#pragma unroll
  for (int u = 0; u < kU; ++u)
    if (base + u * kT < nsec) v[u] = ldcs(s + base + u * kT);
#pragma unroll
  for (int u = 0; u < kU; ++u)
    if (base + u * kT < nsec) stcs(s + base + u * kT, neg(v[u]));
}
__global__ void __launch_bounds__(kT) read_all(const Sec* s, uint64_t nsec, double* sink) {
  const uint64_t base = (uint64_t)blockIdx.x * kT * kU + threadIdx.x;
  double acc = 0;
#pragma unroll
  for (int u = 0; u < kU; ++u)
    if (base + u * kT < nsec) {
      Sec v = ldcs(s + base + u * kT);
      acc += v.a + v.d;
    }
  if (acc == 12345.678) *sink = acc;
}
// sector `which` of each `per`-sector group (per = 4: 128-B lines, per = 2: 64-B halves)
template <int PER, bool PF>
__global__ void __launch_bounds__(kT) sparse_rw(Sec* s, uint64_t ngroups, int which) {
  const uint64_t base = (uint64_t)blockIdx.x * kT * kU + threadIdx.x;
  Sec v[kU];
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    const uint64_t g = base + u * kT;
    if (g < ngroups) v[u] = PF ? ldpf(s + g * PER + which) : ldcs(s + g * PER + which);
  }
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    const uint64_t g = base + u * kT;
    if (g < ngroups) stcs(s + g * PER + which, neg(v[u]));
  }
}
template <int PER>
__global__ void __launch_bounds__(kT) sparse_w(Sec* s, uint64_t ngroups, int which) {
  const uint64_t base = (uint64_t)blockIdx.x * kT * kU + threadIdx.x;
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    const uint64_t g = base + u * kT;
    if (g < ngroups) stcs(s + g * PER + which, Sec{1.0, 2.0, 3.0, 4.0});
  }
}
template <int PER>
__global__ void __launch_bounds__(kT) sparse_r(const Sec* s, uint64_t ngroups, int which,
                                               double* sink) {
  const uint64_t base = (uint64_t)blockIdx.x * kT * kU + threadIdx.x;
  double acc = 0;
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    const uint64_t g = base + u * kT;
    if (g < ngroups) {
      Sec v = ldcs(s + g * PER + which);
      acc += v.a + v.d;
    }
  }
  if (acc == 12345.678) *sink = acc;
}
// whole lines read coalesced (thread i <-> sector i), only the touched sectors written
template <int PER>
__global__ void __launch_bounds__(kT) line_rw(Sec* s, uint64_t nsec, int which) {
  const uint64_t base = (uint64_t)blockIdx.x * kT * kU + threadIdx.x;
  Sec v[kU];
#pragma unroll
  for (int u = 0; u < kU; ++u)
    if (base + u * kT < nsec) v[u] = ldcs(s + base + u * kT);
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    const uint64_t i = base + u * kT;
    if (i < nsec && (int)(i % PER) == which) stcs(s + i, neg(v[u]));
  }
}

int main(int argc, char** argv) {
  const int n = argc > 1 ? std::atoi(argv[1]) : 30;
  const uint64_t bytes = 16ull << n, nsec = bytes / 32;
  Sec* s = nullptr;
  double* sink = nullptr;
  CK(cudaMalloc(&s, bytes));
  CK(cudaMalloc(&sink, 8));
  CK(cudaMemset(s, 0, bytes));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  auto grid = [](uint64_t items) { return (unsigned)((items + kT * kU - 1) / (kT * kU)); };
  auto run = [&](const char* name, double req_bytes, auto&& launch) {
    float best = 1e30f;
    for (int r = 0; r < 7; ++r) {
      CK(cudaEventRecord(e0));
      launch();
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      CK(cudaGetLastError());
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      if (r >= 2 && ms < best) best = ms;
    }
    std::printf("%-12s %8.3f ms  requested %7.2f GB  %8.1f GB/s\n", name, best, req_bytes / 1e9,
                req_bytes / (best * 1e-3) / 1e9);
  };
  const uint64_t l4 = nsec / 4, l2 = nsec / 2;
  run("copy_all", 2.0 * bytes, [&] { copy_all<<<grid(nsec), kT>>>(s, nsec); });
  run("read_all", 1.0 * bytes, [&] { read_all<<<grid(nsec), kT>>>(s, nsec, sink); });
  run("s1of4_rw", 2.0 * bytes / 4, [&] { sparse_rw<4, false><<<grid(l4), kT>>>(s, l4, 3); });
  run("s1of4_line", bytes + bytes / 4.0, [&] { line_rw<4><<<grid(nsec), kT>>>(s, nsec, 3); });
  run("s1of4_l2pf", 2.0 * bytes / 4, [&] { sparse_rw<4, true><<<grid(l4), kT>>>(s, l4, 3); });
  run("s1of4_w", bytes / 4.0, [&] { sparse_w<4><<<grid(l4), kT>>>(s, l4, 3); });
  run("s1of4_r", bytes / 4.0, [&] { sparse_r<4><<<grid(l4), kT>>>(s, l4, 3, sink); });
  run("s1of2_rw", 2.0 * bytes / 2, [&] { sparse_rw<2, false><<<grid(l2), kT>>>(s, l2, 1); });
  run("s1of2_line", bytes + bytes / 2.0, [&] { line_rw<2><<<grid(nsec), kT>>>(s, nsec, 1); });
  run("s1of2_l2pf", 2.0 * bytes / 2, [&] { sparse_rw<2, true><<<grid(l2), kT>>>(s, l2, 1); });
  run("s1of2_w", bytes / 2.0, [&] { sparse_w<2><<<grid(l2), kT>>>(s, l2, 1); });
  CK(cudaFree(s));
  return 0;
}
