// probe_fp64.cu -- FP64 FMA throughput of one B200 (the ALU roofline of the FP64-bound
// compiled passes, profiles/r02_heavy_passes.md).  Standalone: not part of liblfqs.
//
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/probe_fp64 tools/probe_fp64.cu
//   /tmp/probe_fp64
//
// Every thread runs 8 independent DFMA chains (enough independent work to cover the FP64
// pipe latency) for `iters` iterations; grids of 148 x {2, 4, 8} CTAs x 256 threads.
// Printed: DFMA/s and FP64 TFLOP/s (2 flops per FMA), best of 5 after a warm-up.
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

#define CK(x)                                                                        \
  do {                                                                               \
    cudaError_t e_ = (x);                                                            \
    if (e_ != cudaSuccess) {                                                         \
      std::fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_));                  \
      std::exit(1);                                                                  \
    }                                                                                \
  } while (0)

__global__ void __launch_bounds__(256) dfma_chains(double* out, int iters, double a, double b) {
  double x[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 1e-3 + k;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = fma(x[k], a, b);
  }
  double s = 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) s += x[k];
  if (s == 1.2345) out[threadIdx.x] = s;  // keep the chains alive
}

int main() {
  double* out = nullptr;
  CK(cudaMalloc(&out, 256 * sizeof(double)));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const int iters = 1 << 16;
  for (int per_sm : {2, 4, 8}) {
    const int blocks = 148 * per_sm;
    dfma_chains<<<blocks, 256>>>(out, iters, 0.999999, 1e-9);
    CK(cudaDeviceSynchronize());
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
      CK(cudaEventRecord(e0));
      dfma_chains<<<blocks, 256>>>(out, iters, 0.999999, 1e-9);
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      if (ms < best) best = ms;
    }
    const double fmas = (double)blocks * 256 * iters * 8;
    std::printf("blocks %4d (%d per SM): %8.3f ms  %.3e DFMA/s  %.2f FP64 TFLOP/s\n", blocks,
                per_sm, best, fmas / (best * 1e-3), 2.0 * fmas / (best * 1e-3) / 1e12);
  }
  return 0;
}
