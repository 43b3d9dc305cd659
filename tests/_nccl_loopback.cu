// Test driver (tests/test_gpu_nccl_loopback.py): the NCCL transport of the sharded state
// (paper_conf_cgo_tarabkhahdds25_b200/csrc/comm.cu) run for real on one GPU.  NCCL refuses
// two ranks on one device, so the communicator has one rank and every exchange is with
// itself: ncclSend of each piece and ncclRecv into the staging buffers in one group, then the
// staged copies back into place on the compute stream -- the same calls, chunking, staging
// reuse across calls and events as between two GPUs, with the identity as the expected
// result (a wrong offset, chunk size or a staging buffer reused too early changes data).
// Also the all-reduce and the async-error polling wait.  Prints "ok" or the first failure.
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "comm.h"

int main() {
  using namespace lfqs;
  try {
    uint8_t uid[128];
    Comm::unique_id(uid);
    Comm c(0, 1, uid, 3u << 20);  // 3 MiB staging buffers: many chunks per piece
    const uint64_t N = 1ull << 22;  // amplitudes of 16 B
    std::vector<double> h(2 * N);
    for (uint64_t i = 0; i < 2 * N; ++i) h[i] = (double)(i * 2654435761ull % 1000003) - 5e5;
    double* d = nullptr;
    LFQS_CUDA_CHECK(cudaMalloc(&d, N * 16));
    LFQS_CUDA_CHECK(cudaMemcpy(d, h.data(), N * 16, cudaMemcpyHostToDevice));
    cudaStream_t s;
    LFQS_CUDA_CHECK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    // the pieces of a half-shard exchange at a low position (many pieces), one at the top
    // position (one large piece), and an overlapped exchange's parts (consecutive calls)
    std::vector<Piece> low, top = {{N / 2, N / 2}};
    for (uint64_t k = 0; k < N; k += 1u << 14) low.push_back(Piece{k + (1u << 13), 1u << 13});
    c.exchange(d, 16, low, 0, s);
    c.exchange(d, 16, top, 0, s);
    cudaEvent_t ready;
    LFQS_CUDA_CHECK(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming));
    for (int part = 0; part < 4; ++part) {
      LFQS_CUDA_CHECK(cudaEventRecord(ready, s));
      const std::vector<Piece> pc = {{part * (N / 4), N / 8}, {part * (N / 4) + N / 8 + 7, 1000}};
      c.exchange(d, 16, pc, 0, s, ready);
    }
    c.wait(s);
    std::vector<double> out(2 * N);
    LFQS_CUDA_CHECK(cudaMemcpy(out.data(), d, N * 16, cudaMemcpyDeviceToHost));
    for (uint64_t i = 0; i < 2 * N; ++i)
      if (out[i] != h[i]) {
        std::printf("exchange changed double %llu: %g != %g\n", (unsigned long long)i, out[i], h[i]);
        return 1;
      }
    // all-reduce over the one rank: the values themselves
    double* r = nullptr;
    const double v[5] = {1.5, -2.25, 3e-300, 0.0, 7.0};
    LFQS_CUDA_CHECK(cudaMalloc(&r, sizeof v));
    LFQS_CUDA_CHECK(cudaMemcpy(r, v, sizeof v, cudaMemcpyHostToDevice));
    c.allreduce_sum(r, 5, s);
    c.wait(s);
    double w[5];
    LFQS_CUDA_CHECK(cudaMemcpy(w, r, sizeof w, cudaMemcpyDeviceToHost));
    for (int i = 0; i < 5; ++i)
      if (w[i] != v[i]) {
        std::printf("allreduce changed value %d\n", i);
        return 1;
      }
    cudaFree(r);
    cudaFree(d);
    cudaStreamDestroy(s);
    std::printf("ok chunks=%zu+%zu+8\n", low.size(), top.size());
    return 0;
  } catch (const std::exception& e) {
    std::printf("error: %s\n", e.what());
    return 2;
  }
}
