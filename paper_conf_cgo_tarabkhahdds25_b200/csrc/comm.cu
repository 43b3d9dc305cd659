// comm.cu -- global-qubit exchange and reductions across GPUs over NCCL.
//
// No multi-GPU component exists in the paper (single node OpenMP or one GPU,
// P:551); this is the B200 sharding that BASELINE.json's north_star asks
// for.  A gate whose target is a global qubit g is made local by swapping g with
// a local qubit l: rank r (global bit b) and its partner r ^ 2^(g - n_local)
// exchange the half-shard whose l-bit is 1 - b (16 * 2^(n_local-1) bytes each
// way).  The transfer is chunked through two staging buffers on a dedicated
// communication stream; each landed chunk is copied into place on the compute
// stream while the next chunk is in flight (events hand buffers back and forth).
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <string>
#include <thread>

#include "comm.h"

namespace lfqs {

#define LFQS_NCCL_CHECK(expr)                                                                \
  do {                                                                                       \
    ncclResult_t _r = (expr);                                                                \
    if (_r != ncclSuccess)                                                                   \
      throw ::lfqs::Error(LFQS_ERR_NCCL, std::string(#expr) + ": " + ncclGetErrorString(_r)); \
  } while (0)

static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId must be 128 bytes");

void Comm::unique_id(uint8_t uid[128]) {
  ncclUniqueId id;
  LFQS_NCCL_CHECK(ncclGetUniqueId(&id));
  std::memcpy(uid, &id, 128);
}

Comm::Comm(int rank_, int world_, const uint8_t uid[128], size_t stage_bytes)
    : rank(rank_), world(world_) {
  ncclUniqueId id;
  std::memcpy(&id, uid, 128);
  LFQS_NCCL_CHECK(ncclCommInitRank(&comm, world, id, rank));
  LFQS_CUDA_CHECK(cudaStreamCreateWithFlags(&cstream, cudaStreamNonBlocking));
  this->stage_bytes = stage_bytes;
  for (int i = 0; i < 2; ++i) {
    LFQS_CUDA_CHECK(cudaMalloc(&stage[i], stage_bytes));
    LFQS_CUDA_CHECK(cudaEventCreateWithFlags(&ev_recv[i], cudaEventDisableTiming));
    LFQS_CUDA_CHECK(cudaEventCreateWithFlags(&ev_free[i], cudaEventDisableTiming));
  }
  LFQS_CUDA_CHECK(cudaEventCreateWithFlags(&ev_start, cudaEventDisableTiming));
  LFQS_CUDA_CHECK(cudaMalloc(&d_reduce, 8 * 1024));
}

Comm::~Comm() {
  if (comm) cudaStreamSynchronize(cstream);
  for (int i = 0; i < 2; ++i) {
    cudaFree(stage[i]);
    cudaEventDestroy(ev_recv[i]);
    cudaEventDestroy(ev_free[i]);
  }
  cudaEventDestroy(ev_start);
  cudaFree(d_reduce);
  cudaStreamDestroy(cstream);
  if (comm) ncclCommDestroy(comm);
}

// Exchanges the amplitudes at `pieces` (offset, count in amplitudes, in this
// rank's shard) with the same pieces of `partner`, in place.
void Comm::exchange(void* shard, int amp_bytes, const std::vector<Piece>& pieces, int partner,
                    cudaStream_t compute, cudaEvent_t ready) {
  require(comm != nullptr, "NCCL communicator was aborted after an earlier error");
  // The comm stream must see every kernel the exchanged data depends on: `ready`, or
  // everything already queued on the compute stream.
  if (ready == nullptr) {
    LFQS_CUDA_CHECK(cudaEventRecord(ev_start, compute));
    ready = ev_start;
  }
  LFQS_CUDA_CHECK(cudaStreamWaitEvent(cstream, ready, 0));
  const uint64_t stage_amps = stage_bytes / amp_bytes;
  unsigned char* base = static_cast<unsigned char*>(shard);
  for (const Piece& pc : pieces) {
    for (uint64_t off = 0; off < pc.count; off += stage_amps) {
      const uint64_t cnt = std::min<uint64_t>(stage_amps, pc.count - off);
      const size_t bytes = cnt * amp_bytes;
      // A staging buffer is reused only after the compute stream has copied its previous
      // contents out -- also across calls: the parts of an overlapped exchange are separate
      // calls whose `ready` events may precede the previous part's copies.
      const int b = next_stage;
      next_stage ^= 1;
      if (stage_used[b]) LFQS_CUDA_CHECK(cudaStreamWaitEvent(cstream, ev_free[b], 0));
      stage_used[b] = true;
      unsigned char* src = base + (pc.offset + off) * amp_bytes;
      LFQS_NCCL_CHECK(ncclGroupStart());
      LFQS_NCCL_CHECK(ncclSend(src, bytes, ncclUint8, partner, comm, cstream));
      LFQS_NCCL_CHECK(ncclRecv(stage[b], bytes, ncclUint8, partner, comm, cstream));
      LFQS_NCCL_CHECK(ncclGroupEnd());
      LFQS_CUDA_CHECK(cudaEventRecord(ev_recv[b], cstream));
      LFQS_CUDA_CHECK(cudaStreamWaitEvent(compute, ev_recv[b], 0));
      LFQS_CUDA_CHECK(cudaMemcpyAsync(src, stage[b], bytes, cudaMemcpyDeviceToDevice, compute));
      LFQS_CUDA_CHECK(cudaEventRecord(ev_free[b], compute));
    }
  }
}

void Comm::wait(cudaStream_t s) {
  double timeout_s = 300.0;
  if (const char* e = std::getenv("LFQS_NCCL_TIMEOUT_S")) timeout_s = std::atof(e);
  const auto t0 = std::chrono::steady_clock::now();
  for (unsigned spin = 0;; ++spin) {
    const cudaError_t q = cudaStreamQuery(s);
    if (q == cudaSuccess) return;
    if (q != cudaErrorNotReady) LFQS_CUDA_CHECK(q);
    ncclResult_t async = ncclSuccess;
    LFQS_NCCL_CHECK(ncclCommGetAsyncError(comm, &async));
    if (async != ncclSuccess && async != ncclInProgress) {
      ncclCommAbort(comm);
      comm = nullptr;
      throw Error(LFQS_ERR_NCCL, std::string("NCCL asynchronous error: ") +
                                     ncclGetErrorString(async));
    }
    const double el =
        std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    if (timeout_s > 0 && el > timeout_s) {
      ncclCommAbort(comm);
      comm = nullptr;
      throw Error(LFQS_ERR_NCCL, "NCCL operation did not complete within " +
                                     std::to_string(timeout_s) + " s (peer lost?); "
                                     "communicator aborted");
    }
    std::this_thread::sleep_for(std::chrono::microseconds(spin < 100 ? 20 : 500));
  }
}

void Comm::allreduce_sum(double* d, size_t count, cudaStream_t s) {
  require(comm != nullptr, "NCCL communicator was aborted after an earlier error");
  LFQS_NCCL_CHECK(ncclAllReduce(d, d, count, ncclDouble, ncclSum, comm, s));
}

}  // namespace lfqs
