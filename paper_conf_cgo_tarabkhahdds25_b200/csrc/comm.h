// comm.h -- NCCL wrapper for the sharded state (see comm.cu).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <vector>

#include "lfqs_internal.h"

typedef struct ncclComm* ncclComm_t;

namespace lfqs {

struct Piece {
  uint64_t offset;  // amplitudes from the shard start
  uint64_t count;   // amplitudes
};

struct Comm {
  int rank = 0, world = 1;
  ncclComm_t comm = nullptr;
  cudaStream_t cstream = nullptr;
  unsigned char* stage[2] = {nullptr, nullptr};
  uint64_t stage_bytes = 0;
  cudaEvent_t ev_recv[2], ev_free[2], ev_start;
  int next_stage = 0;                   // staging buffer of the next chunk
  bool stage_used[2] = {false, false};  // ev_free[b] marks the end of its last use
  double* d_reduce = nullptr;

  static void unique_id(uint8_t uid[128]);
  Comm(int rank, int world, const uint8_t uid[128], size_t stage_bytes);
  ~Comm();
  // pieces are in amplitudes of `amp_bytes` bytes each.
  // ready: the transfers wait for this event (NULL: for all work queued on `compute`);
  // landed chunks are copied into place on `compute`.
  void exchange(void* shard, int amp_bytes, const std::vector<Piece>& pieces, int partner,
                cudaStream_t compute, cudaEvent_t ready = nullptr);
  void allreduce_sum(double* d, size_t count, cudaStream_t s);
  // Waits for stream s while polling ncclCommGetAsyncError: a failed or hung peer
  // (no progress for timeout_s seconds; LFQS_NCCL_TIMEOUT_S, default 300) aborts the
  // communicator and throws LFQS_ERR_NCCL instead of blocking forever.
  void wait(cudaStream_t s);
};

}  // namespace lfqs
