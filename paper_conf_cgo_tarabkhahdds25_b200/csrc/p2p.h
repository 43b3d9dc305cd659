// p2p.h -- peer-memory transport for the sharded state (NEXT-3).
//
// Every rank exports its shard and a small "aux" buffer (signal slots + a
// reduction area) through CUDA IPC; each rank maps all peers' buffers.  The
// global-qubit exchange then runs as ONE in-place swap kernel that
// loads and stores both shards directly (NVLink / NVSwitch peer accesses, no
// staging buffer, no extra HBM copy), the pairs split between the two partner
// ranks so both GPUs drive the link in both directions.  Ordering between ranks
// uses device-side flags: a one-thread kernel releases a counter into the
// peer's slot (st.release.sys) and waits, with a timeout, for the peer's counter
// in its own slot (ld.acquire.sys).  The reduction of measurement histograms
// sums every rank's buffer in rank order (deterministic).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "lfqs_internal.h"

namespace lfqs {

constexpr int kP2PHandleBytes = 256;    // LFQS_P2P_HANDLE_BYTES
constexpr size_t kP2PReduceDoubles = 1u << 20;  // measure_probs bins (n_q <= 20)

struct P2P {
  int rank = 0, world = 1, device = 0;
  unsigned char* peer_amps[64] = {};   // shard of every rank (own: the local pointer)
  unsigned char* peer_aux[64] = {};    // aux buffer of every rank
  unsigned char* aux = nullptr;        // own aux: [0, 512) signal slots, then reduce, result
  uint64_t sent[64] = {};              // barriers completed with each peer
  int* err_host = nullptr;             // mapped pinned flag: a barrier timed out
  int* err_dev = nullptr;
  bool attached = false;

  P2P(int rank, int world, int device);
  ~P2P();
  // 256 bytes: magic, rank, world, device, n_local, amp bytes, then the IPC
  // handles of the shard and of the aux buffer.
  void handle(const void* shard, int n_local, int amp_bytes, uint8_t out[kP2PHandleBytes]) const;
  void attach(unsigned char* own_shard, int n_local, int amp_bytes, const uint8_t* all);
  // Pairwise barrier with `peer` on stream s.
  void barrier_pair(int peer, cudaStream_t s);
  // All-rank barrier on stream s.
  void barrier_all(cudaStream_t s);
  // In-place half-shard exchange with the partner across global bit j (local
  // position l): this rank swaps its half of the pairs.  The exchange covers the
  // amplitudes of both shards whose bits `chunk` spell v in ascending position order
  // (a whole shard: chunk = 0; one block of an overlapped exchange otherwise), on
  // ctx.stream (barriers included); ctas > 0 bounds the swap kernel's grid.
  void exchange(const LaunchCtx& ctx, int l, int j, uint64_t chunk = 0, uint64_t v = 0,
                int ctas = 0);
  // out[0..count) = sum over ranks (in rank order) of every rank's in[0..count)
  // (host arrays).  Synchronous.
  void allreduce_sum(double* host, size_t count, cudaStream_t s);
  void check() const;  // throws if a barrier timed out
  double* reduce_area(int r) const {
    return reinterpret_cast<double*>(peer_aux[r] + 4096);
  }
  double* result_area() const {
    return reinterpret_cast<double*>(aux + 4096 + kP2PReduceDoubles * sizeof(double));
  }
  static size_t aux_bytes() { return 4096 + 2 * kP2PReduceDoubles * sizeof(double); }
};

}  // namespace lfqs
