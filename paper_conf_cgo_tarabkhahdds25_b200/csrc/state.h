// state.h -- the state allocator and executor of planned ops.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <vector>

#include "lfqs_internal.h"
#include "planner.h"

struct lfqs_state {
  virtual ~lfqs_state() = default;
};
struct lfqs_circuit {
  virtual ~lfqs_circuit() = default;
};

namespace lfqs {

struct Comm;  // NCCL communicator wrapper (comm.cu)
struct P2P;   // peer-memory transport (p2p.cu)

// Layout in HBM: a shard is 2^n_local interleaved complex128
// amplitudes, contiguous, 256-byte aligned.  Physical bit positions
// [0, n_local) are local; [n_local, n) are "global" and equal the rank's bits.
// The planner's l2p maps a logical qubit to its physical position.
struct State : lfqs_state {
  int n = 0, n_local = 0, rank = 0, world = 1, p = 0, device = 0;
  bool virt = false;            // `world` shards in one allocation (single GPU)
  unsigned char* amps = nullptr;  // shard 0 (virtual: all shards back to back)
  bool c64 = false;             // complex64 amplitudes (NEXT-4); default complex128
  bool soa = false;             // structure-of-arrays planes (NEXT-4); default AOS
  int ab = 16;                  // bytes per amplitude
  bool owned = false;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  uint64_t launches = 0;
  uint64_t passes = 0;          // state passes run (lfqs_state_pass_count)
  Options opt;
  double* d_partials = nullptr; // reduction scratch (grown on demand)
  double* d_probs = nullptr;    // 2^nq result bins (grown on demand)
  size_t partials_cap = 0, probs_cap = 0;  // doubles
  Planner plan;
  Comm* comm = nullptr;
  P2P* p2p = nullptr;           // CUDA-IPC peer transport (instead of comm)
  // exchange statistics (benchmark accounting)
  uint64_t exchanges = 0, exchange_bytes = 0;
  uint64_t ov_exchanges = 0, ov_block_passes = 0, ov_strided = 0, ov_chained = 0;

  static State* create_local(int n, int device, cudaStream_t stream, void* borrowed,
                             bool c64 = false, bool soa = false);
  static State* create_virtual(int n, int world, int device, cudaStream_t stream,
                               bool c64 = false);
  static State* create_dist(int n, int rank, int world, const uint8_t uid[128], int device,
                            cudaStream_t stream);
  // One rank of a P2P-sharded state: peers are attached later (p2p_attach).
  static State* create_p2p(int n, int rank, int world, int device, cudaStream_t stream,
                           bool c64 = false);
  void p2p_handle(uint8_t* out);
  void p2p_attach(const uint8_t* all);
  static void nccl_unique_id(uint8_t uid[128]);
  ~State() override;

  void set_stream(cudaStream_t s);
  void init_basis(uint64_t index);
  void init_random(uint64_t seed);
  // Host buffers: interleaved doubles (converted for complex64 states) ...
  void copy(uint64_t offset, uint64_t count, double* host, bool to_device);
  // ... or raw amplitudes of the state's own type (no conversion).
  void copy_raw(uint64_t offset, uint64_t count, void* host, bool to_device);
  void apply(const Decoded& g);
  void run(const std::vector<Decoded>& gates, uint32_t flags);
  // Uploads the whole state from `host` in 2^chunk_bits pieces on a copy stream while the
  // circuit prefix that stays inside pieces runs on each landed piece; then the rest.
  void run_streamed(const void* host, const std::vector<Decoded>& gates, uint32_t flags,
                    int chunk_bits);
  // Captures the launches of run(gates, flags) into a CUDA graph (no GPU work).
  struct Graph* compile(const std::vector<Decoded>& gates, uint32_t flags);
  void measure_probs(const int* qubits, int nq, double* out);
  void local_probs(int shard, const int* lq, int nl, double* host);
  // Zeroes amplitudes whose measured bits != outcome, scales the rest by `scale`.
  void collapse(const int* qubits, int nq, uint64_t outcome, double scale);
  void synchronize();
  // Waits for the state's stream (NCCL states: polling the communicator's async errors
  // with a timeout, Comm::wait).
  void wait_stream();
  void* shard_ptr() const { return amps; }

 private:
  State() = default;
  void common_init(int n_, int world_, int device_, cudaStream_t s, bool c64_ = false);
  LaunchCtx ctx(int shard);
  bool phase_tables = false;  // LFQS_FUSE_PHASE of the run in progress
  bool jit = false;           // LFQS_FUSE_JIT of the run in progress
  cudaStream_t copy_stream = nullptr;  // run_streamed uploads (created on first use)
  cudaStream_t xstream = nullptr;      // overlapped exchanges (device / P2P transports)
  std::vector<cudaEvent_t> ev_tail, ev_done;  // per exchange part, reused
  int overlap_bits() const;
  cudaEvent_t part_event(std::vector<cudaEvent_t>& pool, int v);
  std::vector<Decoded> segment(const std::vector<PlanOp>& ops, size_t b, size_t e, int shard);
  // A run of LOCAL ops planned into passes, per shard (rank-specialised gates + passes).
  struct ShardRun {
    std::vector<Decoded> seg;
    std::vector<FusedPass> passes;
  };
  std::vector<ShardRun> plan_run(const std::vector<PlanOp>& ops, size_t b, size_t e, bool fuse);
  // Launches passes [from[s], to[s]) of every shard, on the whole shard (chunk = 0) or on
  // block v of the chunk qubits (the passes do not mix them: pass_blockwise).
  void launch_passes(const std::vector<ShardRun>& run, const std::vector<size_t>& from,
                     const std::vector<size_t>& to, uint64_t chunk, uint64_t v);
  // Chunk qubits of the overlapped exchange ops[ex[k]] (0: serial); prev: the previous
  // exchange's, when its run may continue block by block.
  uint64_t choose_chunk(const std::vector<PlanOp>& ops, const std::vector<size_t>& ex, size_t k,
                        bool fuse, uint64_t prev) const;
  // One block of an exchange; the data it moves is final once `ready` has fired.  Returns
  // the event the compute stream must wait for before using the block (NULL: the copies
  // already sit on the compute stream, NCCL transport).
  cudaEvent_t exchange_part(int l, int g, uint64_t chunk, uint64_t v, cudaEvent_t ready);
  int n_shards() const { return virt ? world : 1; }
  int rank_of_shard(int shard) const { return virt ? shard : rank; }
  void execute(const std::vector<PlanOp>& ops, bool fuse);
  void run_local(const LaunchCtx& c, const std::vector<Decoded>& gates, bool fuse);
  void exchange_data(int l, int g);  // swap physical positions l (local) and g (global)
  void canonicalize();
  void plan_window();  // the planner's exchange window for this state's transport
};

// A circuit captured by State::compile; launch() replays it on the state's stream.
struct Graph : lfqs_circuit {
  State* st = nullptr;
  cudaGraphExec_t exec = nullptr;
  uint64_t kernels = 0;  // kernels per replay
  void launch();
  ~Graph() override;
};

}  // namespace lfqs
