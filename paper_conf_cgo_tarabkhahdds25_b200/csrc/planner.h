// planner.h -- host-only distributed gate planner (component C10/C12).
//
// Pure host logic (no CUDA calls), shared by the NCCL path, the single-GPU
// virtual partition and lfqs_plan_circuit (which the CPU gloo tests drive).
#pragma once
#include <cstdint>
#include <vector>

#include "lfqs_internal.h"

namespace lfqs {

struct PlanOp {
  enum Kind : int { LOCAL = 0, EXCHANGE = 1 };
  int kind = LOCAL;
  Decoded gate;   // LOCAL: gate on physical positions (controls may be global)
  int l = 0;      // EXCHANGE: local physical position
  int g = 0;      // EXCHANGE: global physical position (rank bit g - n_local)
  uint64_t gflip = 0;  // LOCAL: the global-position flips in force for this op
};

struct Planner {
  int n = 0, n_local = 0, world = 1;
  int l2p[64], p2l[64];
  // Global-X relabeling (NEXT-1): bit P set = the data at global position P holds
  // the complement of its logical qubit (rank bit = logical value ^ 1).  An
  // uncontrolled X on a global qubit toggles it instead of moving data; the flip
  // is materialised (an X pass on the local position) when the qubit is
  // exchanged back into the shard.
  uint64_t gflip = 0;

  Planner() { reset(); }
  Planner(int n_, int world_);
  void reset();
  bool identity() const;
  // Appends the physical ops for logical gate g and updates the qubit map.
  // next_use(q) (optional) = index of the next gate that has logical qubit q as
  // a non-diagonal target (a large value if none): the evicted local qubit is
  // the one used furthest in the future (Belady), among the top kSwapWindow
  // local positions (so exchanged pieces stay >= 2^(n_local - kSwapWindow) amps).
  static constexpr int kSwapWindow = 8;
  // >= 0: exchange positions may go down to this local position instead (the device and
  // P2P transports swap any block in place, so small pieces cost nothing extra there; the
  // NCCL transport keeps the window for its message sizes).  Set per run by the State.
  int swap_lo = -1;
  // The top reserve_top local positions are never chosen as the exchange position l by
  // plan_gate: they are the chunk bits of overlapped exchanges (state.cu execute), which
  // split an exchange into parts by them while the neighbouring local ops run part by part.
  // kOverlapBits (Options::exchange_chunk_bits' default) whatever that option is, so serial
  // and overlapped executions run the same plan; fewer for tiny shards.
  static constexpr int kOverlapBits = 2;
  int reserve_top = kOverlapBits;
  void plan_gate(const Decoded& g, std::vector<PlanOp>& out,
                 const std::vector<int>* next_use = nullptr);
  // Plans a whole circuit with Belady lookahead.
  void plan_circuit(const std::vector<Decoded>& gates, std::vector<PlanOp>& out);
  // Appends the ops that restore the identity map.
  void plan_canonicalize(std::vector<PlanOp>& out);
  // Specialises a LOCAL op for rank r: false if a global control is 0 there;
  // otherwise *out has only local targets/controls (diagonals on global targets
  // folded into a smaller diagonal; cls NOOP if nothing is left to do).
  // gflip: the op's flips (PlanOp::gflip); r is read through them.
  bool rank_local(const Decoded& pg, int r, uint64_t gflip, Decoded* out) const;
  // The logical value of global position P on rank r under flips f.
  int global_bit(int r, int P, uint64_t f) const {
    return ((r >> (P - n_local)) & 1) ^ (int)((f >> P) & 1);
  }

 private:
  Decoded to_physical(const Decoded& g) const;
  void exchange(int l, int g, std::vector<PlanOp>& out);
  void swap_local(int a, int b, std::vector<PlanOp>& out);
};

}  // namespace lfqs
