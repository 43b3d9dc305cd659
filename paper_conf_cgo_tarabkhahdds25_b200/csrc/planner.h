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
};

struct Planner {
  int n = 0, n_local = 0, world = 1;
  int l2p[64], p2l[64];

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
  void plan_gate(const Decoded& g, std::vector<PlanOp>& out,
                 const std::vector<int>* next_use = nullptr);
  // Plans a whole circuit with Belady lookahead.
  void plan_circuit(const std::vector<Decoded>& gates, std::vector<PlanOp>& out);
  // Appends the ops that restore the identity map.
  void plan_canonicalize(std::vector<PlanOp>& out);
  // Specialises a LOCAL op for rank r: false if a global control is 0 there;
  // otherwise *out has only local targets/controls (diagonals on global targets
  // folded into a smaller diagonal; cls NOOP if nothing is left to do).
  bool rank_local(const Decoded& pg, int r, Decoded* out) const;

 private:
  Decoded to_physical(const Decoded& g) const;
  void exchange(int l, int g, std::vector<PlanOp>& out);
  void swap_local(int a, int b, std::vector<PlanOp>& out);
};

}  // namespace lfqs
