// planner.cpp -- host-only distributed gate planner.
//
// P = 2^p ranks; rank r owns the amplitudes whose top p physical bits equal r.
// l2p maps a logical qubit to its physical bit position; positions >= n_local
// are "global" (rank bits).  For each logical gate:
//   (i)   targets local, controls anywhere -> LOCAL op; global controls become
//         a rank predicate (rank_local);
//   (ii)  diagonal with global targets -> LOCAL op; the rank's global bits fold
//         into a smaller diagonal on the local targets (no communication);
//   (iii) other gates with a global target g -> EXCHANGE(l, g) with the highest
//         local position l that is not a target (the half-shard swap of comm.cu),
//         then (i);
//   SWAP(global, local) without controls -> relabel of the map (no op at all).
// No multi-GPU component exists in the paper; this is the
// sharding BASELINE.json's north_star asks for.
#include "planner.h"

#include <algorithm>

namespace lfqs {

Planner::Planner(int n_, int world_) : n(n_), world(world_) {
  int p = 0;
  while ((1 << p) < world) ++p;
  require((1 << p) == world, "world size must be a power of two");
  n_local = n - p;
  require(world == 1 || n_local >= 4, "each shard needs at least 4 local qubits");
  reset();
}

void Planner::reset() {
  for (int q = 0; q < 64; ++q) l2p[q] = p2l[q] = q;
  gflip = 0;
}

bool Planner::identity() const {
  if (gflip != 0) return false;
  for (int q = 0; q < n; ++q)
    if (l2p[q] != q) return false;
  return true;
}

Decoded Planner::to_physical(const Decoded& g) const {
  Decoded pg = g;
  for (int s = 0; s < g.m; ++s) pg.targets[s] = l2p[g.targets[s]];
  uint64_t cm = 0;
  for (int q = 0; q < n; ++q)
    if (g.cmask >> q & 1) cm |= 1ull << l2p[q];
  pg.cmask = cm;
  return pg;
}

void Planner::exchange(int l, int g, std::vector<PlanOp>& out) {
  require(l >= 0 && l < n_local && g >= n_local && g < n, "internal: bad exchange positions");
  PlanOp op;
  op.kind = PlanOp::EXCHANGE;
  op.l = l;
  op.g = g;
  out.push_back(op);
  const int qa = p2l[l], qb = p2l[g];
  l2p[qa] = g;
  l2p[qb] = l;
  p2l[l] = qb;
  p2l[g] = qa;
  if (gflip >> g & 1) {
    // The incoming qubit was relabelled by global X gates: materialise the flip
    // on its new local position (the qubit now at g carries no flip).
    gflip &= ~(1ull << g);
    const int t[1] = {l};
    PlanOp x;
    x.kind = PlanOp::LOCAL;
    x.gate = decode_gate(n, LFQS_X, t, 1, 0, nullptr, 0, nullptr);
    x.gflip = gflip;
    out.push_back(x);
  }
}

void Planner::swap_local(int a, int b, std::vector<PlanOp>& out) {
  const int t[2] = {a, b};
  PlanOp op;
  op.kind = PlanOp::LOCAL;
  op.gate = decode_gate(n, LFQS_SWAP, t, 2, 0, nullptr, 0, nullptr);
  op.gflip = gflip;
  out.push_back(op);
  const int qa = p2l[a], qb = p2l[b];
  l2p[qa] = b;
  l2p[qb] = a;
  p2l[a] = qb;
  p2l[b] = qa;
}

void Planner::plan_canonicalize(std::vector<PlanOp>& out) {
  // Phase 0: materialise global flips (each costs one exchange and an X pass;
  // the phases below then move every qubit home).
  for (int G = n_local; G < n; ++G)
    if (gflip >> G & 1) exchange(n_local - 1, G, out);
  // Phase 1: bring each global home position G its logical qubit G -- one exchange
  // when that qubit sits at a local position, two (through a local staging position
  // L) when it sits at another global one.  L is chosen as the home of the qubit that
  // leaves G, so that qubit lands where phase 2 wants it.
  // Every exchange stays inside the top kSwapWindow local positions, as in plan_gate: a
  // low position l would split the exchanged half-shard into 2^(n_local-1-l) pieces of
  // 2^l amplitudes (the NCCL transport sends one message per piece).  A qubit that sits
  // lower is first moved to the top local position by one local SWAP pass.
  const int wlo = swap_lo >= 0 ? std::min(swap_lo, n_local - 1) : std::max(0, n_local - kSwapWindow);
  for (int G = n - 1; G >= n_local; --G) {
    int P = l2p[G];
    if (P == G) continue;
    if (P < n_local) {
      if (P < wlo) {
        swap_local(P, n_local - 1, out);
        P = n_local - 1;
      }
      exchange(P, G, out);
    } else {
      const int x = p2l[G];
      const int L = (x < n_local && x >= wlo) ? x : n_local - 1;
      exchange(L, P, out);
      exchange(L, G, out);
    }
  }
  // Phase 2: the local positions now hold a permutation of the local qubits; fix it
  // with local SWAP passes (no communication).
  for (int q = 0; q < n_local; ++q)
    if (l2p[q] != q) swap_local(l2p[q], q, out);
}

void Planner::plan_circuit(const std::vector<Decoded>& gates, std::vector<PlanOp>& out) {
  // uses[q] = ascending gate indices where logical q is a non-diagonal target.
  std::vector<std::vector<int>> uses(n);
  for (size_t i = 0; i < gates.size(); ++i) {
    const Decoded& g = gates[i];
    if (g.cls == GClass::NOOP || g.cls == GClass::DIAG) continue;
    if (g.cls == GClass::PERM_X && g.cmask == 0) continue;  // relabel when global
    for (int s = 0; s < g.m; ++s) uses[g.targets[s]].push_back((int)i);
  }
  std::vector<int> next_use(n);
  for (size_t i = 0; i < gates.size(); ++i) {
    for (int q = 0; q < n; ++q) {
      auto it = std::upper_bound(uses[q].begin(), uses[q].end(), (int)i);
      next_use[q] = it == uses[q].end() ? (1 << 30) : *it;
    }
    plan_gate(gates[i], out, &next_use);
  }
}

void Planner::plan_gate(const Decoded& g, std::vector<PlanOp>& out,
                        const std::vector<int>* next_use) {
  if (g.cls == GClass::NOOP) return;
  Decoded pg = to_physical(g);
  if (world > 1 && pg.cls == GClass::PERM_X && pg.cmask == 0 && pg.targets[0] >= n_local) {
    gflip ^= 1ull << pg.targets[0];  // global X: relabel, no data movement
    return;
  }
  if (world > 1 && pg.cls == GClass::PERM_SWAP && pg.cmask == 0 &&
      (pg.targets[0] >= n_local || pg.targets[1] >= n_local)) {
    // SWAP of logical qubits = exchange their physical positions in the map.
    const int qa = g.targets[0], qb = g.targets[1];
    std::swap(l2p[qa], l2p[qb]);
    p2l[l2p[qa]] = qa;
    p2l[l2p[qb]] = qb;
    return;
  }
  if (pg.cls != GClass::DIAG) {
    for (int s = 0; s < pg.m; ++s) {
      const int gq = pg.targets[s];
      if (gq < n_local) continue;
      uint64_t tmask = 0;
      for (int u = 0; u < pg.m; ++u) tmask |= 1ull << pg.targets[u];
      int l = -1, best = -1;
      const int rsv = std::max(0, std::min(reserve_top, n_local - 4));
      const int top = n_local - 1 - rsv;
      const int lo = swap_lo >= 0 ? std::min(swap_lo, top) : std::max(0, top + 1 - kSwapWindow);
      for (int p = top; p >= lo; --p) {
        if (tmask >> p & 1) continue;
        const int score = next_use ? (*next_use)[p2l[p]] : 0;
        if (score > best) {
          best = score;
          l = p;
        }
      }
      for (int p = lo - 1; l < 0 && p >= 0; --p)
        if (!(tmask >> p & 1)) l = p;
      for (int p = n_local - 1; l < 0 && p > top; --p)  // only the reserved ones are left
        if (!(tmask >> p & 1)) l = p;
      require(l >= 0, "internal: no free local qubit");
      exchange(l, gq, out);
      pg.targets[s] = l;
      if (pg.cmask >> l & 1) pg.cmask = (pg.cmask & ~(1ull << l)) | (1ull << gq);
    }
  }
  PlanOp op;
  op.kind = PlanOp::LOCAL;
  op.gate = pg;
  op.gflip = gflip;
  out.push_back(op);
}

bool Planner::rank_local(const Decoded& pg, int r_phys, uint64_t f, Decoded* out) const {
  const uint64_t local_mask = (n_local >= 64) ? ~0ull : ((1ull << n_local) - 1);
  // The logical values of the global positions on this rank (flips applied).
  const int r = r_phys ^ (int)(f >> n_local);
  const uint64_t gctrl = pg.cmask >> n_local;
  if ((gctrl & (uint64_t)r) != gctrl) return false;  // a global control is 0 on this rank
  *out = pg;
  out->cmask = pg.cmask & local_mask;
  bool all_local = true;
  for (int s = 0; s < pg.m; ++s) all_local &= pg.targets[s] < n_local;
  if (all_local) return true;
  require(pg.cls == GClass::DIAG, "internal: non-diagonal gate with a global target");
  // Diagonal: fold the rank's global target bits into a smaller diagonal.
  const int d = 1 << pg.m;
  int lt[3], ls[3], mp = 0;
  for (int s = 0; s < pg.m; ++s)
    if (pg.targets[s] < n_local) {
      lt[mp] = pg.targets[s];
      ls[mp] = s;
      ++mp;
    }
  cplx dd[8];
  for (int jp = 0; jp < (1 << mp); ++jp) {
    int j = 0;
    for (int s = 0, u = 0; s < pg.m; ++s) {
      int bit;
      if (u < mp && ls[u] == s) {
        bit = (jp >> (mp - 1 - u)) & 1;
        ++u;
      } else {
        bit = (r >> (pg.targets[s] - n_local)) & 1;
      }
      j |= bit << (pg.m - 1 - s);
    }
    dd[jp] = pg.M[j * d + j];
  }
  out->m = mp;
  for (int s = 0; s < 3; ++s) out->targets[s] = s < mp ? lt[s] : 0;
  const int dp = 1 << mp;
  for (int i = 0; i < 64; ++i) out->M[i] = cplx{0.0, 0.0};
  bool ones = true;
  for (int j = 0; j < dp; ++j) {
    out->M[j * dp + j] = dd[j];
    ones &= dd[j].re == 1.0 && dd[j].im == 0.0;
  }
  out->cls = ones ? GClass::NOOP : GClass::DIAG;
  out->is_h = false;
  out->kind = LFQS_UNITARY1 + (mp > 0 ? mp - 1 : 0);
  return true;
}

}  // namespace lfqs
