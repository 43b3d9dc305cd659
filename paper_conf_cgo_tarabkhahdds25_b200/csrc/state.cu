// state.cu -- state allocator, logical<->physical qubit map and the distributed
// gate planner (components C10 and C12).
//
// One GPU: the map is the identity and every gate is one launch_gate() pass.
// P = 2^p ranks: rank r owns the amplitudes whose top p physical bits equal r.
//   (i)  targets local, controls anywhere: global controls are a rank predicate;
//   (ii) diagonal gate with global targets: the factor of the global bits is
//        rank-constant -> a smaller diagonal on the local targets, no traffic;
//   (iii) other gates with a global target g: swap g with the highest local
//        position l that is not a target (half-shard exchange), then (i);
//   SWAP(global, local) without controls is a relabel of the map (no traffic).
// copy_out / copy_in canonicalise the map first; measure_probs translates the
// measured qubits through the map instead (no data movement).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <memory>
#include <string>

#include "comm.h"
#include "state.h"

namespace lfqs {

// Defined in apply_kernels.cu.
void launch_half_swap(const LaunchCtx& ctx, int l, uint64_t partner_offset_amps);
bool run_fused_circuit(const LaunchCtx& ctx, const std::vector<Decoded>& gates, size_t begin,
                       size_t end, int tile_qubits, size_t* consumed);

namespace {
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) LFQS_CUDA_CHECK(cudaSetDevice(dev));
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

int log2_exact(int x) {
  int p = 0;
  while ((1 << p) < x) ++p;
  return (1 << p) == x ? p : -1;
}

double* alloc_amps(uint64_t n_amps) {
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, n_amps * 16);
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    throw Error(LFQS_ERR_OUT_OF_MEMORY,
                "cannot allocate " + std::to_string(n_amps * 16) + " bytes of device memory");
  }
  LFQS_CUDA_CHECK(e);
  return static_cast<double*>(p);
}
}  // namespace

void State::common_init(int n_, int world_, int device_, cudaStream_t s) {
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    throw Error(LFQS_ERR_CUDA, "no CUDA device available (this library has no CPU fallback)");
  }
  require(device_ >= 0 && device_ < ndev, "device index out of range");
  require(world_ >= 1 && log2_exact(world_) >= 0, "world size must be a power of two");
  n = n_;
  world = world_;
  p = log2_exact(world_);
  n_local = n - p;
  device = device_;
  require(n >= 1 && n <= 40, "n_qubits must be in [1, 40]");
  require(world == 1 || n_local >= 4, "each shard needs at least 4 local qubits");
  LFQS_CUDA_CHECK(cudaSetDevice(device));
  if (s) {
    stream = s;
  } else {
    LFQS_CUDA_CHECK(cudaStreamCreateWithFlags(&stream, cudaStreamNonBlocking));
    own_stream = true;
  }
  LFQS_CUDA_CHECK(cudaMalloc(&d_partials, sizeof(double) * probs_blocks() * 1024));
  LFQS_CUDA_CHECK(cudaMalloc(&d_probs, sizeof(double) * 1024));
  reset_map();
}

State* State::create_local(int n, int device, cudaStream_t stream, void* borrowed) {
  require(n >= 1 && n <= 36, "n_qubits must be in [1, 36] on one GPU");
  std::unique_ptr<State> st(new State());
  st->common_init(n, 1, device, stream);
  if (borrowed) {
    st->amps = static_cast<double*>(borrowed);
  } else {
    st->amps = alloc_amps(1ull << n);
    st->owned = true;
    st->init_basis(0);
  }
  return st.release();
}

State* State::create_virtual(int n, int world, int device, cudaStream_t stream) {
  require(world >= 2, "virtual partition needs world >= 2");
  std::unique_ptr<State> st(new State());
  st->virt = true;
  st->common_init(n, world, device, stream);
  st->amps = alloc_amps(1ull << n);
  st->owned = true;
  st->init_basis(0);
  return st.release();
}

void State::nccl_unique_id(uint8_t uid[128]) { Comm::unique_id(uid); }

State* State::create_dist(int n, int rank, int world, const uint8_t uid[128], int device,
                          cudaStream_t stream) {
  require(rank >= 0 && rank < world, "rank out of range");
  std::unique_ptr<State> st(new State());
  st->common_init(n, world, device, stream);
  st->rank = rank;
  st->amps = alloc_amps(1ull << st->n_local);
  st->owned = true;
  if (world > 1) {
    const uint64_t half = 16ull << (st->n_local - 1);
    st->comm = new Comm(rank, world, uid, std::min<uint64_t>(256ull << 20, half));
  }
  st->init_basis(0);
  return st.release();
}

State::~State() {
  if (device >= 0) cudaSetDevice(device);
  if (stream) cudaStreamSynchronize(stream);
  delete comm;
  if (owned && amps) cudaFree(amps);
  if (d_partials) cudaFree(d_partials);
  if (d_probs) cudaFree(d_probs);
  if (own_stream && stream) cudaStreamDestroy(stream);
}

void State::set_stream(cudaStream_t s) {
  DeviceGuard dg(device);
  LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
  if (own_stream) {
    cudaStreamDestroy(stream);
    own_stream = false;
  }
  if (s) {
    stream = s;
  } else {
    LFQS_CUDA_CHECK(cudaStreamCreateWithFlags(&stream, cudaStreamNonBlocking));
    own_stream = true;
  }
}

LaunchCtx State::ctx(int shard) {
  LaunchCtx c;
  c.amps = amps + 2 * ((uint64_t)shard << n_local);
  c.n_local = n_local;
  c.stream = stream;
  c.launch_counter = &launches;
  c.opt = &opt;
  return c;
}

bool State::identity_map() const {
  for (int q = 0; q < n; ++q)
    if (l2p[q] != q) return false;
  return true;
}

void State::reset_map() {
  for (int q = 0; q < 64; ++q) l2p[q] = p2l[q] = q;
}

void State::init_basis(uint64_t index) {
  DeviceGuard dg(device);
  require(n >= 64 || index < (1ull << n), "basis index out of range");
  reset_map();
  for (int s = 0; s < n_shards(); ++s) {
    const uint64_t lo = (uint64_t)rank_of_shard(s) << n_local;
    const int64_t li = (index >= lo && index - lo < (1ull << n_local)) ? (int64_t)(index - lo) : -1;
    launch_init_basis(ctx(s), li);
  }
}

void State::init_random(uint64_t seed) {
  DeviceGuard dg(device);
  reset_map();
  for (int s = 0; s < n_shards(); ++s)
    launch_init_random(ctx(s), seed, (uint64_t)rank_of_shard(s) << n_local);
}

void State::synchronize() {
  DeviceGuard dg(device);
  LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
  LFQS_CUDA_CHECK(cudaGetLastError());
}

void State::copy(uint64_t offset, uint64_t count, double* host, bool to_device) {
  DeviceGuard dg(device);
  const uint64_t total = 1ull << n;
  require(offset <= total && count <= total - offset, "amplitude range out of bounds");
  if (!identity_map()) canonicalize();
  const uint64_t lo = virt ? 0 : (uint64_t)rank << n_local;
  const uint64_t hi = virt ? total : lo + (1ull << n_local);
  const uint64_t a = std::max(offset, lo), b = std::min(offset + count, hi);
  if (a < b) {
    double* dev = amps + 2 * (a - lo);
    double* h = host + 2 * (a - offset);
    const size_t bytes = (b - a) * 16;
    if (to_device)
      LFQS_CUDA_CHECK(cudaMemcpyAsync(dev, h, bytes, cudaMemcpyHostToDevice, stream));
    else
      LFQS_CUDA_CHECK(cudaMemcpyAsync(h, dev, bytes, cudaMemcpyDeviceToHost, stream));
  }
  LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
}

// ---------------------------------------------------------------------------
// Gates
// ---------------------------------------------------------------------------
Decoded State::to_physical(const Decoded& g) const {
  Decoded pg = g;
  for (int s = 0; s < g.m; ++s) pg.targets[s] = l2p[g.targets[s]];
  uint64_t cm = 0;
  for (int q = 0; q < n; ++q)
    if (g.cmask >> q & 1) cm |= 1ull << l2p[q];
  pg.cmask = cm;
  return pg;
}

bool State::rank_local(const Decoded& pg, int r, Decoded* out) const {
  const uint64_t local_mask = (n_local >= 64) ? ~0ull : ((1ull << n_local) - 1);
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
  for (int i = 0; i < dp * dp; ++i) out->M[i] = cplx{0.0, 0.0};
  bool ones = true;
  for (int j = 0; j < dp; ++j) {
    out->M[j * dp + j] = dd[j];
    ones &= dd[j].re == 1.0 && dd[j].im == 0.0;
  }
  out->cls = ones ? GClass::NOOP : GClass::DIAG;
  out->is_h = false;
  return true;
}

void State::exchange(int l, int g) {
  require(l >= 0 && l < n_local && g >= n_local && g < n, "internal: bad exchange positions");
  const int j = g - n_local;
  if (virt) {
    for (int r = 0; r < world; ++r) {
      if (r >> j & 1) continue;
      const int r2 = r | (1 << j);
      launch_half_swap(ctx(r), l, ((uint64_t)(r2 - r)) << n_local);
    }
  } else {
    const int b = (rank >> j) & 1;
    std::vector<Piece> pieces;
    if (l == n_local - 1) {
      pieces.push_back(Piece{(uint64_t)(1 - b) << (n_local - 1), 1ull << (n_local - 1)});
    } else {
      for (uint64_t hi = 0; hi < (1ull << (n_local - 1 - l)); ++hi)
        pieces.push_back(Piece{(hi << (l + 1)) | ((uint64_t)(1 - b) << l), 1ull << l});
    }
    comm->exchange(amps, pieces, rank ^ (1 << j), stream);
  }
  ++exchanges;
  exchange_bytes += 16ull << (n_local - 1);
  const int qa = p2l[l], qb = p2l[g];
  l2p[qa] = g;
  l2p[qb] = l;
  p2l[l] = qb;
  p2l[g] = qa;
}

void State::swap_local(int a, int b) {
  const int t[2] = {a, b};
  Decoded sw = decode_gate(n_local, LFQS_SWAP, t, 2, 0, nullptr, 0, nullptr);
  for (int s = 0; s < n_shards(); ++s) launch_gate(ctx(s), sw);
  const int qa = p2l[a], qb = p2l[b];
  l2p[qa] = b;
  l2p[qb] = a;
  p2l[a] = qb;
  p2l[b] = qa;
}

void State::canonicalize() {
  for (int q = 0; q < n; ++q) {
    const int P = l2p[q];
    if (P == q) continue;
    const bool pl = P < n_local, ql = q < n_local;
    if (pl && ql) {
      swap_local(P, q);
    } else if (pl != ql) {
      exchange(pl ? P : q, pl ? q : P);
    } else {
      const int L = n_local - 1;  // any local position
      exchange(L, P);
      exchange(L, q);
      exchange(L, P);
    }
  }
}

void State::ensure_local_targets(Decoded& pg) {
  for (int s = 0; s < pg.m; ++s) {
    const int g = pg.targets[s];
    if (g < n_local) continue;
    uint64_t tmask = 0;
    for (int u = 0; u < pg.m; ++u) tmask |= 1ull << pg.targets[u];
    int l = n_local - 1;
    while (l >= 0 && (tmask >> l & 1)) --l;
    require(l >= 0, "internal: no free local qubit");
    exchange(l, g);
    pg.targets[s] = l;
    if (pg.cmask >> l & 1) pg.cmask = (pg.cmask & ~(1ull << l)) | (1ull << g);
  }
}

void State::apply_physical(const Decoded& pg) {
  for (int s = 0; s < n_shards(); ++s) {
    Decoded lg;
    if (rank_local(pg, rank_of_shard(s), &lg)) launch_gate(ctx(s), lg);
  }
}

void State::apply(const Decoded& g) {
  DeviceGuard dg(device);
  if (world == 1) {
    launch_gate(ctx(0), g);
    return;
  }
  Decoded pg = to_physical(g);
  if (pg.cls == GClass::NOOP) return;
  if (pg.cls == GClass::PERM_SWAP && pg.cmask == 0 &&
      (pg.targets[0] >= n_local || pg.targets[1] >= n_local)) {
    // SWAP of logical qubits = relabel: exchange their physical positions in the map.
    const int qa = g.targets[0], qb = g.targets[1];
    std::swap(l2p[qa], l2p[qb]);
    p2l[l2p[qa]] = qa;
    p2l[l2p[qb]] = qb;
    return;
  }
  if (pg.cls != GClass::DIAG) ensure_local_targets(pg);
  apply_physical(pg);
}

void State::run(const std::vector<Decoded>& gates, uint32_t flags) {
  DeviceGuard dg(device);
  if ((flags & LFQS_FUSE_LOW) && world == 1) {
    size_t i = 0;
    while (i < gates.size()) {
      size_t used = 0;
      if (run_fused_circuit(ctx(0), gates, i, gates.size(), opt.fuse_tile_qubits, &used)) {
        i += used;
      } else {
        launch_gate(ctx(0), gates[i]);
        ++i;
      }
    }
    return;
  }
  for (const Decoded& g : gates) apply(g);
}

void State::measure_probs(const int* qubits, int nq, double* out) {
  DeviceGuard dg(device);
  const int nb = 1 << nq;
  if (world == 1) {
    launch_probs(ctx(0), qubits, nq, d_partials, probs_blocks(), d_probs);
    LFQS_CUDA_CHECK(cudaMemcpyAsync(out, d_probs, sizeof(double) * nb, cudaMemcpyDeviceToHost, stream));
    LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
    return;
  }
  int lq[10], ls[10], nl = 0;
  for (int s = 0; s < nq; ++s) {
    const int P = l2p[qubits[s]];
    if (P < n_local) {
      lq[nl] = P;
      ls[nl] = s;
      ++nl;
    }
  }
  std::vector<double> full(nb, 0.0), loc(1 << nl);
  for (int sh = 0; sh < n_shards(); ++sh) {
    const int r = rank_of_shard(sh);
    launch_probs(ctx(sh), lq, nl, d_partials, probs_blocks(), d_probs);
    LFQS_CUDA_CHECK(cudaMemcpyAsync(loc.data(), d_probs, sizeof(double) * (1 << nl),
                                    cudaMemcpyDeviceToHost, stream));
    LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
    int gbits = 0;
    for (int s = 0; s < nq; ++s) {
      const int P = l2p[qubits[s]];
      if (P >= n_local) gbits |= ((r >> (P - n_local)) & 1) << s;
    }
    for (int lb = 0; lb < (1 << nl); ++lb) {
      int v = gbits;
      for (int u = 0; u < nl; ++u) v |= ((lb >> u) & 1) << ls[u];
      full[v] += loc[lb];
    }
  }
  if (!virt && world > 1) {
    LFQS_CUDA_CHECK(cudaMemcpyAsync(comm->d_reduce, full.data(), sizeof(double) * nb,
                                    cudaMemcpyHostToDevice, stream));
    comm->allreduce_sum(comm->d_reduce, nb, stream);
    LFQS_CUDA_CHECK(cudaMemcpyAsync(full.data(), comm->d_reduce, sizeof(double) * nb,
                                    cudaMemcpyDeviceToHost, stream));
    LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
  }
  std::memcpy(out, full.data(), sizeof(double) * nb);
}

}  // namespace lfqs
