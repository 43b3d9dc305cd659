// state.cu -- state allocator, shard layout, and executor of the planner's ops
// (components C10 and C12).
//
// One GPU: the map is the identity and every gate is one launch_gate() pass (or
// a fused pass, LFQS_FUSE_LOW).  P = 2^p ranks (NCCL) or P virtual shards in one
// allocation: planner.cpp turns each logical gate into LOCAL ops (specialised per
// rank) and EXCHANGE ops (half-shard swaps: NCCL send/recv, or a device swap
// between virtual shards).  copy_out / copy_in canonicalise the map first;
// measure_probs translates the measured qubits through it (no data movement).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <memory>
#include <string>

#include "comm.h"
#include "p2p.h"
#include "state.h"

namespace lfqs {

// Defined in apply_kernels.cu / fused_kernels.cu.
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

unsigned char* alloc_amps(uint64_t n_amps, int ab) {
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, n_amps * ab);
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    throw Error(LFQS_ERR_OUT_OF_MEMORY,
                "cannot allocate " + std::to_string(n_amps * ab) + " bytes of device memory");
  }
  LFQS_CUDA_CHECK(e);
  return static_cast<unsigned char*>(p);
}
}  // namespace

void State::common_init(int n_, int world_, int device_, cudaStream_t s, bool c64_) {
  c64 = c64_;
  ab = c64 ? 8 : 16;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    throw Error(LFQS_ERR_CUDA, "no CUDA device available (this library has no CPU fallback)");
  }
  require(device_ >= 0 && device_ < ndev, "device index out of range");
  require(world_ >= 1 && log2_exact(world_) >= 0, "world size must be a power of two");
  require(n_ >= 1 && n_ <= 40, "n_qubits must be in [1, 40]");
  plan = Planner(n_, world_);
  n = n_;
  world = world_;
  p = log2_exact(world_);
  n_local = plan.n_local;
  device = device_;
  LFQS_CUDA_CHECK(cudaSetDevice(device));
  if (s) {
    stream = s;
  } else {
    LFQS_CUDA_CHECK(cudaStreamCreateWithFlags(&stream, cudaStreamNonBlocking));
    own_stream = true;
  }
  partials_cap = size_t(148) * 4 * 1024;  // nq <= 10: one 1024-bin histogram per block
  probs_cap = 1024;
  LFQS_CUDA_CHECK(cudaMalloc(&d_partials, sizeof(double) * partials_cap));
  LFQS_CUDA_CHECK(cudaMalloc(&d_probs, sizeof(double) * probs_cap));
}

State* State::create_local(int n, int device, cudaStream_t stream, void* borrowed, bool c64,
                           bool soa) {
  require(n >= 1 && n <= 36, "n_qubits must be in [1, 36] on one GPU");
  std::unique_ptr<State> st(new State());
  st->common_init(n, 1, device, stream, c64);
  st->soa = soa;
  if (borrowed) {
    st->amps = static_cast<unsigned char*>(borrowed);
  } else {
    st->amps = alloc_amps(1ull << n, st->ab);
    st->owned = true;
    st->init_basis(0);
  }
  return st.release();
}

State* State::create_virtual(int n, int world, int device, cudaStream_t stream, bool c64) {
  require(world >= 2, "virtual partition needs world >= 2");
  std::unique_ptr<State> st(new State());
  st->virt = true;
  st->common_init(n, world, device, stream, c64);
  st->amps = alloc_amps(1ull << n, st->ab);
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
  st->amps = alloc_amps(1ull << st->n_local, st->ab);
  st->owned = true;
  if (world > 1) {
    const uint64_t half = (uint64_t)st->ab << (st->n_local - 1);
    st->comm = new Comm(rank, world, uid, std::min<uint64_t>(256ull << 20, half));
  }
  st->init_basis(0);
  return st.release();
}

State* State::create_p2p(int n, int rank, int world, int device, cudaStream_t stream, bool c64) {
  require(world >= 2, "a p2p state needs world >= 2");
  require(rank >= 0 && rank < world, "rank out of range");
  std::unique_ptr<State> st(new State());
  st->common_init(n, world, device, stream, c64);
  st->rank = rank;
  st->amps = alloc_amps(1ull << st->n_local, st->ab);
  st->owned = true;
  st->p2p = new P2P(rank, world, device);
  st->init_basis(0);
  st->synchronize();
  return st.release();
}

void State::p2p_handle(uint8_t* out) {
  require(p2p != nullptr, "not a p2p state");
  DeviceGuard dg(device);
  p2p->handle(amps, n_local, ab, out);
}

void State::p2p_attach(const uint8_t* all) {
  require(p2p != nullptr, "not a p2p state");
  DeviceGuard dg(device);
  p2p->attach(amps, n_local, ab, all);
}

State::~State() {
  if (device >= 0) cudaSetDevice(device);
  if (stream) cudaStreamSynchronize(stream);
  delete comm;
  delete p2p;  // barrier: no peer touches this shard any more
  if (owned && amps) cudaFree(amps);
  if (d_partials) cudaFree(d_partials);
  if (d_probs) cudaFree(d_probs);
  if (own_stream && stream) cudaStreamDestroy(stream);
  if (copy_stream) cudaStreamDestroy(copy_stream);
  if (xstream) cudaStreamDestroy(xstream);
  for (cudaEvent_t e : ev_tail) cudaEventDestroy(e);
  for (cudaEvent_t e : ev_done) cudaEventDestroy(e);
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
  c.amps = amps + ((uint64_t)shard << n_local) * ab;
  c.n_local = n_local;
  c.stream = stream;
  c.launch_counter = &launches;
  c.opt = &opt;
  c.c64 = c64;
  c.soa = soa;
  c.phase_tables = phase_tables;
  c.jit = jit;
  return c;
}

void State::init_basis(uint64_t index) {
  DeviceGuard dg(device);
  require(n >= 64 || index < (1ull << n), "basis index out of range");
  plan.reset();
  for (int s = 0; s < n_shards(); ++s) {
    const uint64_t lo = (uint64_t)rank_of_shard(s) << n_local;
    const int64_t li = (index >= lo && index - lo < (1ull << n_local)) ? (int64_t)(index - lo) : -1;
    launch_init_basis(ctx(s), li);
  }
}

void State::init_random(uint64_t seed) {
  DeviceGuard dg(device);
  plan.reset();
  for (int s = 0; s < n_shards(); ++s)
    launch_init_random(ctx(s), seed, (uint64_t)rank_of_shard(s) << n_local);
}

void State::wait_stream() {
  if (comm)
    comm->wait(stream);
  else
    LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
}

void State::synchronize() {
  DeviceGuard dg(device);
  wait_stream();
  LFQS_CUDA_CHECK(cudaGetLastError());
  if (p2p) p2p->check();
}

void State::copy_raw(uint64_t offset, uint64_t count, void* host, bool to_device) {
  DeviceGuard dg(device);
  const uint64_t total = 1ull << n;
  require(offset <= total && count <= total - offset, "amplitude range out of bounds");
  if (!plan.identity()) canonicalize();
  const uint64_t lo = virt ? 0 : (uint64_t)rank << n_local;
  const uint64_t hi = virt ? total : lo + (1ull << n_local);
  const uint64_t a = std::max(offset, lo), b = std::min(offset + count, hi);
  if (a < b && soa) {
    // interleaved host pairs <-> the two planes: strided 2-D copies
    const size_t es = ab / 2;
    unsigned char* h = static_cast<unsigned char*>(host) + (a - offset) * ab;
    for (int part = 0; part < 2; ++part) {
      unsigned char* dev = amps + ((uint64_t)part << n_local) * es + (a - lo) * es;
      if (to_device)
        LFQS_CUDA_CHECK(cudaMemcpy2DAsync(dev, es, h + part * es, ab, es, b - a,
                                          cudaMemcpyHostToDevice, stream));
      else
        LFQS_CUDA_CHECK(cudaMemcpy2DAsync(h + part * es, ab, dev, es, es, b - a,
                                          cudaMemcpyDeviceToHost, stream));
    }
  } else if (a < b) {
    unsigned char* dev = amps + (a - lo) * ab;
    unsigned char* h = static_cast<unsigned char*>(host) + (a - offset) * ab;
    const size_t bytes = (b - a) * ab;
    if (to_device)
      LFQS_CUDA_CHECK(cudaMemcpyAsync(dev, h, bytes, cudaMemcpyHostToDevice, stream));
    else
      LFQS_CUDA_CHECK(cudaMemcpyAsync(h, dev, bytes, cudaMemcpyDeviceToHost, stream));
  }
  wait_stream();
}

void State::copy(uint64_t offset, uint64_t count, double* host, bool to_device) {
  if (!c64) {
    copy_raw(offset, count, host, to_device);
    return;
  }
  // complex64 state, complex128 host buffer: convert on the host -- only the sub-range
  // this rank owns (a sharded rank's copy leaves the rest of the caller's buffer as it was,
  // in full complex128 precision).  Bounds are checked before anything is allocated.
  const uint64_t total = 1ull << n;
  require(offset <= total && count <= total - offset, "amplitude range out of bounds");
  const uint64_t lo = virt ? 0 : (uint64_t)rank << n_local;
  const uint64_t hi = virt ? total : lo + (1ull << n_local);
  const uint64_t a = std::max(offset, lo), b = std::min(offset + count, hi);
  if (!plan.identity()) {
    DeviceGuard dg(device);
    canonicalize();
  }
  if (a >= b) return;
  double* h = host + 2 * (a - offset);
  const uint64_t cnt = b - a;
  std::vector<float> tmp(2 * cnt);
  if (to_device) {
    for (uint64_t i = 0; i < 2 * cnt; ++i) tmp[i] = (float)h[i];
    copy_raw(a, cnt, tmp.data(), true);
  } else {
    copy_raw(a, cnt, tmp.data(), false);
    for (uint64_t i = 0; i < 2 * cnt; ++i) h[i] = (double)tmp[i];
  }
}

// ---------------------------------------------------------------------------
// Executing planned ops
// ---------------------------------------------------------------------------
void State::exchange_data(int l, int g) {
  const int j = g - n_local;
  if (virt) {
    for (int r = 0; r < world; ++r) {
      if (r >> j & 1) continue;
      const int r2 = r | (1 << j);
      launch_half_swap(ctx(r), l, ((uint64_t)(r2 - r)) << n_local, opt.exchange_ctas);
    }
  } else if (p2p) {
    p2p->exchange(ctx(0), l, j, 0, 0, opt.exchange_ctas);
  } else {
    const int b = (rank >> j) & 1;
    std::vector<Piece> pieces;
    if (l == n_local - 1) {
      pieces.push_back(Piece{(uint64_t)(1 - b) << (n_local - 1), 1ull << (n_local - 1)});
    } else {
      for (uint64_t hi = 0; hi < (1ull << (n_local - 1 - l)); ++hi)
        pieces.push_back(Piece{(hi << (l + 1)) | ((uint64_t)(1 - b) << l), 1ull << l});
    }
    comm->exchange(amps, ab, pieces, rank ^ (1 << j), stream);
  }
  ++exchanges;
  exchange_bytes += (uint64_t)ab << (n_local - 1);
}

// A run of local gates on one shard: fused passes where possible, else one
// class kernel per gate.
void State::run_local(const LaunchCtx& c, const std::vector<Decoded>& gates, bool fuse) {
  if (fuse && opt.fuse_reorder) {
    std::vector<FusedPass> ps;
    plan_fused_schedule(c, gates, opt.fuse_tile_qubits, ps);
    for (const FusedPass& p : ps) launch_fused_pass(c, gates, p);
    passes += ps.size();
    return;
  }
  size_t i = 0;
  while (i < gates.size()) {
    size_t used = 0;
    if (fuse && run_fused_circuit(c, gates, i, gates.size(), opt.fuse_tile_qubits, &used)) {
      i += used;
      ++passes;
    } else {
      launch_gate(c, gates[i]);
      if (gates[i].cls != GClass::NOOP) ++passes;
      ++i;
    }
  }
}

std::vector<Decoded> State::segment(const std::vector<PlanOp>& ops, size_t b, size_t e,
                                    int shard) {
  std::vector<Decoded> seg;
  seg.reserve(e - b);
  for (size_t k = b; k < e; ++k) {
    Decoded lg;
    if (plan.rank_local(ops[k].gate, rank_of_shard(shard), ops[k].gflip, &lg) &&
        lg.cls != GClass::NOOP)
      seg.push_back(lg);
  }
  return seg;
}

std::vector<State::ShardRun> State::plan_run(const std::vector<PlanOp>& ops, size_t b, size_t e,
                                             bool fuse) {
  std::vector<ShardRun> run(n_shards());
  for (int s = 0; s < n_shards(); ++s) {
    ShardRun& r = run[s];
    r.seg = segment(ops, b, e, s);
    if (fuse) {
      plan_fused_schedule(ctx(s), r.seg, opt.fuse_tile_qubits, r.passes);
    } else {  // one pass per gate (LFQS_FUSE_NONE)
      for (size_t i = 0; i < r.seg.size(); ++i) {
        FusedPass ps;
        ps.gate = (int)i;
        uint64_t m = 0;
        for (int t = 0; t < r.seg[i].m; ++t) m |= 1ull << r.seg[i].targets[t];
        ps.qmask = m | r.seg[i].cmask;
        ps.nd_mask = r.seg[i].cls == GClass::DIAG ? 0 : m;
        r.passes.push_back(std::move(ps));
      }
    }
  }
  return run;
}

void State::launch_passes(const std::vector<ShardRun>& run, const std::vector<size_t>& from,
                          const std::vector<size_t>& to, uint64_t chunk, uint64_t v) {
  for (int s = 0; s < n_shards(); ++s) {
    if (from[s] >= to[s]) continue;
    const LaunchCtx x = ctx(s);
    if (chunk == 0 || v == 0) passes += to[s] - from[s];
    for (size_t i = from[s]; i < to[s]; ++i) {
      if (chunk)
        launch_fused_pass_part(x, run[s].seg, run[s].passes[i], chunk, v);
      else
        launch_fused_pass(x, run[s].seg, run[s].passes[i]);
    }
  }
}

int State::overlap_bits() const {
  const int c = opt.exchange_chunk_bits;
  if (world <= 1 || c <= 0 || n_local - c < 4) return 0;
  return c;
}

cudaEvent_t State::part_event(std::vector<cudaEvent_t>& pool, int v) {
  while ((int)pool.size() <= v) {
    cudaEvent_t e = nullptr;
    LFQS_CUDA_CHECK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    pool.push_back(e);
  }
  return pool[v];
}

// Chunk qubits of the exchange ops[ex[k]] (0: run it serially).  The choice depends only
// on the planned ops, never on a rank's own passes, so every rank of a P2P / NCCL state
// picks the same blocks.  Per-gate execution (no fused passes) and the NCCL transport use
// the top c local qubits (contiguous blocks, single-gate passes can run on them; NCCL
// sends each block's pieces).  Fused execution on the device / P2P transports picks the
// c positions among the local qubits at or above the tile size (a fused pass holds such a
// qubit in its tile only when it mixes it, fused_kernels.cu) that stay unmixed longest
// around the exchange: the most ops before it (back to the previous exchange) plus after
// it (to the next one) free of non-diagonal gates on them; the previous exchange's chunk
// qubits win when the whole run between the two leaves them unmixed (the run then runs
// block by block between the two exchanges' parts: a pipeline, state.cu execute).
uint64_t State::choose_chunk(const std::vector<PlanOp>& ops, const std::vector<size_t>& ex,
                             size_t k, bool fuse, uint64_t prev) const {
  const int c = overlap_bits();
  if (c == 0) return 0;
  const PlanOp& X = ops[ex[k]];
  const uint64_t top = ((1ull << c) - 1) << (n_local - c);
  const bool strided = fuse && (virt || p2p) && opt.exchange_chunk_select;
  if (!strided) return (top >> X.l & 1) ? 0 : top;
  const size_t b = k > 0 ? ex[k - 1] + 1 : 0, e = k + 1 < ex.size() ? ex[k + 1] : ops.size();
  auto mixed = [&](const PlanOp& o) -> uint64_t {
    uint64_t m = 0;
    if (o.kind == PlanOp::EXCHANGE) return ~0ull;
    if (o.gate.cls != GClass::DIAG && o.gate.cls != GClass::NOOP)
      for (int t = 0; t < o.gate.m; ++t) m |= 1ull << o.gate.targets[t];
    return m;
  };
  uint64_t run_mixed = 0;  // mixed by the run between the previous exchange and this one
  for (size_t i = b; i < ex[k]; ++i) run_mixed |= mixed(ops[i]);
  if (prev && !(prev >> X.l & 1) && !(run_mixed & prev)) return prev;
  const int lo = std::max(opt.fuse_tile_qubits, 1);
  if (n_local - lo < c + 1) return (top >> X.l & 1) ? 0 : top;
  // ops before / after the exchange free of mixing, per position
  int before[64], after[64];
  for (int q = 0; q < 64; ++q) before[q] = after[q] = 0;
  uint64_t seen = 0;
  for (size_t i = ex[k]; i-- > b;) {
    const uint64_t m = mixed(ops[i]);
    seen |= m;
    for (int q = lo; q < n_local; ++q)
      if (!(seen >> q & 1)) ++before[q];
  }
  seen = 0;
  for (size_t i = ex[k] + 1; i < e; ++i) {
    const uint64_t m = mixed(ops[i]);
    seen |= m;
    for (int q = lo; q < n_local; ++q)
      if (!(seen >> q & 1)) ++after[q];
  }
  std::vector<int> cand;
  for (int q = lo; q < n_local; ++q)
    if (q != X.l) cand.push_back(q);
  uint64_t best = 0;
  long best_score = -1;
  auto consider = [&](uint64_t m) {
    int tb = 1 << 30, ta = 1 << 30;
    for (int q = 0; q < 64; ++q)
      if (m >> q & 1) tb = std::min(tb, before[q]), ta = std::min(ta, after[q]);
    const long sc = (long)tb + ta;
    // ties: the top qubits (the contiguous blocks of the serial planner), then higher ones
    if (sc > best_score || (sc == best_score && (m == top || (best != top && m > best)))) {
      best = m;
      best_score = sc;
    }
  };
  const int nc = (int)cand.size();
  for (int i0 = 0; i0 < nc; ++i0) {
    const uint64_t m0 = 1ull << cand[i0];
    if (c == 1) { consider(m0); continue; }
    for (int i1 = i0 + 1; i1 < nc; ++i1) {
      const uint64_t m1 = m0 | 1ull << cand[i1];
      if (c == 2) { consider(m1); continue; }
      for (int i2 = i1 + 1; i2 < nc; ++i2) consider(m1 | 1ull << cand[i2]);
    }
  }
  return best;
}

cudaEvent_t State::exchange_part(int l, int g, uint64_t chunk, uint64_t v, cudaEvent_t ready) {
  const int j = g - n_local;
  if (virt || p2p) {
    if (xstream == nullptr) {
      // highest priority: the link transfer is on the critical path, so its CTAs are
      // dispatched ahead of the compute stream's pending tiles
      int lo = 0, hi = 0;
      LFQS_CUDA_CHECK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
      LFQS_CUDA_CHECK(cudaStreamCreateWithPriority(&xstream, cudaStreamNonBlocking, hi));
    }
    LFQS_CUDA_CHECK(cudaStreamWaitEvent(xstream, ready, 0));
    uint64_t fz = 0, fo = 0;
    int i = 0;
    for (int q = 0; q < n_local; ++q)
      if (chunk >> q & 1) ((v >> i++ & 1) ? fo : fz) |= 1ull << q;
    if (virt) {
      for (int r = 0; r < world; ++r) {
        if (r >> j & 1) continue;
        const int r2 = r | (1 << j);
        LaunchCtx x = ctx(r);
        x.stream = xstream;
        launch_half_swap(x, l, ((uint64_t)(r2 - r)) << n_local, opt.exchange_ctas, fz, fo);
      }
    } else {
      LaunchCtx x = ctx(0);
      x.stream = xstream;
      p2p->exchange(x, l, j, chunk, v, opt.exchange_ctas);
    }
    cudaEvent_t done = part_event(ev_done, (int)v);
    LFQS_CUDA_CHECK(cudaEventRecord(done, xstream));
    return done;
  }
  // NCCL: the top c local qubits (choose_chunk); this part's half (local bit l = 1 - own
  // global bit) as contiguous pieces.
  const int c = __builtin_popcountll(chunk), ns = n_local - c;
  require(chunk == ((1ull << c) - 1) << ns, "internal: NCCL exchange blocks must be the top qubits");
  const uint64_t off = v << ns;
  const int b = (rank >> j) & 1;
  std::vector<Piece> pieces;
  if (l == ns - 1) {
    pieces.push_back(Piece{off + ((uint64_t)(1 - b) << (ns - 1)), 1ull << (ns - 1)});
  } else {
    for (uint64_t hi = 0; hi < (1ull << (ns - 1 - l)); ++hi)
      pieces.push_back(Piece{off + ((hi << (l + 1)) | ((uint64_t)(1 - b) << l)), 1ull << l});
  }
  comm->exchange(amps, ab, pieces, rank ^ (1 << j), stream, ready);
  return nullptr;
}

// Executes planned ops: maximal runs of LOCAL ops are rank-specialised per shard and
// planned into passes (fused if requested); EXCHANGE ops move data between shards.
//
// Global-qubit exchange overlapped with local work (BASELINE north_star
// "overlapped with local work on separate streams"), Options::exchange_chunk_bits = c > 0:
// an exchange at local position l moves data only inside each block of the state whose c
// chunk qubits (choose_chunk; never l) hold fixed values, so it splits into 2^c
// independent parts.  The trailing passes of the run before it that do not mix the chunk
// qubits run part by part on the compute stream; part v moves (exchange stream, or the
// NCCL stream) as soon as its tail is done, while the compute stream goes on with the
// next part; the leading passes of the next run that do not mix them run on part v as
// soon as it has landed.  When those leading passes are the whole run and the next
// exchange uses the same chunk qubits, its part v starts as soon as part v's run is done
// (a pipeline across consecutive exchanges).  A pass "mixes" a qubit when a non-diagonal
// gate targets it; controls and diagonal entries on the chunk qubits are resolved per
// part (fused passes take them as fixed bits of the tile index; single gates are
// specialised on the host), so e.g. every QFT CPhase pass can run part by part.  The
// passes are exactly the ones the serial execution launches (no extra HBM pass), each
// applied block by block with the same kernels, and every pass sees the data it would see
// in the serial order (Eq. 3; ops on disjoint blocks commute): results are
// bit-identical to serial exchanges (tests/test_gpu_overlap.py, tests/test_gpu_p2p.py).
void State::execute(const std::vector<PlanOp>& ops, bool fuse) {
  std::vector<size_t> ex;
  for (size_t i = 0; i < ops.size(); ++i)
    if (ops[i].kind == PlanOp::EXCHANGE) ex.push_back(i);
  if (fuse && !opt.fuse_reorder) {  // prefix fusion (a tuning mode): serial, run by run
    size_t i = 0;
    for (size_t k = 0; k <= ex.size(); ++k) {
      const size_t e = k < ex.size() ? ex[k] : ops.size();
      for (int s = 0; s < n_shards(); ++s) run_local(ctx(s), segment(ops, i, e, s), true);
      if (k < ex.size()) exchange_data(ops[e].l, ops[e].g);
      i = e + 1;
    }
    return;
  }
  const int S = n_shards();
  std::vector<ShardRun> cur = plan_run(ops, 0, ex.empty() ? ops.size() : ex[0], fuse);
  std::vector<size_t> from(S, 0), end(S);
  // chunk qubits of the previous exchange (0: serial).  choose_chunk keeps them when the
  // planned ops in between leave them unmixed -- a rank-independent decision (P2P ranks
  // must pick the same blocks); whether this rank's passes in between all ran block by
  // block (so the exchanges chain) is a local scheduling matter.
  uint64_t prev = 0;
  bool prev_whole = false;  // the previous exchange's leading passes were its whole run
  for (size_t k = 0;; ++k) {
    for (int s = 0; s < S; ++s) end[s] = cur[s].passes.size();
    if (k == ex.size()) {
      launch_passes(cur, from, end, 0, 0);
      break;
    }
    const PlanOp& X = ops[ex[k]];
    const size_t nb = ex[k] + 1, ne = k + 1 < ex.size() ? ex[k + 1] : ops.size();
    std::vector<ShardRun> next = plan_run(ops, nb, ne, fuse);
    const uint64_t chunk = choose_chunk(ops, ex, k, fuse, prev);
    NvtxRange nv(chunk ? "lfqs_exchange_overlapped" : "lfqs_exchange");
    if (chunk == 0) {
      launch_passes(cur, from, end, 0, 0);
      exchange_data(X.l, X.g);
      cur = std::move(next);
      std::fill(from.begin(), from.end(), 0);
      prev = 0;
      prev_whole = false;
      continue;
    }
    // tail: trailing passes that do not mix the chunk qubits; head: leading ones of the
    // next run
    std::vector<size_t> ts(S), he(S, 0), zero(S, 0);
    bool chained = prev == chunk && prev_whole, whole = true;
    for (int s = 0; s < S; ++s) {
      ts[s] = end[s];
      while (ts[s] > from[s] && pass_blockwise(cur[s].passes[ts[s] - 1], chunk, n_local)) --ts[s];
      while (he[s] < next[s].passes.size() && pass_blockwise(next[s].passes[he[s]], chunk, n_local))
        ++he[s];
      chained &= from[s] == end[s];
      whole &= he[s] == next[s].passes.size();
    }
    const int parts = 1 << __builtin_popcountll(chunk);
    if (!chained) {
      // (chained: the whole run between the previous exchange and this one already ran
      // part by part, each part's ev_tail recorded after it)
      launch_passes(cur, from, ts, 0, 0);  // the body of the run
      for (int v = 0; v < parts; ++v) {
        launch_passes(cur, ts, end, chunk, (uint64_t)v);
        LFQS_CUDA_CHECK(cudaEventRecord(part_event(ev_tail, v), stream));
      }
    }
    for (int v = 0; v < parts; ++v) {
      cudaEvent_t done = exchange_part(X.l, X.g, chunk, (uint64_t)v, part_event(ev_tail, v));
      if (done) LFQS_CUDA_CHECK(cudaStreamWaitEvent(stream, done, 0));
      launch_passes(next, zero, he, chunk, (uint64_t)v);
      if (whole) LFQS_CUDA_CHECK(cudaEventRecord(part_event(ev_tail, v), stream));
    }
    ++exchanges;
    exchange_bytes += (uint64_t)ab << (n_local - 1);
    ++ov_exchanges;
    for (int s = 0; s < S; ++s) ov_block_passes += (end[s] - ts[s]) + he[s];
    const int c = __builtin_popcountll(chunk);
    ov_strided += chunk != ((1ull << c) - 1) << (n_local - c);
    ov_chained += chained;
    prev = chunk;
    prev_whole = whole;
    cur = std::move(next);
    from = he;
  }
}

// The canonicalising ops are local SWAP passes (and X passes for global flips) between
// exchanges: moves only, so they run fused (LFQS_OPT_CANON_FUSE, default 1) -- runs of
// SWAPs share one tile pass, bit-identical to one pass per SWAP, and the exchanges between
// them may take strided chunk qubits and overlap with them (QFT(33) on 8 ranks: 8 SWAP
// passes -> 3).  The interpreting kernel runs them (no compiled passes outside a run).
void State::plan_window() {
  plan.swap_lo = (opt.exchange_wide && (virt || p2p)) ? std::min(3, n_local - 1) : -1;
}

void State::canonicalize() {
  NvtxRange nv("lfqs_canonicalize");
  std::vector<PlanOp> ops;
  plan_window();
  plan.plan_canonicalize(ops);
  struct Restore {  // the run's pass-compiler flags, also when execute throws
    bool &j, &pt;
    const bool j0, pt0;
    ~Restore() {
      j = j0;
      pt = pt0;
    }
  } restore{jit, phase_tables, jit, phase_tables};
  jit = phase_tables = false;
  execute(ops, opt.canon_fuse && !soa);
}

void State::apply(const Decoded& g) {
  DeviceGuard dg(device);
  if (world == 1) {
    launch_gate(ctx(0), g);
    if (g.cls != GClass::NOOP) ++passes;
    return;
  }
  std::vector<PlanOp> ops;
  plan_window();
  plan.plan_gate(g, ops);
  execute(ops, false);
}

void State::run(const std::vector<Decoded>& gates, uint32_t flags) {
  DeviceGuard dg(device);
  NvtxRange nv("lfqs_run_circuit");
  const bool fuse = (flags & LFQS_FUSE_LOW) != 0;
  if (fuse && soa)
    throw Error(LFQS_ERR_UNSUPPORTED, "fused passes need an AOS state (LFQS_STATE_SOA is per-gate only)");
  phase_tables = fuse && (flags & LFQS_FUSE_PHASE) != 0;
  jit = fuse && (flags & LFQS_FUSE_JIT) != 0;
  struct Reset {
    bool& f;
    bool& g;
    ~Reset() { f = g = false; }
  } reset{phase_tables, jit};
  if (world == 1) {
    run_local(ctx(0), gates, fuse);
    return;
  }
  std::vector<PlanOp> ops;
  plan_window();
  plan.plan_circuit(gates, ops);  // Belady lookahead over the whole circuit
  execute(ops, fuse);
}

// Upload overlapped with computation (lfqs_run_circuit_streamed).  The state is split by
// its top chunk_bits qubits into pieces of 2^(n - chunk_bits) amplitudes.  Every gate of
// the longest circuit prefix whose targets and controls all lie below n - chunk_bits acts
// inside each piece independently (G = I (x) G' on the piece index, Eq. 1), so piece c
// runs that prefix as soon as its copy has landed -- with the same kernels and the same
// per-amplitude arithmetic as on the whole state -- while later pieces are still in flight;
// the rest of the circuit then runs on the whole state.  Without fusion bit-identical to
// copy_in + run; fused, the prefix and the rest form separate passes (rounding only).
void State::run_streamed(const void* host, const std::vector<Decoded>& gates, uint32_t flags,
                         int chunk_bits) {
  NvtxRange nv("lfqs_run_circuit_streamed");
  DeviceGuard dg(device);
  require(!virt && !soa, "streamed runs need an AOS state on one GPU or one shard per rank");
  require(chunk_bits >= 0 && chunk_bits <= 8 && chunk_bits < n_local,
          "chunk_bits must be in [0, 8] and below the local qubit count");
  const bool fuse = (flags & LFQS_FUSE_LOW) != 0;
  const int nl = n_local - chunk_bits;
  plan.reset();  // the whole (local) state is overwritten: canonical qubit map
  size_t pre = 0;
  for (; pre < gates.size(); ++pre) {
    if (opt.stream_max_prefix > 0 && pre >= (size_t)opt.stream_max_prefix) break;
    uint64_t m = gates[pre].cmask;
    for (int s = 0; s < gates[pre].m; ++s) m |= 1ull << gates[pre].targets[s];
    if (m >> nl) break;
  }
  if (copy_stream == nullptr)
    LFQS_CUDA_CHECK(cudaStreamCreateWithFlags(&copy_stream, cudaStreamNonBlocking));
  const int pieces = 1 << chunk_bits;
  const size_t piece_bytes = (size_t)ab << nl;
  std::vector<cudaEvent_t> ev(pieces, nullptr);
  struct Events {
    std::vector<cudaEvent_t>& e;
    ~Events() {
      for (cudaEvent_t x : e)
        if (x) cudaEventDestroy(x);
    }
  } guard{ev};
  // the copies must not overtake work already queued on the state's stream
  cudaEvent_t start = nullptr;
  LFQS_CUDA_CHECK(cudaEventCreateWithFlags(&start, cudaEventDisableTiming));
  ev.push_back(start);
  LFQS_CUDA_CHECK(cudaEventRecord(start, stream));
  LFQS_CUDA_CHECK(cudaStreamWaitEvent(copy_stream, start, 0));
  phase_tables = fuse && (flags & LFQS_FUSE_PHASE) != 0;
  jit = fuse && (flags & LFQS_FUSE_JIT) != 0;
  struct Reset {
    bool& f;
    bool& g;
    ~Reset() { f = g = false; }
  } reset{phase_tables, jit};
  const std::vector<Decoded> prefix(gates.begin(), gates.begin() + pre);
  for (int c = 0; c < pieces; ++c) {
    LFQS_CUDA_CHECK(cudaEventCreateWithFlags(&ev[c], cudaEventDisableTiming));
    LFQS_CUDA_CHECK(cudaMemcpyAsync(amps + (size_t)c * piece_bytes,
                                    static_cast<const unsigned char*>(host) + (size_t)c * piece_bytes,
                                    piece_bytes, cudaMemcpyHostToDevice, copy_stream));
    LFQS_CUDA_CHECK(cudaEventRecord(ev[c], copy_stream));
  }
  for (int c = 0; c < pieces; ++c) {
    LFQS_CUDA_CHECK(cudaStreamWaitEvent(stream, ev[c], 0));
    if (prefix.empty()) continue;
    LaunchCtx pc = ctx(0);
    pc.amps = amps + (size_t)c * piece_bytes;
    pc.n_local = nl;
    run_local(pc, prefix, fuse);
  }
  const std::vector<Decoded> rest(gates.begin() + pre, gates.end());
  if (rest.empty()) return;
  if (world == 1) {
    run_local(ctx(0), rest, fuse);
  } else {
    std::vector<PlanOp> ops;
    plan_window();
    plan.plan_circuit(rest, ops);  // exchanges for the global qubits, as in run()
    execute(ops, fuse);
  }
}

Graph* State::compile(const std::vector<Decoded>& gates, uint32_t flags) {
  DeviceGuard dg(device);
  if (comm != nullptr || p2p != nullptr)
    throw Error(LFQS_ERR_UNSUPPORTED, "circuit capture of a multi-process (NCCL / p2p) state");
  if (!plan.identity()) canonicalize();  // eager: the graph starts from the canonical map
  cudaStream_t cs = nullptr;
  LFQS_CUDA_CHECK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  const cudaStream_t saved = stream;
  const uint64_t launches0 = launches, ex0 = exchanges, exb0 = exchange_bytes;
  stream = cs;
  cudaGraph_t graph = nullptr;
  LFQS_CUDA_CHECK(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
  try {
    run(gates, flags);
    if (!plan.identity()) canonicalize();  // the graph ends canonical: replays compose
  } catch (...) {
    cudaStreamEndCapture(cs, &graph);
    if (graph) cudaGraphDestroy(graph);
    stream = saved;
    plan.reset();
    launches = launches0;
    cudaStreamDestroy(cs);
    throw;
  }
  stream = saved;
  const cudaError_t e = cudaStreamEndCapture(cs, &graph);
  cudaStreamDestroy(cs);
  LFQS_CUDA_CHECK(e);
  std::unique_ptr<Graph> g(new Graph);
  g->st = this;
  g->kernels = launches - launches0;
  launches = launches0;  // nothing ran yet
  exchanges = ex0;
  exchange_bytes = exb0;
  const cudaError_t ei = cudaGraphInstantiate(&g->exec, graph, 0);
  cudaGraphDestroy(graph);
  LFQS_CUDA_CHECK(ei);
  return g.release();
}

void Graph::launch() {
  DeviceGuard dg(st->device);
  LFQS_CUDA_CHECK(cudaGraphLaunch(exec, st->stream));
  st->launches += kernels;
}

Graph::~Graph() {
  if (exec) cudaGraphExecDestroy(exec);
}

void State::collapse(const int* qubits, int nq, uint64_t outcome, double scale) {
  DeviceGuard dg(device);
  for (int sh = 0; sh < n_shards(); ++sh) {
    const int r = rank_of_shard(sh);
    uint64_t mask = 0, pat = 0;
    bool rank_matches = true;
    for (int s = 0; s < nq; ++s) {
      const int P = plan.l2p[qubits[s]];
      const uint64_t bit = (outcome >> s) & 1;
      if (P < n_local) {
        mask |= 1ull << P;
        pat |= bit << P;
      } else if ((uint64_t)plan.global_bit(r, P, plan.gflip) != bit) {
        rank_matches = false;
      }
    }
    launch_collapse(ctx(sh), mask, pat, rank_matches ? scale : 0.0, !rank_matches);
  }
}

// Probabilities of the local physical qubits lq[0..nl) of one shard into host[2^nl]
// (bit u of the bin = bit lq[u]): one read pass (two-level binning, reduce_kernels.cu).
void State::local_probs(int shard, const int* lq, int nl, double* host) {
  const size_t need = probs_partials_doubles(n_local, lq, nl);
  auto grow = [&](double*& p, size_t& cap, size_t want) {
    if (cap >= want) return;
    LFQS_CUDA_CHECK(cudaStreamSynchronize(stream));
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    LFQS_CUDA_CHECK(cudaMalloc(&p, sizeof(double) * want));
    cap = want;
  };
  grow(d_partials, partials_cap, need);
  grow(d_probs, probs_cap, size_t(1) << nl);
  launch_probs(ctx(shard), lq, nl, d_partials, partials_cap, d_probs);
  LFQS_CUDA_CHECK(cudaMemcpyAsync(host, d_probs, sizeof(double) << nl, cudaMemcpyDeviceToHost,
                                  stream));
  wait_stream();
}

void State::measure_probs(const int* qubits, int nq, double* out) {
  NvtxRange nv("lfqs_measure_probs");
  DeviceGuard dg(device);
  const size_t nb = size_t(1) << nq;
  if (world == 1) {
    local_probs(0, qubits, nq, out);
    return;
  }
  int lq[64], ls[64], nl = 0;
  for (int s = 0; s < nq; ++s) {
    const int P = plan.l2p[qubits[s]];
    if (P < n_local) {
      lq[nl] = P;
      ls[nl] = s;
      ++nl;
    }
  }
  std::vector<double> full(nb, 0.0), loc(size_t(1) << nl);
  for (int sh = 0; sh < n_shards(); ++sh) {
    const int r = rank_of_shard(sh);
    local_probs(sh, lq, nl, loc.data());
    uint64_t gbits = 0;
    for (int s = 0; s < nq; ++s) {
      const int P = plan.l2p[qubits[s]];
      if (P >= n_local) gbits |= (uint64_t)plan.global_bit(r, P, plan.gflip) << s;
    }
    for (uint64_t lb = 0; lb < (1ull << nl); ++lb) {
      uint64_t v = gbits;
      for (int u = 0; u < nl; ++u) v |= ((lb >> u) & 1ull) << ls[u];
      full[v] += loc[lb];
    }
  }
  if (p2p) {
    p2p->allreduce_sum(full.data(), nb, stream);
  } else if (!virt && world > 1) {
    double* d = comm->d_reduce;
    if (nb > 1024) LFQS_CUDA_CHECK(cudaMalloc(&d, sizeof(double) * nb));
    LFQS_CUDA_CHECK(cudaMemcpyAsync(d, full.data(), sizeof(double) * nb, cudaMemcpyHostToDevice,
                                    stream));
    comm->allreduce_sum(d, nb, stream);
    LFQS_CUDA_CHECK(cudaMemcpyAsync(full.data(), d, sizeof(double) * nb, cudaMemcpyDeviceToHost,
                                    stream));
    wait_stream();
    if (d != comm->d_reduce) cudaFree(d);
  }
  std::memcpy(out, full.data(), sizeof(double) * nb);
}

}  // namespace lfqs
