// p2p.cu -- peer-memory transport (NEXT-3): CUDA IPC mappings of every rank's
// shard, device-side pairwise / all-rank barriers, the in-place NVLink swap
// and a deterministic rank-ordered sum for measurement (a8).
// See p2p.h for the protocol.  No paper passage covers multi-GPU execution
// (P:551); this is the sharding BASELINE.json's north_star asks for.
#include "p2p.h"

#include <algorithm>
#include <cstring>
#include <string>

namespace lfqs {

namespace {

constexpr uint32_t kMagic = 0x4c465150;  // "LFQP"
constexpr uint64_t kTimeoutNs = 30ull * 1000 * 1000 * 1000;

struct BarrierArgs {
  uint64_t* remote[64];       // the peer's slot for this rank
  const uint64_t* mine[64];   // this rank's slot for the peer
  uint64_t value[64];         // barrier count with that peer (both sides agree)
  int n;
  int* err;
};

__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Thread i: make this GPU's earlier writes visible system-wide, release the count
// into the peer's slot, then wait (bounded) until the peer's count arrives.
__global__ void k_barrier(const BarrierArgs a) {
  const int i = threadIdx.x;
  if (i >= a.n) return;
  __threadfence_system();
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(a.remote[i]), "l"(a.value[i])
               : "memory");
  const uint64_t t0 = global_ns();
  while (true) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(a.mine[i]) : "memory");
    if (v >= a.value[i]) break;
    if (global_ns() - t0 > kTimeoutNs) {
      atomicExch(a.err, 1);
      break;
    }
    __nanosleep(256);
  }
  __threadfence_system();
}

struct SumArgs {
  const double* in[64];
  int world;
};

// out[i] = in_0[i] + in_1[i] + ... (rank order, so every rank gets identical bits).
__global__ void k_sum_ranks(const SumArgs a, double* __restrict__ out, size_t count) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
       i += (size_t)gridDim.x * blockDim.x) {
    double s = a.in[0][i];
    for (int r = 1; r < a.world; ++r) s += a.in[r][i];
    out[i] = s;
  }
}

struct Blob {
  uint32_t magic;
  int32_t rank, world, device, n_local, amp_bytes;
  cudaIpcMemHandle_t shard, aux;
};
static_assert(sizeof(Blob) <= kP2PHandleBytes, "p2p handle blob too large");
static_assert(kP2PHandleBytes == LFQS_P2P_HANDLE_BYTES, "ABI handle size");

}  // namespace

P2P::P2P(int rank_, int world_, int device_) : rank(rank_), world(world_), device(device_) {
  require(world <= 64, "world size must be <= 64");
  LFQS_CUDA_CHECK(cudaMalloc(&aux, aux_bytes()));
  LFQS_CUDA_CHECK(cudaMemset(aux, 0, 4096));
  LFQS_CUDA_CHECK(cudaHostAlloc(&err_host, sizeof(int), cudaHostAllocMapped));
  *err_host = 0;
  LFQS_CUDA_CHECK(cudaHostGetDevicePointer(&err_dev, err_host, 0));
  LFQS_CUDA_CHECK(cudaDeviceSynchronize());
}

P2P::~P2P() {
  if (attached) {
    // Nobody may free a shard a peer could still be reading or writing.
    cudaStream_t s = nullptr;
    if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) == cudaSuccess) {
      try {
        barrier_all(s);
      } catch (...) {
      }
      cudaStreamSynchronize(s);
      cudaStreamDestroy(s);
    }
    for (int r = 0; r < world; ++r) {
      if (r == rank) continue;
      if (peer_amps[r]) cudaIpcCloseMemHandle(peer_amps[r]);
      if (peer_aux[r]) cudaIpcCloseMemHandle(peer_aux[r]);
    }
  }
  if (aux) cudaFree(aux);
  if (err_host) cudaFreeHost(err_host);
}

void P2P::handle(const void* shard, int n_local, int amp_bytes, uint8_t out[kP2PHandleBytes]) const {
  Blob b;
  std::memset(&b, 0, sizeof b);
  b.magic = kMagic;
  b.rank = rank;
  b.world = world;
  b.device = device;
  b.n_local = n_local;
  b.amp_bytes = amp_bytes;
  LFQS_CUDA_CHECK(cudaIpcGetMemHandle(&b.shard, const_cast<void*>(shard)));
  LFQS_CUDA_CHECK(cudaIpcGetMemHandle(&b.aux, aux));
  std::memset(out, 0, kP2PHandleBytes);
  std::memcpy(out, &b, sizeof b);
}

void P2P::attach(unsigned char* own_shard, int n_local, int amp_bytes, const uint8_t* all) {
  require(!attached, "peers already attached");
  require(all != nullptr, "handles is NULL");
  for (int r = 0; r < world; ++r) {
    Blob b;
    std::memcpy(&b, all + (size_t)r * kP2PHandleBytes, sizeof b);
    const std::string who = "p2p handle " + std::to_string(r) + ": ";
    require(b.magic == kMagic, who + "not an lfqs_state_p2p_handle blob");
    require(b.rank == r, who + "handles must be ordered by rank");
    require(b.world == world && b.n_local == n_local && b.amp_bytes == amp_bytes,
            who + "world / qubit count / precision differ between ranks");
    if (r == rank) {
      peer_amps[r] = own_shard;
      peer_aux[r] = aux;
      continue;
    }
    void* p = nullptr;
    LFQS_CUDA_CHECK(cudaIpcOpenMemHandle(&p, b.shard, cudaIpcMemLazyEnablePeerAccess));
    peer_amps[r] = static_cast<unsigned char*>(p);
    LFQS_CUDA_CHECK(cudaIpcOpenMemHandle(&p, b.aux, cudaIpcMemLazyEnablePeerAccess));
    peer_aux[r] = static_cast<unsigned char*>(p);
  }
  attached = true;
}

void P2P::barrier_pair(int peer, cudaStream_t s) {
  require(attached, "p2p state: peers not attached (lfqs_state_p2p_attach)");
  BarrierArgs a;
  std::memset(&a, 0, sizeof a);
  a.remote[0] = reinterpret_cast<uint64_t*>(peer_aux[peer]) + rank;
  a.mine[0] = reinterpret_cast<const uint64_t*>(aux) + peer;
  a.value[0] = ++sent[peer];
  a.n = 1;
  a.err = err_dev;
  k_barrier<<<1, 32, 0, s>>>(a);
  LFQS_CUDA_CHECK(cudaGetLastError());
}

void P2P::barrier_all(cudaStream_t s) {
  require(attached, "p2p state: peers not attached (lfqs_state_p2p_attach)");
  BarrierArgs a;
  std::memset(&a, 0, sizeof a);
  int k = 0;
  for (int r = 0; r < world; ++r) {
    if (r == rank) continue;
    a.remote[k] = reinterpret_cast<uint64_t*>(peer_aux[r]) + rank;
    a.mine[k] = reinterpret_cast<const uint64_t*>(aux) + r;
    a.value[k] = ++sent[r];
    ++k;
  }
  a.n = k;
  a.err = err_dev;
  k_barrier<<<1, 64, 0, s>>>(a);
  LFQS_CUDA_CHECK(cudaGetLastError());
}

void P2P::exchange(const LaunchCtx& ctx, int l, int j, uint64_t chunk, uint64_t v, int ctas) {
  const int partner = rank ^ (1 << j);
  const int b = (rank >> j) & 1;
  const int low = b ? partner : rank, high = b ? rank : partner;
  const int ab = ctx.c64 ? 8 : 16;
  const int nl = ctx.n_local;
  require(l < nl && nl >= 2 && !(chunk >> l & 1) && (chunk >> nl) == 0,
          "internal: exchange position inside the block's fixed bits");
  // Pairs (low[k | 2^l], high[k]) for k with bit l = 0 in the block.  The highest free
  // index bit hb splits them: rank b swaps the pairs whose bit hb equals b.
  int hb = nl - 1;
  while (hb == l || (chunk >> hb & 1)) --hb;
  require(hb >= 1, "internal: no free bit to split the exchange");
  uint64_t fz = 0, fo = 0;
  int i = 0;
  for (int q = 0; q < nl; ++q)
    if (chunk >> q & 1) ((v >> i++ & 1) ? fo : fz) |= 1ull << q;
  (b ? fo : fz) |= 1ull << hb;
  const int64_t d = reinterpret_cast<intptr_t>(peer_amps[high]) -
                    reinterpret_cast<intptr_t>(peer_amps[low]);
  require(d % (2 * ab) == 0, "internal: peer shards are not 32-byte aligned");
  barrier_pair(partner, ctx.stream);  // both blocks are final up to here
  LaunchCtx c = ctx;
  c.amps = peer_amps[low];
  launch_half_swap(c, l, (uint64_t)(d / ab), ctas, fz, fo);
  barrier_pair(partner, ctx.stream);  // both halves swapped before either moves on
}

void P2P::allreduce_sum(double* host, size_t count, cudaStream_t s) {
  require(count <= kP2PReduceDoubles, "reduction too large for the p2p buffer");
  LFQS_CUDA_CHECK(cudaMemcpyAsync(reduce_area(rank), host, count * sizeof(double),
                                  cudaMemcpyHostToDevice, s));
  barrier_all(s);
  SumArgs a;
  std::memset(&a, 0, sizeof a);
  for (int r = 0; r < world; ++r) a.in[r] = reduce_area(r);
  a.world = world;
  const unsigned blocks = (unsigned)std::min<size_t>((count + 255) / 256, 1184);
  k_sum_ranks<<<blocks, 256, 0, s>>>(a, result_area(), count);
  LFQS_CUDA_CHECK(cudaGetLastError());
  barrier_all(s);  // every rank has read every reduce area
  LFQS_CUDA_CHECK(cudaMemcpyAsync(host, result_area(), count * sizeof(double),
                                  cudaMemcpyDeviceToHost, s));
  LFQS_CUDA_CHECK(cudaStreamSynchronize(s));
  check();
}

void P2P::check() const {
  if (*reinterpret_cast<volatile int*>(err_host))
    throw Error(LFQS_ERR_CUDA, "p2p barrier timed out (a peer rank stopped participating)");
}

}  // namespace lfqs
