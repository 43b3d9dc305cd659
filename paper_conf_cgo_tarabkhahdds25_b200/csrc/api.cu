// api.cu -- the C ABI (include/lfqs.h): state lifetime, gates, circuits, measurement.
//
// The ABI follows the paper's statement of the problem: an n-qubit state
// (P:93-101), a circuit G_D ... G_1 applied gate by gate (Eq. 3) with the
// state available after each gate, updated in place in AOS
// complex layout, then measured.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <memory>
#include <string>
#include <vector>

#include "lfqs_internal.h"
#include "planner.h"
#include "state.h"

using namespace lfqs;

namespace {
thread_local std::string g_last_error;

template <class F>
lfqs_status guarded(F&& f) {
  try {
    f();
    return LFQS_OK;
  } catch (const Error& e) {
    g_last_error = e.what();
    return e.status;
  } catch (const std::bad_alloc&) {
    g_last_error = "host out of memory";
    return LFQS_ERR_OUT_OF_MEMORY;
  } catch (const std::exception& e) {
    g_last_error = e.what();
    return LFQS_ERR_INVALID_ARG;
  } catch (...) {
    g_last_error = "unknown error";
    return LFQS_ERR_INVALID_ARG;
  }
}

// Borrowed buffers must be aligned for the widest access any kernel issues: two adjacent
// amplitudes per vector access (ld/st.global.v4: 32 B complex128, 16 B complex64) and TMA
// bulk copies (cp.async.bulk, 16 B).  A merely element-aligned torch view (e.g. t[1:]) is
// rejected here instead of faulting with a misaligned address inside a kernel.
void require_wrap_alignment(const void* p, bool c64) {
  const uintptr_t need = c64 ? 16 : 32;
  require((reinterpret_cast<uintptr_t>(p) & (need - 1)) == 0,
          std::string("dev_ptr must be ") + (c64 ? "16" : "32") +
              "-byte aligned (two amplitudes per vector access)");
}

uint64_t mask_of(const int* qs, int nq, int n) {
  uint64_t m = 0;
  require(nq >= 0 && (nq == 0 || qs != nullptr), "bad control list");
  for (int i = 0; i < nq; ++i) {
    require(qs[i] >= 0 && qs[i] < n, "control qubit out of range");
    require(!(m >> qs[i] & 1), "duplicate control qubit");
    m |= 1ull << qs[i];
  }
  return m;
}
}  // namespace

extern "C" {

const char* lfqs_last_error(void) { return g_last_error.c_str(); }
int lfqs_abi_version(void) { return LFQS_ABI_VERSION; }

lfqs_status lfqs_state_create(int n_qubits, int device, void* stream, lfqs_state** out) {
  return guarded([&] {
    require(out != nullptr, "out is NULL");
    *out = State::create_local(n_qubits, device, static_cast<cudaStream_t>(stream), nullptr);
  });
}

lfqs_status lfqs_state_wrap(int n_qubits, int device, void* dev_ptr, void* stream,
                            lfqs_state** out) {
  return guarded([&] {
    require(out != nullptr && dev_ptr != nullptr, "NULL argument");
    require_wrap_alignment(dev_ptr, false);
    *out = State::create_local(n_qubits, device, static_cast<cudaStream_t>(stream), dev_ptr);
  });
}

lfqs_status lfqs_state_create_ex(int n_qubits, int world, int device, void* stream,
                                 uint32_t flags, lfqs_state** out) {
  return guarded([&] {
    require(out != nullptr, "out is NULL");
    require((flags & ~(LFQS_STATE_C64 | LFQS_STATE_SOA)) == 0, "unknown state flags");
    const bool c64 = (flags & LFQS_STATE_C64) != 0, soa = (flags & LFQS_STATE_SOA) != 0;
    if (soa && world > 1)
      throw Error(LFQS_ERR_UNSUPPORTED, "LFQS_STATE_SOA states are single-shard");
    if (world <= 1)
      *out = State::create_local(n_qubits, device, static_cast<cudaStream_t>(stream), nullptr, c64,
                                 soa);
    else
      *out = State::create_virtual(n_qubits, world, device, static_cast<cudaStream_t>(stream), c64);
  });
}

lfqs_status lfqs_state_wrap_ex(int n_qubits, int device, void* dev_ptr, void* stream,
                               uint32_t flags, lfqs_state** out) {
  return guarded([&] {
    require(out != nullptr && dev_ptr != nullptr, "NULL argument");
    require((flags & ~(LFQS_STATE_C64 | LFQS_STATE_SOA)) == 0, "unknown state flags");
    const bool c64 = (flags & LFQS_STATE_C64) != 0, soa = (flags & LFQS_STATE_SOA) != 0;
    require_wrap_alignment(dev_ptr, c64);
    *out = State::create_local(n_qubits, device, static_cast<cudaStream_t>(stream), dev_ptr, c64,
                               soa);
  });
}

lfqs_status lfqs_copy_in_c64(lfqs_state* s, uint64_t offset, uint64_t count, const float* host) {
  return guarded([&] {
    require(s != nullptr && (count == 0 || host != nullptr), "NULL argument");
    State* st = static_cast<State*>(s);
    require(st->c64, "not a complex64 state");
    st->copy_raw(offset, count, const_cast<float*>(host), true);
  });
}

lfqs_status lfqs_copy_out_c64(lfqs_state* s, uint64_t offset, uint64_t count, float* host) {
  return guarded([&] {
    require(s != nullptr && (count == 0 || host != nullptr), "NULL argument");
    State* st = static_cast<State*>(s);
    require(st->c64, "not a complex64 state");
    st->copy_raw(offset, count, host, false);
  });
}

lfqs_status lfqs_state_create_virtual(int n_qubits, int world, int device, void* stream,
                                      lfqs_state** out) {
  return guarded([&] {
    require(out != nullptr, "out is NULL");
    *out = State::create_virtual(n_qubits, world, device, static_cast<cudaStream_t>(stream));
  });
}

lfqs_status lfqs_dist_unique_id(uint8_t uid[128]) {
  return guarded([&] {
    require(uid != nullptr, "uid is NULL");
    State::nccl_unique_id(uid);
  });
}

lfqs_status lfqs_state_create_dist(int n_qubits, int rank, int world, const uint8_t uid[128],
                                   int device, void* stream, lfqs_state** out) {
  return guarded([&] {
    require(out != nullptr && uid != nullptr, "NULL argument");
    *out = State::create_dist(n_qubits, rank, world, uid, device, static_cast<cudaStream_t>(stream));
  });
}

lfqs_status lfqs_state_create_p2p(int n_qubits, int rank, int world, int device, void* stream,
                                  uint32_t flags, lfqs_state** out) {
  return guarded([&] {
    require(out != nullptr, "out is NULL");
    require((flags & ~(uint32_t)LFQS_STATE_C64) == 0, "unknown flags");
    *out = State::create_p2p(n_qubits, rank, world, device, static_cast<cudaStream_t>(stream),
                             (flags & LFQS_STATE_C64) != 0);
  });
}

lfqs_status lfqs_state_p2p_handle(lfqs_state* s, uint8_t* blob) {
  return guarded([&] {
    require(s != nullptr && blob != nullptr, "NULL argument");
    static_cast<State*>(s)->p2p_handle(blob);
  });
}

lfqs_status lfqs_state_p2p_attach(lfqs_state* s, const uint8_t* all_blobs) {
  return guarded([&] {
    require(s != nullptr && all_blobs != nullptr, "NULL argument");
    static_cast<State*>(s)->p2p_attach(all_blobs);
  });
}

lfqs_status lfqs_state_destroy(lfqs_state* s) {
  return guarded([&] { delete static_cast<State*>(s); });
}

lfqs_status lfqs_state_set_stream(lfqs_state* s, void* stream) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    static_cast<State*>(s)->set_stream(static_cast<cudaStream_t>(stream));
  });
}

lfqs_status lfqs_state_init_basis(lfqs_state* s, uint64_t index) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    static_cast<State*>(s)->init_basis(index);
  });
}

lfqs_status lfqs_state_init_random(lfqs_state* s, uint64_t seed) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    static_cast<State*>(s)->init_random(seed);
  });
}

lfqs_status lfqs_copy_in(lfqs_state* s, uint64_t offset, uint64_t count, const double* host) {
  return guarded([&] {
    require(s != nullptr && (count == 0 || host != nullptr), "NULL argument");
    static_cast<State*>(s)->copy(offset, count, const_cast<double*>(host), /*to_device=*/true);
  });
}

lfqs_status lfqs_copy_out(lfqs_state* s, uint64_t offset, uint64_t count, double* host) {
  return guarded([&] {
    require(s != nullptr && (count == 0 || host != nullptr), "NULL argument");
    static_cast<State*>(s)->copy(offset, count, host, /*to_device=*/false);
  });
}

lfqs_status lfqs_apply_gate(lfqs_state* s, int kind, const int* targets, int n_targets,
                            const int* controls, int n_controls, const double* params,
                            int n_params, const double* matrix) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    State* st = static_cast<State*>(s);
    require(n_targets >= 1 && n_targets <= 3 && targets != nullptr, "bad target list");
    require(n_params == 0 || params != nullptr, "params is NULL");
    const uint64_t cm = mask_of(controls, n_controls, st->n);
    Decoded g = decode_gate(st->n, kind, targets, n_targets, cm, params, n_params, matrix);
    st->apply(g);
  });
}

namespace {
std::vector<Decoded> decode_circuit(const State* st, const lfqs_gate* gates, size_t n_gates,
                                    uint32_t flags) {
  require(n_gates == 0 || gates != nullptr, "gates is NULL");
  require((flags & ~(LFQS_FUSE_LOW | LFQS_FUSE_PHASE | LFQS_FUSE_JIT)) == 0, "unknown flags");
  std::vector<Decoded> dec;
  dec.reserve(n_gates);
  for (size_t i = 0; i < n_gates; ++i) {
    const lfqs_gate& G = gates[i];
    require(G.n_controls == __builtin_popcountll(G.control_mask),
            "gate " + std::to_string(i) + ": n_controls != popcount(control_mask)");
    try {
      dec.push_back(decode_gate(st->n, G.kind, G.targets, G.n_targets, G.control_mask, G.params,
                                kind_nparams(G.kind), G.matrix));
    } catch (const Error& e) {
      throw Error(e.status, "gate " + std::to_string(i) + ": " + e.what());
    }
  }
  return dec;
}
}  // namespace

lfqs_status lfqs_run_circuit(lfqs_state* s, const lfqs_gate* gates, size_t n_gates,
                             uint32_t flags) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    State* st = static_cast<State*>(s);
    st->run(decode_circuit(st, gates, n_gates, flags), flags);
  });
}

lfqs_status lfqs_run_circuit_streamed(lfqs_state* s, const double* host_interleaved,
                                      const lfqs_gate* gates, size_t n_gates, uint32_t flags,
                                      int chunk_bits) {
  return guarded([&] {
    require(s != nullptr && host_interleaved != nullptr, "NULL argument");
    State* st = static_cast<State*>(s);
    require(!st->c64, "streamed runs take complex128 host data (complex128 states)");
    st->run_streamed(host_interleaved, decode_circuit(st, gates, n_gates, flags), flags,
                     chunk_bits);
  });
}

lfqs_status lfqs_circuit_compile(lfqs_state* s, const lfqs_gate* gates, size_t n_gates,
                                 uint32_t flags, lfqs_circuit** out, uint64_t* kernels_out) {
  return guarded([&] {
    require(s != nullptr && out != nullptr, "NULL argument");
    *out = nullptr;
    State* st = static_cast<State*>(s);
    Graph* g = st->compile(decode_circuit(st, gates, n_gates, flags), flags);
    *out = g;
    if (kernels_out) *kernels_out = g->kernels;
  });
}

lfqs_status lfqs_circuit_launch(lfqs_circuit* c) {
  return guarded([&] {
    require(c != nullptr, "NULL circuit");
    static_cast<Graph*>(c)->launch();
  });
}

lfqs_status lfqs_circuit_destroy(lfqs_circuit* c) {
  return guarded([&] { delete static_cast<Graph*>(c); });
}

lfqs_status lfqs_jit_precompile(int n_qubits, int c64, const lfqs_gate* gates, size_t n_gates,
                                uint32_t flags, uint64_t* n_passes) {
  return guarded([&] {
    require(n_gates == 0 || gates != nullptr, "gates is NULL");
    require(n_qubits >= 1 && n_qubits <= 36, "n_qubits must be in [1, 36]");
    require((flags & (LFQS_FUSE_LOW | LFQS_FUSE_JIT)) == (LFQS_FUSE_LOW | LFQS_FUSE_JIT) &&
                (flags & ~(LFQS_FUSE_LOW | LFQS_FUSE_PHASE | LFQS_FUSE_JIT)) == 0,
            "flags must be LFQS_FUSE_LOW | LFQS_FUSE_JIT [| LFQS_FUSE_PHASE]");
    std::vector<Decoded> dec;
    for (size_t i = 0; i < n_gates; ++i) {
      const lfqs_gate& G = gates[i];
      require(G.n_controls == __builtin_popcountll(G.control_mask),
              "gate " + std::to_string(i) + ": n_controls != popcount(control_mask)");
      dec.push_back(decode_gate(n_qubits, G.kind, G.targets, G.n_targets, G.control_mask,
                                G.params, kind_nparams(G.kind), G.matrix));
    }
    Options opt;
    uint64_t count = 0;
    LaunchCtx c;
    c.amps = nullptr;
    c.n_local = n_qubits;
    c.stream = nullptr;
    c.launch_counter = &count;
    c.opt = &opt;
    c.c64 = c64 != 0;
    c.phase_tables = (flags & LFQS_FUSE_PHASE) != 0;
    c.jit = true;
    c.dry_run = true;
    run_fused_schedule(c, dec, opt.fuse_tile_qubits);
    if (n_passes) *n_passes = count;
  });
}

lfqs_status lfqs_plan_circuit(int n_qubits, int world, int rank, const lfqs_gate* gates,
                              size_t n_gates, int canonicalize, lfqs_plan_op* ops,
                              size_t capacity, size_t* n_ops) {
  return guarded([&] {
    require(n_ops != nullptr, "n_ops is NULL");
    require(n_gates == 0 || gates != nullptr, "gates is NULL");
    require(n_qubits >= 1 && n_qubits <= 40, "n_qubits must be in [1, 40]");
    require(world >= 1 && rank >= 0 && rank < world, "bad rank / world");
    Planner plan(n_qubits, world);
    if (canonicalize & LFQS_PLAN_WIDE) plan.swap_lo = std::min(3, plan.n_local - 1);
    std::vector<PlanOp> raw;
    std::vector<Decoded> dec;
    for (size_t i = 0; i < n_gates; ++i) {
      const lfqs_gate& G = gates[i];
      require(G.n_controls == __builtin_popcountll(G.control_mask),
              "gate " + std::to_string(i) + ": n_controls != popcount(control_mask)");
      dec.push_back(decode_gate(n_qubits, G.kind, G.targets, G.n_targets, G.control_mask,
                                G.params, kind_nparams(G.kind), G.matrix));
    }
    if (world == 1) {
      for (const Decoded& d : dec) {
        PlanOp op;
        op.gate = d;
        raw.push_back(op);
      }
    } else {
      plan.plan_circuit(dec, raw);  // the same planning State::run uses
    }
    if (canonicalize & 1) plan.plan_canonicalize(raw);
    // Rank-specialise and convert.
    std::vector<lfqs_plan_op> out;
    for (const PlanOp& op : raw) {
      lfqs_plan_op o;
      std::memset(&o, 0, sizeof o);
      if (op.kind == PlanOp::EXCHANGE) {
        o.kind = LFQS_PLAN_EXCHANGE;
        o.l = op.l;
        o.g = op.g;
        out.push_back(o);
        continue;
      }
      Decoded lg;
      if (!plan.rank_local(op.gate, rank, op.gflip, &lg) || lg.cls == GClass::NOOP) continue;
      o.kind = LFQS_PLAN_LOCAL;
      if (lg.m == 0) {
        // Scalar on the control-satisfying amplitudes: express as a 1-target gate.
        const cplx c = lg.M[0];
        int q = -1;
        for (int b = 0; b < plan.n_local; ++b)
          if (!(lg.cmask >> b & 1)) { q = b; break; }
        lg.m = 1;
        for (int i = 0; i < 4; ++i) lg.M[i] = cplx{0.0, 0.0};
        if (q >= 0) {
          lg.M[0] = c;
          lg.M[3] = c;
        } else {  // every local qubit is a control: move one into the target
          q = 0;
          lg.cmask &= ~1ull;
          lg.M[0] = cplx{1.0, 0.0};
          lg.M[3] = c;
        }
        lg.targets[0] = q;
      }
      const int d = 1 << lg.m;
      o.gate.kind = LFQS_UNITARY1 + lg.m - 1;
      o.gate.n_targets = lg.m;
      for (int s = 0; s < lg.m; ++s) o.gate.targets[s] = lg.targets[s];
      o.gate.control_mask = lg.cmask;
      o.gate.n_controls = __builtin_popcountll(lg.cmask);
      std::memcpy(o.matrix, lg.M, sizeof(cplx) * d * d);
      out.push_back(o);
    }
    *n_ops = out.size();
    require(ops != nullptr || out.empty(), "ops is NULL");
    require(capacity >= out.size(), "capacity < required plan length (see *n_ops)");
    for (size_t i = 0; i < out.size(); ++i) {
      ops[i] = out[i];
      if (ops[i].kind == LFQS_PLAN_LOCAL) ops[i].gate.matrix = ops[i].matrix;
    }
  });
}

lfqs_status lfqs_measure_probs(lfqs_state* s, const int* qubits, int n_q, double* probs_out,
                               size_t probs_len) {
  return guarded([&] {
    require(s != nullptr && probs_out != nullptr, "NULL argument");
    State* st = static_cast<State*>(s);
    require(n_q >= 0 && n_q <= 20, "n_q must be in [0, 20]");
    require(probs_len >= (size_t(1) << n_q), "probs_len < 2^n_q");
    const uint64_t qm = mask_of(qubits, n_q, st->n);
    (void)qm;
    st->measure_probs(qubits, n_q, probs_out);
  });
}

lfqs_status lfqs_measure_sample(lfqs_state* s, const int* qubits, int n_q, const double* uniforms,
                                size_t shots, uint64_t* outcomes) {
  return guarded([&] {
    require(s != nullptr && (shots == 0 || (uniforms != nullptr && outcomes != nullptr)),
            "NULL argument");
    State* st = static_cast<State*>(s);
    require(n_q >= 0 && n_q <= 20, "n_q must be in [0, 20]");
    mask_of(qubits, n_q, st->n);
    std::vector<double> p(size_t(1) << n_q);
    st->measure_probs(qubits, n_q, p.data());
    std::vector<double> c(p.size());
    double acc = 0.0;
    for (size_t v = 0; v < p.size(); ++v) c[v] = acc = acc + p[v];
    for (size_t i = 0; i < shots; ++i) {
      require(uniforms[i] >= 0.0 && uniforms[i] < 1.0, "uniforms must be in [0, 1)");
      const double x = uniforms[i] * c.back();
      outcomes[i] = (uint64_t)(std::upper_bound(c.begin(), c.end(), x) - c.begin());
      if (outcomes[i] >= c.size()) outcomes[i] = c.size() - 1;
    }
  });
}

lfqs_status lfqs_measure_collapse(lfqs_state* s, const int* qubits, int n_q, uint64_t outcome,
                                  double* probability) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    State* st = static_cast<State*>(s);
    require(n_q >= 0 && n_q <= 20, "n_q must be in [0, 20]");
    require(outcome < (uint64_t(1) << n_q), "outcome out of range");
    mask_of(qubits, n_q, st->n);
    std::vector<double> p(size_t(1) << n_q);
    st->measure_probs(qubits, n_q, p.data());
    require(p[outcome] > 0.0, "outcome has probability 0");
    st->collapse(qubits, n_q, outcome, 1.0 / std::sqrt(p[outcome]));
    if (probability) *probability = p[outcome];
  });
}

lfqs_status lfqs_synchronize(lfqs_state* s) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    static_cast<State*>(s)->synchronize();
  });
}

lfqs_status lfqs_state_exchange_stats(const lfqs_state* s, uint64_t* exchanges,
                                      uint64_t* bytes_per_rank) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    const State* st = static_cast<const State*>(s);
    if (exchanges) *exchanges = st->exchanges;
    if (bytes_per_rank) *bytes_per_rank = st->exchange_bytes;
  });
}

lfqs_status lfqs_state_overlap_stats(const lfqs_state* s, uint64_t* overlapped_exchanges,
                                     uint64_t* block_passes, uint64_t* strided_exchanges,
                                     uint64_t* chained_exchanges) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    const State* st = static_cast<const State*>(s);
    if (overlapped_exchanges) *overlapped_exchanges = st->ov_exchanges;
    if (block_passes) *block_passes = st->ov_block_passes;
    if (strided_exchanges) *strided_exchanges = st->ov_strided;
    if (chained_exchanges) *chained_exchanges = st->ov_chained;
  });
}

lfqs_status lfqs_state_info(const lfqs_state* s, int* n_qubits, int* n_local, int* rank,
                            int* world, void** dev_ptr) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    const State* st = static_cast<const State*>(s);
    if (n_qubits) *n_qubits = st->n;
    if (n_local) *n_local = st->n_local;
    if (rank) *rank = st->rank;
    if (world) *world = st->world;
    if (dev_ptr) *dev_ptr = st->shard_ptr();
  });
}

lfqs_status lfqs_kernel_launches(const lfqs_state* s, uint64_t* count) {
  return guarded([&] {
    require(s != nullptr && count != nullptr, "NULL argument");
    *count = static_cast<const State*>(s)->launches;
  });
}

lfqs_status lfqs_state_pass_count(const lfqs_state* s, uint64_t* passes) {
  return guarded([&] {
    require(s != nullptr && passes != nullptr, "NULL argument");
    *passes = static_cast<const State*>(s)->passes;
  });
}

lfqs_status lfqs_set_option(lfqs_state* s, int option, int64_t value) {
  return guarded([&] {
    require(s != nullptr, "NULL state");
    State* st = static_cast<State*>(s);
    switch (option) {
      case LFQS_OPT_LOWQ_SHUFFLE: st->opt.lowq_shuffle = value != 0; break;
      case LFQS_OPT_FUSE_TILE_QUBITS:
        require(value >= 6 && value <= 13, "tile qubits must be in [6, 13]");
        st->opt.fuse_tile_qubits = (int)value;
        break;
      case LFQS_OPT_ITEMS_PER_THREAD: st->opt.items_per_thread = (int)value; break;
      case LFQS_OPT_WIDE256: st->opt.wide256 = value != 0; break;
      case LFQS_OPT_LINE_READS: st->opt.line_reads = value != 0; break;
      case LFQS_OPT_FUSE_MERGE_2Q: st->opt.fuse_merge_2q = value != 0; break;
      case LFQS_OPT_FUSE_H_SCALE: st->opt.fuse_h_scale = value != 0; break;
      case LFQS_OPT_FUSE_PHASE_EXTRACT: st->opt.fuse_phase_extract = value != 0; break;
      case LFQS_OPT_CANON_FUSE: st->opt.canon_fuse = value != 0; break;
      case LFQS_OPT_EXCHANGE_WIDE: st->opt.exchange_wide = value != 0; break;
      case LFQS_OPT_FUSE_PERM:
        require(value == 0 || value == 1 || (value >= 8 && value <= 12),
                "LFQS_OPT_FUSE_PERM must be 0, 1 or a tile size in [8, 12]");
        st->opt.fuse_perm = (int)value;
        break;
      case LFQS_OPT_EXCHANGE_CHUNK_BITS:
        require(value >= 0 && value <= 3, "LFQS_OPT_EXCHANGE_CHUNK_BITS must be in [0, 3]");
        st->opt.exchange_chunk_bits = (int)value;  // the plan is the same for every value
        break;
      case LFQS_OPT_EXCHANGE_CHUNK_SELECT: st->opt.exchange_chunk_select = value != 0; break;
      case LFQS_OPT_EXCHANGE_RATE_GBS:
        require(value >= 0 && value <= 100000, "LFQS_OPT_EXCHANGE_RATE_GBS must be in [0, 100000]");
        st->opt.exchange_rate_gbs = (int)value;
        break;
      case LFQS_OPT_EXCHANGE_CTAS:
        require(value >= 0 && value <= 65535, "LFQS_OPT_EXCHANGE_CTAS must be in [0, 65535]");
        st->opt.exchange_ctas = (int)value;
        break;
      case LFQS_OPT_FUSE_LOW_QUBITS:
        require(value == 0 || (value >= 3 && value <= 12),
                "fused low qubits must be 0 (auto) or in [3, 12]");
        st->opt.fuse_low_qubits = (int)value;
        break;
      case LFQS_OPT_FUSE_REORDER: st->opt.fuse_reorder = value != 0; break;
      case LFQS_OPT_JIT_THREADS:
        require(value == 0 || value == 128 || value == 256 || value == 512,
                "LFQS_OPT_JIT_THREADS must be 0 (per pass), 128, 256 or 512");
        st->opt.jit_threads = (int)value;
        break;
      case LFQS_OPT_JIT_LANE_MOVE: st->opt.jit_lane_move = value != 0; break;
      case LFQS_OPT_FUSE_MERGE_COMMUTING: st->opt.fuse_merge_commuting = value != 0; break;
      case LFQS_OPT_JIT_GREEDY_PLACE: st->opt.jit_greedy_place = value != 0; break;
      case LFQS_OPT_JIT_LANE_REG2: st->opt.jit_lane_reg2 = value != 0; break;
      case LFQS_OPT_JIT_LANE_POOL: st->opt.jit_lane_pool = value != 0; break;
      case LFQS_OPT_JIT_PARTIAL_RT: st->opt.jit_partial_rt = value != 0; break;
      case LFQS_OPT_FUSE_PHASE_SPLIT: st->opt.fuse_phase_split = value != 0; break;
      case LFQS_OPT_L2_FETCH_GRANULARITY: {
        require(value == 0 || value == 32 || value == 64 || value == 128,
                "LFQS_OPT_L2_FETCH_GRANULARITY must be 0, 32, 64 or 128");
        int prev = -1;
        cudaGetDevice(&prev);
        if (prev != st->device) LFQS_CUDA_CHECK(cudaSetDevice(st->device));
        const cudaError_t err = cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, (size_t)value);
        if (prev >= 0 && prev != st->device) cudaSetDevice(prev);
        LFQS_CUDA_CHECK(err);
        break;
      }
      case LFQS_OPT_STREAM_MAX_PREFIX:
        require(value >= 0, "LFQS_OPT_STREAM_MAX_PREFIX must be >= 0");
        st->opt.stream_max_prefix = (int)value;
        break;
      case LFQS_OPT_LANE_GROUP:
        require(value >= 0 && value <= 2, "LFQS_OPT_LANE_GROUP must be 0, 1 or 2");
        st->opt.lane_group = (int)value;
        break;
      case LFQS_OPT_FUSE_TMA_MAX_CHUNKS:
        require(value >= 0 && value <= 256, "TMA max chunks must be in [0, 256]");
        st->opt.fuse_tma_max_chunks = (int)value;
        break;
      default: require(false, "unknown option");
    }
  });
}

}  // extern "C"
