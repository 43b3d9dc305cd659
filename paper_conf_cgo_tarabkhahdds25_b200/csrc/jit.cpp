// jit.cpp -- pass compiler: each fused pass's gate program (fused_prog.h) is
// compiled into its own straight-line sm_100a kernel (LFQS_FUSE_JIT).
//
// The paper synthesises a simulator by compiling the circuit: vector fusion,
// loop unrolling and static matrix specialisation turn
// every gate into code with its structure baked in.  The interpreting kernel
// k_fused (fused_kernels.cu) re-decodes each op of a pass for every tile; on
// B200 that decode (constant-bank header loads, predicate arithmetic, branch
// trees) costs more issue slots than the FP64 math of phase-heavy passes
// (ncu: ~65% of stall samples, profiles/r01_fused_jit.md).  Here the program
// of a pass is emitted as PTX with every index, predicate, register selection
// and op type resolved at generation time; only the coefficients stay a kernel
// parameter (constant bank), so one compiled pass serves every angle set of
// the same circuit structure.  PTX is compiled in-process by nvPTXCompiler
// (no NVVM: compiling generated CUDA C++ through NVRTC took seconds per pass),
// passes are compiled in parallel and cached by their structure, and loaded
// with cudaLibraryLoadData.
//
// The emitted arithmetic replicates k_fused op by op (same formulas, same FMA
// and rounding order, same tile/register transitions), so a JIT pass is
// bit-identical to the interpreted pass (tests/test_gpu_jit.py).
#include "jit.h"

#include <nvPTXCompiler.h>

#include <atomic>
#include <cmath>
#include <condition_variable>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

namespace lfqs {

namespace {

// ---------------------------------------------------------------------------
// PTX emitter
// ---------------------------------------------------------------------------
struct Gen {
  const FProg& P;
  const int K;
  const bool c64;
  const char* FT;       // "f64" | "f32"
  int ES;               // bytes per amplitude
  int R;                // amplitudes per thread
  std::string body;
  int nr = 0, nrd = 0, nf = 0, np = 0, nl = 0;
  bool in_regs = true;

  // Placement of tile bits in (thread, slot): thread bit j holds tile bit tpos[j],
  // slot bit j holds rpos[j].  The low FL lane bits always hold tile bits 0..FL-1, so
  // the 16-B (8-B for complex64) shared-memory accesses of a quarter-warp (half-warp)
  // cover distinct banks; FL = 5 unless lane moves are on (LFQS_OPT_JIT_LANE_MOVE),
  // then lane bits FL..4 are movable like the 3 warp positions (thread bits 5..7).
  // The interpreter's placement is the identity; the compiled pass moves a tile bit
  // into a register position (a tile round trip, `remap`) when a gate needs it
  // there, so 1-target gates on warp bits (and, with lane moves, on lane bits >= FL)
  // and multi-target gates on movable bits run in registers instead of as
  // shared-memory ops or shuffles.  Every amplitude still sees the same arithmetic
  // (a moved lane bit keeps the interpreter's lane formulas), so results stay
  // bit-identical to the interpreter.
  int NT = 256;   // threads per CTA (128 for K >= 8, 256, or 512 for K >= 9)
  int NWB = 3;    // warp bits of the thread index
  int FL = 5;     // fixed lane bits
  bool greedy = false;  // greedy placement (JIT_GREEDY_PLACE)
  bool lane_reg2 = false;  // SWAP / U4 with one fixed-lane target by shuffles (JIT_LANE_REG2)
  bool pool = false;       // lane-pool placement (JIT_LANE_POOL)
  bool partial_rt = false; // round trips move only re-placed amplitudes (JIT_PARTIAL_RT)
  int tpos[9] = {0, 1, 2, 3, 4, 5, 6, 7, 8};
  int rpos[8] = {8, 9, 10, 11, 12, 13, 14, 15};
  int nreg = 0;

  Gen(const FProg& p, int k, bool c, int jc) : P(p), K(k), c64(c) {
    FT = c64 ? "f32" : "f64";
    ES = c64 ? 8 : 16;
    NT = jc & JIT_THREADS_MASK;
    NWB = NT == 512 ? 4 : NT == 128 ? 2 : 3;
    R = (1 << K) / NT;
    nreg = K - 5 - NWB;
    FL = ((jc & JIT_LANE_MOVE) && nreg >= 1) ? (c64 ? 4 : 3) : 5;
    greedy = (jc & JIT_GREEDY_PLACE) != 0;
    lane_reg2 = (jc & JIT_LANE_REG2) != 0;
    pool = (jc & JIT_LANE_POOL) && greedy && lane_reg2 && FL < 5 && nreg >= 1;
    // complex64: measured slower with partial round trips (QFT(31) 83 -> 96 ms), off there
    partial_rt = (jc & JIT_PARTIAL_RT) != 0 && !c64;
    for (int j = 0; j < 5 + NWB; ++j) tpos[j] = j;
    for (int j = 0; j < nreg; ++j) rpos[j] = 5 + NWB + j;
  }

  // .minnctapersm: complex64 tiles are half the bytes, so more CTAs fit per SM (up
  // to 1024 threads and the shared memory the tile allows); complex128 keeps 2 (3 at
  // 128 threads), which its register-resident amplitudes need.
  int min_ctas() const {
    const int base = NT == 128 ? 3 : 2;
    if (!c64) return base;
    const int by_smem = (200 * 1024) / ((ES << K) + 4096);
    return std::max(base, std::min(by_smem, 1024 / NT));
  }

  int reg_of(int b) const {
    for (int j = 0; j < nreg; ++j)
      if (rpos[j] == b) return j;
    return -1;
  }
  // Thread bit holding tile bit b, or -1 when b is register-held.
  int tbit(int b) const {
    for (int j = 0; j < 5 + NWB; ++j)
      if (tpos[j] == b) return j;
    return -1;
  }
  // Tile bit b sits at a lane position (0..4).
  bool at_lane(int b) const {
    const int t = tbit(b);
    return t >= 0 && t < 5;
  }
  // Lane pool: the movable lane positions are "cheap" positions like the registers.
  bool cheap(int b) const { return reg_of(b) >= 0 || (pool && at_lane(b)); }
  // Tile bit b sits at a fixed lane position (shuffle path only).
  bool fixed_lane(int b) const {
    const int t = tbit(b);
    return t >= 0 && t < FL;
  }
  // (i & m) == v split into a thread part and a slot part.
  void split(uint32_t m, uint32_t v, uint32_t& tm, uint32_t& tv, uint32_t& rm, uint32_t& rv) const {
    tm = tv = rm = rv = 0;
    for (int b = 0; b < K; ++b) {
      if (!((m >> b) & 1)) continue;
      const uint32_t bit = (v >> b) & 1;
      const int t = tbit(b);
      if (t >= 0) {
        tm |= 1u << t;
        tv |= bit << t;
      } else {
        const int j = reg_of(b);
        rm |= 1u << j;
        rv |= bit << j;
      }
    }
  }
  // Tile-index offset of slot r.
  uint32_t roff(int r) const {
    uint32_t o = 0;
    for (int j = 0; j < nreg; ++j)
      if ((r >> j) & 1) o |= 1u << rpos[j];
    return o;
  }
  // %taddr = tile + ES * (thread part of the tile index).
  void emit_taddr() {
    const std::string t = r();
    e("and.b32 %s, %%ltid, %d;", t.c_str(), (1 << FL) - 1);
    for (int j = FL; j < 5 + NWB; ++j) {
      const std::string x = r();
      e("bfe.u32 %s, %%ltid, %d, 1;", x.c_str(), j);
      e("shl.b32 %s, %s, %d;", x.c_str(), x.c_str(), tpos[j]);
      e("or.b32 %s, %s, %s;", t.c_str(), t.c_str(), x.c_str());
    }
    e("mad.lo.u32 %%taddr, %s, %d, %%tile;", t.c_str(), ES);
  }

  void e(const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    body += "  ";
    body += buf;
    body += "\n";
  }
  std::string r() { return "%r" + std::to_string(nr++); }
  std::string rd() { return "%rd" + std::to_string(nrd++); }
  std::string f() { return "%f" + std::to_string(nf++); }
  std::string p() { return "%p" + std::to_string(np++); }
  std::string L() { return "L" + std::to_string(nl++); }
  void label(const std::string& l) { body += l + ":\n"; }

  // Amplitude registers of slot r.
  static std::string vx(int r) { return "%vx" + std::to_string(r); }
  static std::string vy(int r) { return "%vy" + std::to_string(r); }

  // A complex value in registers.  For program coefficients the value is known at
  // generation time (kv): exact zeros / ones in it are specialised away (static
  // matrix specialisation) -- value-identical to the interpreter,
  // whose products with those exact constants are exact.
  struct Cx {
    std::string x, y;
    bool kv = false;
    double vx = 0, vy = 0;
    bool zx() const { return kv && vx == 0.0; }
    bool zy() const { return kv && vy == 0.0; }
  };

  // Coefficient j of the pool as amplitude-type registers (cvs<S>).
  Cx coef(int j) {
    Cx c{f(), f()};
    c.kv = true;
    c.vx = c64 ? (double)(float)P.c[j].x : P.c[j].x;
    c.vy = c64 ? (double)(float)P.c[j].y : P.c[j].y;
    if (!c64) {
      e("ld.param.v2.f64 {%s, %s}, [pc+%d];", c.x.c_str(), c.y.c_str(), j * 16);
    } else {
      const std::string a = "%dd" + std::to_string(nrd), b = "%dd" + std::to_string(nrd + 1);
      nrd += 2;
      e("ld.param.v2.f64 {%s, %s}, [pc+%d];", a.c_str(), b.c_str(), j * 16);
      e("cvt.rn.f32.f64 %s, %s;", c.x.c_str(), a.c_str());
      e("cvt.rn.f32.f64 %s, %s;", c.y.c_str(), b.c_str());
    }
    return c;
  }
  std::string coef_re(int j) { return coef(j).x; }
  std::string coef_im(int j) { return coef(j).y; }

  std::string neg(const std::string& a) {
    std::string t = f();
    e("neg.%s %s, %s;", FT, t.c_str(), a.c_str());
    return t;
  }
  std::string mul(const std::string& a, const std::string& b) {
    std::string t = f();
    e("mul.rn.%s %s, %s, %s;", FT, t.c_str(), a.c_str(), b.c_str());
    return t;
  }
  std::string add(const std::string& a, const std::string& b) {
    std::string t = f();
    e("add.rn.%s %s, %s, %s;", FT, t.c_str(), a.c_str(), b.c_str());
    return t;
  }
  std::string sub(const std::string& a, const std::string& b) {
    std::string t = f();
    e("sub.rn.%s %s, %s, %s;", FT, t.c_str(), a.c_str(), b.c_str());
    return t;
  }
  std::string fma(const std::string& a, const std::string& b, const std::string& c) {
    std::string t = f();
    e("fma.rn.%s %s, %s, %s, %s;", FT, t.c_str(), a.c_str(), b.c_str(), c.c_str());
    return t;
  }
  std::string zero() { return c64 ? "0f00000000" : "0d0000000000000000"; }
  std::string sel(const std::string& a, const std::string& b, const std::string& pr) {
    std::string t = f();
    e("selp.%s %s, %s, %s, %s;", FT, t.c_str(), a.c_str(), b.c_str(), pr.c_str());
    return t;
  }
  // cmul_rn(d, a) (cx.cuh): (dx ax - dy ay, dx ay + dy ax), RN, no FMA.
  Cx cmul(const Cx& d, const Cx& a) {
    if (d.zy()) {  // real factor: (dx ax, dx ay); dx = +-1: copy / negate
      if (d.vx == 1.0) return a;
      if (d.vx == -1.0) return {neg(a.x), neg(a.y)};
      return {mul(d.x, a.x), mul(d.x, a.y)};
    }
    if (d.zx()) {  // imaginary factor: (-(dy ay), dy ax)
      if (d.vy == 1.0) return {neg(a.y), a.x};
      if (d.vy == -1.0) return {a.y, neg(a.x)};
      return {neg(mul(d.y, a.y)), mul(d.y, a.x)};
    }
    const std::string t1 = mul(d.x, a.x), t2 = mul(d.y, a.y);
    const std::string nx = sub(t1, t2);
    const std::string t3 = mul(d.x, a.y), t4 = mul(d.y, a.x);
    const std::string ny = add(t3, t4);
    return {nx, ny};
  }
  // cfma(acc, m, v) with acc == (0, 0) when first.
  // cmul_fma(d, a) (cx.cuh): (fma(dx, ax, -(dy ay)), fma(dx, ay, dy ax)) -- phase tables.
  Cx cmulf(const Cx& d, const Cx& a) {
    if (d.zy()) {
      if (d.vx == 1.0) return a;
      if (d.vx == -1.0) return {neg(a.x), neg(a.y)};
      return {mul(d.x, a.x), mul(d.x, a.y)};
    }
    if (d.zx()) {
      if (d.vy == 1.0) return {neg(a.y), a.x};
      if (d.vy == -1.0) return {a.y, neg(a.x)};
      return {neg(mul(d.y, a.y)), mul(d.y, a.x)};
    }
    return {fma(d.x, a.x, neg(mul(d.y, a.y))), fma(d.x, a.y, mul(d.y, a.x))};
  }
  // Terms with an exactly-zero coefficient part are skipped (fma(0, v, acc) == acc).
  void cfma(Cx& acc, const Cx& m, const Cx& nmy, const Cx& v, bool first) {
    // nmy.x holds -m.y (precomputed)
    if (first) acc = Cx{zero(), zero()};
    if (!m.zx()) acc.x = fma(m.x, v.x, acc.x);
    if (!m.zy()) acc.x = fma(nmy.x, v.y, acc.x);
    if (!m.zx()) acc.y = fma(m.x, v.y, acc.y);
    if (!m.zy()) acc.y = fma(m.y, v.x, acc.y);
  }
  // selp of two known coefficients: known zero parts when both agree.
  Cx sel_c(const Cx& a, const Cx& b, const std::string& bit) {
    Cx o{sel(a.x, b.x, bit), sel(a.y, b.y, bit)};
    if (a.kv && b.kv) {
      if (a.vx == 0.0 && b.vx == 0.0) { o.kv = true; o.vx = 0.0; o.vy = 1.0; }
      if (a.vy == 0.0 && b.vy == 0.0) {
        if (!o.kv) { o.kv = true; o.vx = 1.0; }
        o.vy = 0.0;
      }
      if (o.kv && o.vx != 0.0) o.vx = 2.0;  // nonzero, not a special value
      if (o.kv && o.vy != 0.0) o.vy = 2.0;
    }
    return o;
  }
  Cx copy(const Cx& z) {
    Cx c{f(), f()};
    e("mov.%s %s, %s;", FT, c.x.c_str(), z.x.c_str());
    e("mov.%s %s, %s;", FT, c.y.c_str(), z.y.c_str());
    return c;
  }
  // (dx, dy) = z; safe when z.y names dx (e.g. z = (-a.y, a.x) for a = (dx, dy)).
  void assign(const std::string& dx, const std::string& dy, Cx z) {
    if (z.y == dx) z.y = copy({z.y, z.y}).x;
    if (z.x != dx) e("mov.%s %s, %s;", FT, dx.c_str(), z.x.c_str());
    if (z.y != dy) e("mov.%s %s, %s;", FT, dy.c_str(), z.y.c_str());
  }
  void set(int r, const Cx& z) { assign(vx(r), vy(r), z); }

  // ---- integer helpers -----------------------------------------------------
  // Branch to `skip` unless (base & mhi) == phi.
  void tile_pred(uint64_t mhi, uint64_t phi, const std::string& skip) {
    if (mhi == 0) return;
    const std::string t = rd(), q = p();
    e("and.b64 %s, %%base, %llu;", t.c_str(), (unsigned long long)mhi);
    e("setp.ne.b64 %s, %s, %llu;", q.c_str(), t.c_str(), (unsigned long long)phi);
    e("@%s bra %s;", q.c_str(), skip.c_str());
  }
  // Predicate register: (tid & m) == pv  (m == 0: none -> "")
  std::string thread_pred(uint32_t m, uint32_t pv) {
    uint32_t rm, rv;
    split(m, pv, m, pv, rm, rv);
    if (m == 0) return "";
    const std::string t = r(), q = p();
    e("and.b32 %s, %%ltid, %u;", t.c_str(), m);
    e("setp.eq.b32 %s, %s, %u;", q.c_str(), t.c_str(), pv);
    return q;
  }
  void skip_unless(const std::string& q, const std::string& skip) {
    if (!q.empty()) e("@!%s bra %s;", q.c_str(), skip.c_str());
  }

  // ---- tile <-> registers ----------------------------------------------------
  void regs_to_tile() {
    for (int r = 0; r < R; ++r)
      e("st.shared.v2.%s [%%taddr+%u], {%s, %s};", FT, roff(r) * ES, vx(r).c_str(),
        vy(r).c_str());
  }
  void tile_to_regs() {
    for (int r = 0; r < R; ++r)
      e("ld.shared.v2.%s {%s, %s}, [%%taddr+%u];", FT, vx(r).c_str(), vy(r).c_str(),
        roff(r) * ES);
  }
  void sync() { e("bar.sync 0;"); }

  // Placement change by a tile round trip that moves only the amplitudes whose (thread,
  // slot) changes (LFQS_OPT_JIT_PARTIAL_RT): amplitude (t, r) of the old placement (ot,
  // orp) stays in its register iff every position holds the same tile-index bit value
  // under the new placement (tpos, rpos); the condition is the same in old and new
  // coordinates, so one predicate per slot guards both the store and the load.  A swap
  // of k position pairs moves 1 - 2^-k of the tile instead of all of it.
  void partial_roundtrip(const int* ot, const int* orp) {
    const int NTB = 5 + NWB;
    auto old_thread_pos = [&](int b) {
      for (int j = 0; j < NTB; ++j)
        if (ot[j] == b) return j;
      return -1;
    };
    auto old_slot_pos = [&](int b) {
      for (int j = 0; j < nreg; ++j)
        if (orp[j] == b) return j;
      return -1;
    };
    // thread-thread equalities (runtime, same for every slot)
    std::string ptt;
    for (int j = 0; j < NTB; ++j) {
      if (tpos[j] == ot[j]) continue;
      const int jt = old_thread_pos(tpos[j]);
      if (jt < 0) continue;
      const std::string a = r(), q = p();
      e("shr.u32 %s, %%ltid, %d;", a.c_str(), jt - j > 0 ? jt - j : 0);
      if (j > jt) e("shl.b32 %s, %%ltid, %d;", a.c_str(), j - jt);
      e("xor.b32 %s, %s, %%ltid;", a.c_str(), a.c_str());
      e("and.b32 %s, %s, %u;", a.c_str(), a.c_str(), 1u << j);
      if (ptt.empty()) {
        e("setp.eq.b32 %s, %s, 0;", q.c_str(), a.c_str());
      } else {
        e("setp.eq.and.b32 %s, %s, 0, %s;", q.c_str(), a.c_str(), ptt.c_str());
      }
      ptt = q;
    }
    // per slot: (t & M) == V from thread-slot equalities; compile-time slot-slot ones
    std::vector<std::string> pslot(R);
    std::map<std::pair<uint32_t, uint32_t>, std::string> cache;
    for (int r_ = 0; r_ < R; ++r_) {
      bool never = false;
      uint32_t M = 0, V = 0;
      for (int j = 0; j < NTB; ++j) {  // new thread bit j holds tile bit tpos[j]
        if (tpos[j] == ot[j]) continue;
        const int js = old_slot_pos(tpos[j]);
        if (js >= 0) {
          M |= 1u << j;
          V |= (uint32_t)((r_ >> js) & 1) << j;
        }
      }
      for (int j = 0; j < nreg; ++j) {  // new slot bit j holds tile bit rpos[j]
        if (rpos[j] == orp[j]) continue;
        const int jt = old_thread_pos(rpos[j]);
        if (jt >= 0) {
          M |= 1u << jt;
          V |= (uint32_t)((r_ >> j) & 1) << jt;
        } else {
          const int js = old_slot_pos(rpos[j]);
          if (((r_ >> js) & 1) != ((r_ >> j) & 1)) never = true;
        }
      }
      if (never) continue;  // always moves
      auto it = cache.find({M, V});
      if (it == cache.end()) {
        const std::string a = r(), q = p();
        e("and.b32 %s, %%ltid, %u;", a.c_str(), M);
        if (ptt.empty())
          e("setp.eq.b32 %s, %s, %u;", q.c_str(), a.c_str(), V);
        else
          e("setp.eq.and.b32 %s, %s, %u, %s;", q.c_str(), a.c_str(), V, ptt.c_str());
        it = cache.emplace(std::make_pair(M, V), q).first;
      }
      pslot[r_] = it->second;
    }
    // stores of moving amplitudes under the old placement (old %taddr, old slot offsets)
    for (int r_ = 0; r_ < R; ++r_) {
      uint32_t o = 0;
      for (int j = 0; j < nreg; ++j)
        if ((r_ >> j) & 1) o |= 1u << orp[j];
      const std::string g = pslot[r_].empty() ? "" : "@!" + pslot[r_] + " ";
      e("%sst.shared.v2.%s [%%taddr+%u], {%s, %s};", g.c_str(), FT, o * ES, vx(r_).c_str(),
        vy(r_).c_str());
    }
    sync();
    emit_taddr();
    for (int r_ = 0; r_ < R; ++r_) {
      const std::string g = pslot[r_].empty() ? "" : "@!" + pslot[r_] + " ";
      e("%sld.shared.v2.%s {%s, %s}, [%%taddr+%u];", g.c_str(), FT, vx(r_).c_str(),
        vy(r_).c_str(), roff(r_) * ES);
    }
    in_regs = true;
  }

  // ---- 2x2 functor semantics (fused_kernels.cu FX_/FY_/FH_/FR_/FI_/FU_) -----
  struct Op2 {
    int type;
    std::string s;                  // F_H
    bool s1 = false;                // F_H coefficient exactly 1: the unscaled butterfly
    std::string m00, m01, m10, m11; // F_UR
    std::string d0, e01, e10, d1;   // F_UI
    Cx c0, c1, c2, c3, n0, n1, n2, n3;  // F_U2 (n*.x = -c*.y)
  };
  Op2 load_op2(const FHdr& h) {
    Op2 o;
    o.type = h.type;
    const int c = h.coef;
    switch (h.type) {
      case F_H: {
        const Cx k = coef(c);
        o.s = k.x;
        o.s1 = k.vx == 1.0;
        break;
      }
      case F_UR:
        o.m00 = coef_re(c); o.m01 = coef_re(c + 1); o.m10 = coef_re(c + 2); o.m11 = coef_re(c + 3);
        break;
      case F_UI:
        o.d0 = coef_re(c); o.e01 = coef_im(c + 1); o.e10 = coef_im(c + 2); o.d1 = coef_re(c + 3);
        break;
      case F_U2:
        o.c0 = coef(c); o.c1 = coef(c + 1); o.c2 = coef(c + 2); o.c3 = coef(c + 3);
        o.n0 = {neg(o.c0.y), ""}; o.n1 = {neg(o.c1.y), ""};
        o.n2 = {neg(o.c2.y), ""}; o.n3 = {neg(o.c3.y), ""};
        break;
      default: break;
    }
    return o;
  }
  // s * v of F_H; with s == 1 (fold_h_scales) the exact product is dropped
  std::string hs(const Op2& o, const std::string& v) { return o.s1 ? v : mul(o.s, v); }
  void pair(const Op2& o, Cx& a0, Cx& a1) {
    const Cx x0 = a0, x1 = a1;
    switch (o.type) {
      case F_X: a0 = x1; a1 = x0; return;
      case F_Y:
        a0 = {x1.y, neg(x1.x)};
        a1 = {neg(x0.y), x0.x};
        return;
      case F_H:
        a0 = {hs(o, add(x0.x, x1.x)), hs(o, add(x0.y, x1.y))};
        a1 = {hs(o, sub(x0.x, x1.x)), hs(o, sub(x0.y, x1.y))};
        return;
      case F_UR:
        a0 = {fma(o.m01, x1.x, mul(o.m00, x0.x)), fma(o.m01, x1.y, mul(o.m00, x0.y))};
        a1 = {fma(o.m11, x1.x, mul(o.m10, x0.x)), fma(o.m11, x1.y, mul(o.m10, x0.y))};
        return;
      case F_UI: {
        const std::string ne01 = neg(o.e01), ne10 = neg(o.e10);
        a0 = {fma(ne01, x1.y, mul(o.d0, x0.x)), fma(o.e01, x1.x, mul(o.d0, x0.y))};
        a1 = {fma(o.d1, x1.x, mul(ne10, x0.y)), fma(o.d1, x1.y, mul(o.e10, x0.x))};
        return;
      }
      default: {  // F_U2
        Cx b0, b1;
        cfma(b0, o.c0, o.n0, x0, true);
        cfma(b0, o.c1, o.n1, x1, false);
        cfma(b1, o.c2, o.n2, x0, true);
        cfma(b1, o.c3, o.n3, x1, false);
        a0 = b0;
        a1 = b1;
        return;
      }
    }
  }
  // Lane form: amplitude a, partner p, runtime bit predicate `bit` (bit == 1);
  // k_fused's FX_/FY_/FH_/FR_/FI_/FU_ lane(): only the coefficients depend on the
  // lane bit, selected once per op (lane_coefs), so no per-amplitude selects
  // except the sign of H and the permutation of Y.
  struct LaneC {
    std::string A, B, D, E, nE;  // F_UR: own A, partner B; F_UI: own D, partner E
    Cx m1, n1, m2, n2;           // F_U2: own m1, partner m2 (n*.x = -m*.y)
  };
  LaneC lane_coefs(const Op2& o, const std::string& bit) {
    LaneC l;
    switch (o.type) {
      case F_UR:
        l.A = sel(o.m11, o.m00, bit);
        l.B = sel(o.m10, o.m01, bit);
        break;
      case F_UI:
        l.D = sel(o.d1, o.d0, bit);
        l.E = sel(o.e10, o.e01, bit);
        l.nE = neg(l.E);
        break;
      case F_U2:
        l.m1 = sel_c(o.c3, o.c0, bit);
        l.n1 = {sel(o.n3.x, o.n0.x, bit), ""};
        l.m2 = sel_c(o.c2, o.c1, bit);
        l.n2 = {sel(o.n2.x, o.n1.x, bit), ""};
        break;
      default: break;
    }
    return l;
  }
  Cx lane(const Op2& o, const LaneC& l, const Cx& a, const Cx& pp, const std::string& bit) {
    switch (o.type) {
      case F_X: return pp;
      case F_Y: {
        // bit ? (-p.y, p.x) : (p.y, -p.x)
        const std::string npy = neg(pp.y), npx = neg(pp.x);
        return {sel(npy, pp.y, bit), sel(pp.x, npx, bit)};
      }
      case F_H: {
        // s (p + (bit ? -a : a))
        const std::string ax = sel(neg(a.x), a.x, bit), ay = sel(neg(a.y), a.y, bit);
        return {hs(o, add(pp.x, ax)), hs(o, add(pp.y, ay))};
      }
      case F_UR:
        return {fma(l.B, pp.x, mul(l.A, a.x)), fma(l.B, pp.y, mul(l.A, a.y))};
      case F_UI:
        return {fma(l.nE, pp.y, mul(l.D, a.x)), fma(l.E, pp.x, mul(l.D, a.y))};
      default: {  // F_U2: own amplitude first, partner second
        Cx acc;
        cfma(acc, l.m1, l.n1, a, true);
        cfma(acc, l.m2, l.n2, pp, false);
        return acc;
      }
    }
  }

  // lane() with the lane bit known at generation time (a lane tile bit moved into
  // a register position): the same operations with the selections resolved.
  Cx lane_const(const Op2& o, const Cx& a, const Cx& pp, int bit) {
    switch (o.type) {
      case F_X: return pp;
      case F_Y: return bit ? Cx{neg(pp.y), pp.x} : Cx{pp.y, neg(pp.x)};
      case F_H: {
        const std::string ax = bit ? neg(a.x) : a.x, ay = bit ? neg(a.y) : a.y;
        return {hs(o, add(pp.x, ax)), hs(o, add(pp.y, ay))};
      }
      case F_UR: {
        const std::string& A = bit ? o.m11 : o.m00;
        const std::string& B = bit ? o.m10 : o.m01;
        return {fma(B, pp.x, mul(A, a.x)), fma(B, pp.y, mul(A, a.y))};
      }
      case F_UI: {
        const std::string& D = bit ? o.d1 : o.d0;
        const std::string& E = bit ? o.e10 : o.e01;
        return {fma(neg(E), pp.y, mul(D, a.x)), fma(E, pp.x, mul(D, a.y))};
      }
      default: {  // F_U2: own amplitude first, partner second
        Cx acc;
        cfma(acc, bit ? o.c3 : o.c0, bit ? o.n3 : o.n0, a, true);
        cfma(acc, bit ? o.c2 : o.c1, bit ? o.n2 : o.n1, pp, false);
        return acc;
      }
    }
  }

  // pair() evaluated by a lane that holds one amplitude of the pair (tile bit >= 5 at
  // a lane position, lane-pool placement): x0 / x1 put back in pair order by value
  // selects, coefficients selected once per op (LaneP), then pair()'s exact operation
  // sequence -- bit-identical to the register / shared-memory pair.
  struct LaneP {
    std::string c1, c2, f1, f2, g1, g2;  // F_UR: c1, c2; F_UI: f* (re), g* (im)
    Cx m1, n1, m2, n2;                   // F_U2
  };
  LaneP lanep_coefs(const Op2& o, const std::string& bit) {
    LaneP l;
    switch (o.type) {
      case F_UR:
        l.c1 = sel(o.m10, o.m00, bit);
        l.c2 = sel(o.m11, o.m01, bit);
        break;
      case F_UI:
        l.f1 = sel(neg(o.e10), o.d0, bit);
        l.f2 = sel(o.d1, neg(o.e01), bit);
        l.g1 = sel(o.e10, o.d0, bit);
        l.g2 = sel(o.d1, o.e01, bit);
        break;
      case F_U2:
        l.m1 = sel_c(o.c2, o.c0, bit);
        l.n1 = {sel(o.n2.x, o.n0.x, bit), ""};
        l.m2 = sel_c(o.c3, o.c1, bit);
        l.n2 = {sel(o.n3.x, o.n1.x, bit), ""};
        break;
      default: break;
    }
    return l;
  }
  Cx lane_pair(const Op2& o, const LaneP& l, const Cx& a, const Cx& pp, const std::string& bit) {
    switch (o.type) {
      case F_X: case F_Y: case F_H:
        // moves, and s(p +- a) == s(x0 +- x1) bit for bit: the lane formulas
        return lane(o, LaneC(), a, pp, bit);
      default: break;
    }
    const Cx x0{sel(pp.x, a.x, bit), sel(pp.y, a.y, bit)};
    const Cx x1{sel(a.x, pp.x, bit), sel(a.y, pp.y, bit)};
    switch (o.type) {
      case F_UR:
        return {fma(l.c2, x1.x, mul(l.c1, x0.x)), fma(l.c2, x1.y, mul(l.c1, x0.y))};
      case F_UI: {
        const std::string o1 = sel(x0.y, x0.x, bit), o2 = sel(x1.x, x1.y, bit);
        const std::string q1 = sel(x0.x, x0.y, bit), q2 = sel(x1.y, x1.x, bit);
        return {fma(l.f2, o2, mul(l.f1, o1)), fma(l.g2, q2, mul(l.g1, q1))};
      }
      default: {  // F_U2: x0 term first, as pair()
        Cx acc;
        cfma(acc, l.m1, l.n1, x0, true);
        cfma(acc, l.m2, l.n2, x1, false);
        return acc;
      }
    }
  }

  Cx shfl(const Cx& v, int t0) {
    Cx o{f(), f()};
    for (int c = 0; c < 2; ++c) {
      const std::string& src = c ? v.y : v.x;
      const std::string& dst = c ? o.y : o.x;
      if (!c64) {
        const std::string lo = r(), hi = r(), lo2 = r(), hi2 = r();
        e("mov.b64 {%s, %s}, %s;", lo.c_str(), hi.c_str(), src.c_str());
        e("shfl.sync.bfly.b32 %s, %s, %d, 31, -1;", lo2.c_str(), lo.c_str(), 1 << t0);
        e("shfl.sync.bfly.b32 %s, %s, %d, 31, -1;", hi2.c_str(), hi.c_str(), 1 << t0);
        e("mov.b64 %s, {%s, %s};", dst.c_str(), lo2.c_str(), hi2.c_str());
      } else {
        const std::string a = r(), b = r();
        e("mov.b32 %s, %s;", a.c_str(), src.c_str());
        e("shfl.sync.bfly.b32 %s, %s, %d, 31, -1;", b.c_str(), a.c_str(), 1 << t0);
        e("mov.b32 %s, %s;", dst.c_str(), b.c_str());
      }
    }
    return o;
  }

  // ---- ops -------------------------------------------------------------------
  void op_diag1(const FHdr& h) {
    const std::string end = L();
    tile_pred(h.mhi, h.phi, end);
    skip_unless(thread_pred(h.mlo, h.plo), end);
    uint32_t tm_, tv_, mr, pr;
    split(h.mlo, h.plo, tm_, tv_, mr, pr);
    bool any = false;
    for (int r = 0; r < R; ++r) any |= ((uint32_t)r & mr) == pr;
    if (any) {
      const Cx d = coef(h.coef);
      for (int r = 0; r < R; ++r)
        if (((uint32_t)r & mr) == pr) set(r, cmul(d, {vx(r), vy(r)}));
    }
    label(end);
  }

  void op_diagn(const FHdr& h) {
    const std::string end = L();
    tile_pred(h.mhi, h.phi, end);
    skip_unless(thread_pred(h.mlo, h.plo), end);
    uint32_t tm_, tv_, mr, pr;
    split(h.mlo, h.plo, tm_, tv_, mr, pr);
    const int m = h.m;
    const int ts[3] = {h.t0, h.t1, h.t2};
    std::vector<Cx> dd;
    for (int j = 0; j < (1 << m); ++j) dd.push_back(coef(h.coef + j));
    // Runtime bits of the entry index (thread bits, tile-base bits) as predicates;
    // register bits are compile-time per slot.
    std::vector<std::string> bitp(3);
    for (int s = 0; s < m; ++s) {
      const int t = ts[s];
      if (t >= 64) {
        const std::string a = rd();
        bitp[s] = p();
        e("and.b64 %s, %%base, %llu;", a.c_str(), 1ull << (t - 64));
        e("setp.ne.b64 %s, %s, 0;", bitp[s].c_str(), a.c_str());
      } else if (tbit(t) >= 0) {
        const std::string a = r();
        bitp[s] = p();
        e("and.b32 %s, %%ltid, %u;", a.c_str(), 1u << tbit(t));
        e("setp.ne.b32 %s, %s, 0;", bitp[s].c_str(), a.c_str());
      }
    }
    // Per slot: entry j = runtime bits + compile-time register bits.
    std::map<uint32_t, Cx> cache;  // compile-time part -> selected d
    for (int r = 0; r < R; ++r) {
      if (((uint32_t)r & mr) != pr) continue;
      uint32_t jc = 0;
      for (int s = 0; s < m; ++s)
        if (ts[s] < 64 && tbit(ts[s]) < 0)
          jc |= (((uint32_t)r >> reg_of(ts[s])) & 1u) << (m - 1 - s);
      auto it = cache.find(jc);
      if (it == cache.end()) {
        // Select among the entries consistent with jc by the runtime bits.
        std::vector<Cx> cand;
        std::vector<int> idx;
        for (int j = 0; j < (1 << m); ++j) {
          bool ok = true;
          for (int s = 0; s < m; ++s)
            if (ts[s] < 64 && tbit(ts[s]) < 0 &&
                (((j >> (m - 1 - s)) & 1u) != ((jc >> (m - 1 - s)) & 1u)))
              ok = false;
          if (ok) idx.push_back(j);
        }
        // Reduce by runtime bits from the least significant index bit upward.
        std::vector<Cx> lvl;
        for (int j : idx) lvl.push_back(dd[j]);
        std::vector<int> lj = idx;
        for (int s = m - 1; s >= 0; --s) {
          if (bitp[s].empty()) continue;
          std::vector<Cx> nx;
          std::vector<int> nj;
          for (size_t a = 0; a < lvl.size(); ++a) {
            if ((lj[a] >> (m - 1 - s)) & 1) continue;
            size_t b = a + 1;
            for (; b < lvl.size(); ++b)
              if (lj[b] == (lj[a] | (1 << (m - 1 - s)))) break;
            nx.push_back({sel(lvl[b].x, lvl[a].x, bitp[s]), sel(lvl[b].y, lvl[a].y, bitp[s])});
            nj.push_back(lj[a]);
          }
          lvl = nx;
          lj = nj;
        }
        it = cache.emplace(jc, lvl[0]).first;
      }
      const Cx d = it->second;
      const Cx z = cmul(d, {vx(r), vy(r)});
      if (m == 1) {
        set(r, z);
      } else {
        // if (!is_one(d)) v = d v
        const std::string q1 = p(), q2 = p();
        e("setp.eq.%s %s, %s, %s;", FT, q1.c_str(), d.x.c_str(), c64 ? "0f3F800000" : "0d3FF0000000000000");
        e("setp.eq.and.%s %s, %s, %s, %s;", FT, q2.c_str(), d.y.c_str(), zero().c_str(), q1.c_str());
        e("selp.%s %s, %s, %s, %s;", FT, vx(r).c_str(), vx(r).c_str(), z.x.c_str(), q2.c_str());
        e("selp.%s %s, %s, %s, %s;", FT, vy(r).c_str(), vy(r).c_str(), z.y.c_str(), q2.c_str());
      }
    }
    label(end);
  }

  void op_reg1q(const FHdr& h) {
    const std::string end = L();
    tile_pred(h.mhi, h.phi, end);
    const Op2 o = load_op2(h);
    const int t0 = h.t0;
    uint32_t tm_, tv_, mr, pr;
    split(h.mlo, h.plo, tm_, tv_, mr, pr);
    const std::string bt = thread_pred(h.mlo, h.plo);
    if (reg_of(t0) >= 0) {  // register-held (remapped there if it was a warp/lane bit)
      const int rb = reg_of(t0);
      skip_unless(bt, end);
      for (int r = 0; r < R; ++r) {
        if ((r >> rb) & 1) continue;
        if (((uint32_t)r & mr) != pr) continue;
        // Snapshot the slot registers: pair() may return them swapped (X, Y).
        Cx a0 = copy({vx(r), vy(r)}), a1 = copy({vx(r | (1 << rb)), vy(r | (1 << rb))});
        if (t0 < 5) {  // a lane bit of the interpreter: its lane formulas
          const Cx z0 = lane_const(o, a0, a1, 0), z1 = lane_const(o, a1, a0, 1);
          a0 = z0;
          a1 = z1;
        } else {
          pair(o, a0, a1);
        }
        set(r, a0);
        set(r | (1 << rb), a1);
      }
    } else {
      const int tl = tbit(t0);  // a lane position
      const std::string bit = p(), a = r();
      e("and.b32 %s, %%ltid, %u;", a.c_str(), 1u << tl);
      e("setp.ne.b32 %s, %s, 0;", bit.c_str(), a.c_str());
      // interpreter lane bit (tile bit < 5): its lane formulas; else pair() order
      const bool lane_form = t0 < 5;
      const LaneC lc = lane_form ? lane_coefs(o, bit) : LaneC();
      const LaneP lp = lane_form ? LaneP() : lanep_coefs(o, bit);
      for (int r = 0; r < R; ++r) {
        if (((uint32_t)r & mr) != pr) continue;
        const Cx pp = shfl({vx(r), vy(r)}, tl);
        const Cx z = lane_form ? lane(o, lc, {vx(r), vy(r)}, pp, bit)
                               : lane_pair(o, lp, {vx(r), vy(r)}, pp, bit);
        if (bt.empty()) {
          set(r, z);
        } else {
          e("selp.%s %s, %s, %s, %s;", FT, vx(r).c_str(), z.x.c_str(), vx(r).c_str(), bt.c_str());
          e("selp.%s %s, %s, %s, %s;", FT, vy(r).c_str(), z.y.c_str(), vy(r).c_str(), bt.c_str());
        }
      }
    }
    label(end);
  }

  // Index helpers for the shared-memory ops: ins0(p, t) on a runtime u32.
  std::string ins0(const std::string& pv, int t) {
    const std::string hi = r(), lo = r(), o = r();
    e("shr.b32 %s, %s, %d;", hi.c_str(), pv.c_str(), t);
    e("shl.b32 %s, %s, %d;", hi.c_str(), hi.c_str(), t + 1);
    e("and.b32 %s, %s, %u;", lo.c_str(), pv.c_str(), (1u << t) - 1);
    e("or.b32 %s, %s, %s;", o.c_str(), hi.c_str(), lo.c_str());
    return o;
  }
  // Shared address of tile element i (runtime u32).
  std::string saddr(const std::string& i) {
    const std::string a = r();
    e("mad.lo.u32 %s, %s, %d, %%tile;", a.c_str(), i.c_str(), ES);
    return a;
  }
  Cx lds(const std::string& addr, int off = 0) {
    Cx v{f(), f()};
    e("ld.shared.v2.%s {%s, %s}, [%s+%d];", FT, v.x.c_str(), v.y.c_str(), addr.c_str(), off);
    return v;
  }
  void sts(const std::string& addr, const Cx& v, int off = 0) {
    e("st.shared.v2.%s [%s+%d], {%s, %s};", FT, addr.c_str(), off, v.x.c_str(), v.y.c_str());
  }
  // Items p = tid, tid + 256, ... < total (the interpreter's strided loop);
  // `fn(pvreg)` emits one item.
  template <class F>
  void for_items(int total, F fn) {
    for (int pp = 0; pp * NT < total; ++pp) {
      const std::string pv = r();
      e("add.u32 %s, %%ltid, %d;", pv.c_str(), pp * NT);
      std::string skip;
      if ((pp + 1) * NT > total) {
        skip = L();
        const std::string q = p();
        e("setp.ge.u32 %s, %s, %d;", q.c_str(), pv.c_str(), total);
        e("@%s bra %s;", q.c_str(), skip.c_str());
      }
      fn(pv);
      if (!skip.empty()) label(skip);
    }
  }
  void pred_skip_i(const std::string& i, uint32_t mlo, uint32_t plo, const std::string& skip) {
    if (mlo == 0) return;
    const std::string t = r(), q = p();
    e("and.b32 %s, %s, %u;", t.c_str(), i.c_str(), mlo);
    e("setp.ne.b32 %s, %s, %u;", q.c_str(), t.c_str(), plo);
    e("@%s bra %s;", q.c_str(), skip.c_str());
  }

  void op_smem(const FHdr& h) {
    const std::string end = L();
    tile_pred(h.mhi, h.phi, end);
    const uint32_t T = 1u << K, mlo = h.mlo, plo = h.plo;
    switch (h.type) {
      case F_X: case F_Y: case F_H: case F_UR: case F_UI: case F_U2: {
        const Op2 o = load_op2(h);
        const int t = h.t0;
        for_items((int)(T >> 1), [&](const std::string& pv) {
          const std::string nx = L();
          const std::string i0 = ins0(pv, t);
          pred_skip_i(i0, mlo, plo, nx);
          const std::string a0a = saddr(i0);
          Cx a0 = lds(a0a), a1 = lds(a0a, (1 << t) * ES);
          pair(o, a0, a1);
          sts(a0a, a0);
          sts(a0a, a1, (1 << t) * ES);
          label(nx);
        });
        break;
      }
      case F_SWAP: {
        const int lo = h.t0 < h.t1 ? h.t0 : h.t1, hi = h.t0 < h.t1 ? h.t1 : h.t0;
        for_items((int)(T >> 2), [&](const std::string& pv) {
          const std::string nx = L();
          const std::string i = ins0(ins0(pv, lo), hi);
          pred_skip_i(i, mlo, plo, nx);
          const std::string ia = saddr(i);
          const Cx x = lds(ia, (1 << lo) * ES), y = lds(ia, (1 << hi) * ES);
          sts(ia, y, (1 << lo) * ES);
          sts(ia, x, (1 << hi) * ES);
          label(nx);
        });
        break;
      }
      case F_U4: case F_U8: {
        const int Lm = h.type == F_U4 ? 4 : 8;
        std::vector<Cx> c, nc;
        for (int j = 0; j < Lm * Lm; ++j) {
          c.push_back(coef(h.coef + j));
          nc.push_back({neg(c.back().y), ""});
        }
        int offs[8];
        int sorted[3];
        if (Lm == 4) {
          const int t0 = h.t0, t1 = h.t1;
          sorted[0] = t0 < t1 ? t0 : t1;
          sorted[1] = t0 < t1 ? t1 : t0;
          offs[0] = 0; offs[1] = 1 << t1; offs[2] = 1 << t0; offs[3] = (1 << t0) | (1 << t1);
        } else {
          const int s0 = h.t0, s1 = h.t1, s2 = h.t2;
          int a0 = s0 < s1 ? s0 : s1, a1 = s0 < s1 ? s1 : s0, a2 = s2;
          if (a2 < a1) { const int x = a1; a1 = a2; a2 = x; }
          if (a1 < a0) { const int x = a0; a0 = a1; a1 = x; }
          sorted[0] = a0; sorted[1] = a1; sorted[2] = a2;
          for (int j = 0; j < 8; ++j)
            offs[j] = (((j >> 2) & 1) << s0) | (((j >> 1) & 1) << s1) | ((j & 1) << s2);
        }
        const int nb = Lm == 4 ? 2 : 3;
        for_items((int)(T / Lm), [&](const std::string& pv) {
          const std::string nx = L();
          std::string i = pv;
          for (int b = 0; b < nb; ++b) i = ins0(i, sorted[b]);
          pred_skip_i(i, mlo, plo, nx);
          const std::string ia = saddr(i);
          std::vector<Cx> v;
          for (int j = 0; j < Lm; ++j) v.push_back(lds(ia, offs[j] * ES));
          std::vector<Cx> w(Lm);
          for (int j = 0; j < Lm; ++j)
            for (int q = 0; q < Lm; ++q) cfma(w[j], c[j * Lm + q], nc[j * Lm + q], v[q], q == 0);
          for (int j = 0; j < Lm; ++j) sts(ia, w[j], offs[j] * ES);
          label(nx);
        });
        break;
      }
      default: break;
    }
    label(end);
  }

  // Factor of diagonal member g at entry pattern ie (u32 reg), multiplied into t
  // when its predicate holds and it is not exactly one (k_fused F_DTAB build).
  void dtab_member(const FHdr& g, const std::string& ie, Cx& t) {
    const std::string skip = L();
    tile_pred(g.mhi, g.phi, skip);
    pred_skip_i(ie, g.mlo, g.plo, skip);
    Cx d;
    if (g.type == F_DIAG1) {
      d = coef(g.coef);
      if (!(d.vx == 1.0 && d.vy == 0.0)) assign(t.x, t.y, cmulf(d, t));  // is_one: compile time
      label(skip);
      return;
    } else {
      const int m = g.m;
      const int ts[3] = {g.t0, g.t1, g.t2};
      // j from the bits of ie / base (all runtime here)
      const std::string j = r();
      e("mov.u32 %s, 0;", j.c_str());
      for (int s = 0; s < m; ++s) {
        const std::string b = r();
        if (ts[s] >= 64) {
          const std::string a = rd();
          e("shr.b64 %s, %%base, %d;", a.c_str(), ts[s] - 64);
          e("cvt.u32.u64 %s, %s;", b.c_str(), a.c_str());
          e("and.b32 %s, %s, 1;", b.c_str(), b.c_str());
        } else {
          e("bfe.u32 %s, %s, %d, 1;", b.c_str(), ie.c_str(), ts[s]);
        }
        e("bfi.b32 %s, %s, %s, %d, 1;", j.c_str(), b.c_str(), j.c_str(), m - 1 - s);
      }
      // select entry j among 2^m
      d = coef(g.coef);
      for (int k = 1; k < (1 << m); ++k) {
        const Cx ck = coef(g.coef + k);
        const std::string q = p();
        e("setp.eq.u32 %s, %s, %d;", q.c_str(), j.c_str(), k);
        d = {sel(ck.x, d.x, q), sel(ck.y, d.y, q)};
      }
    }
    const std::string q1 = p(), q2 = p();
    e("setp.eq.%s %s, %s, %s;", FT, q1.c_str(), d.x.c_str(), c64 ? "0f3F800000" : "0d3FF0000000000000");
    e("setp.eq.and.%s %s, %s, %s, %s;", FT, q2.c_str(), d.y.c_str(), zero().c_str(), q1.c_str());
    e("@%s bra %s;", q2.c_str(), skip.c_str());
    assign(t.x, t.y, cmulf(d, t));
    label(skip);
  }

  // Phase tables built in the prologue, while the tile's TMA load is in flight: a table
  // depends only on the tile index and the coefficients, never on amplitudes, so every
  // table of the pass that fits is built before the first barrier and
  // each F_DTAB op is then a lookup pass with no barrier of its own (the build latency and
  // two barriers per table hide behind the load).  Entries beyond prebuild_entries() are
  // built in place as before.  Entries and arithmetic are exactly
  // op_dtab's / k_fused's, so results stay bit-identical to the interpreter.
  // Table entries built in the prologue: 32 KiB (complex128: 2 CTAs per SM with the 64 KiB
  // tile) or 8 KiB (complex64: 4 CTAs per SM with the 32 KiB tile).
  int prebuild_entries() const { return c64 ? 1024 : 2048; }
  std::map<int, int> dtab_off;  // prebuilt F_DTAB op -> entry offset in lfqs_dtab
  int dtab_pre = 0;             // entries of the prebuilt tables
  int n_dtabc = 0;              // prebuilt tables with hoisted members (lfqs_dtabc slots)
  bool dtab_dyn = false;        // some table is built in place (after the prebuilt ones)
  void plan_prebuild() {
    for (int o = 0; o < P.nops; ++o) {
      const FHdr& h = P.h[o];
      if (h.type != F_DTAB) continue;
      const int sz = 1 << __builtin_popcount(h.mlo);
      if (dtab_pre + sz <= prebuild_entries()) {
        dtab_off[o] = dtab_pre;
        dtab_pre += sz;
      } else {
        dtab_dyn = true;
      }
      o += h.m;
    }
  }
  int dtab_entries() const { return std::max(dtab_pre + (dtab_dyn ? 256 : 0), 1); }

  // Members of table `o` that hold for every entry (one-entry diagonals whose tile-bit
  // predicate is the table's common predicate; only tile bits outside the table, i.e. the
  // tile index, decide them): a per-tile factor.  With >= 2 of them the table is
  // C * partial[e] -- C their product (program order), partial[e] the other members'
  // (program order) -- exactly as k_fused builds it (fused_kernels.cu dtab_hoisted).
  static bool hoisted_member(const FHdr& g, uint32_t cm) { return g.type == F_DIAG1 && g.mlo == cm; }
  int n_hoisted(int o) const {
    const FHdr& h = P.h[o];
    const uint32_t cm = h.plo & 0xffffu;
    int k = 0;
    for (int j = 1; j <= h.m; ++j) k += hoisted_member(P.h[o + j], cm);
    return k;
  }
  // C of table o into `c` (registers): the hoisted members' product.
  void dtab_factor(int o, Cx& c) {
    const FHdr& h = P.h[o];
    const uint32_t cm = h.plo & 0xffffu;
    e("mov.%s %s, %s;", FT, c.x.c_str(), c64 ? "0f3F800000" : "0d3FF0000000000000");
    e("mov.%s %s, %s;", FT, c.y.c_str(), zero().c_str());
    for (int j = 1; j <= h.m; ++j) {
      const FHdr& g = P.h[o + j];
      if (!hoisted_member(g, cm)) continue;
      const std::string skip = L();
      tile_pred(g.mhi, g.phi, skip);
      const Cx d = coef(g.coef);
      if (!(d.vx == 1.0 && d.vy == 0.0)) assign(c.x, c.y, cmulf(d, c));
      label(skip);
    }
  }

  // Builds table `o` into lfqs_dtab entries [off, off + 2^nb): entry e by thread e mod NT.
  // hslot >= 0 (a prebuilt table with hoisted members): the entries are the partial
  // products and lane hslot / W of warp hslot % W (W warps) writes C to lfqs_dtabc[hslot]
  // -- the chains of different tables run in different warps, in parallel (dtab_finalize
  // multiplies them in after the next barrier); otherwise every thread applies C itself.
  void dtab_build(int o, int off, int hslot = -1) {
    const FHdr& h = P.h[o];
    const int nm = h.m;
    const uint32_t U = h.mlo, cm = h.plo & 0xffffu, cp = h.plo >> 16;
    const int nb = __builtin_popcount(U);
    const bool hoist = n_hoisted(o) >= 2;
    Cx c{f(), f()};
    if (hoist && hslot >= 0) {
      const std::string skip = L(), q = p();
      const int nw = NT / 32;
      e("setp.ne.u32 %s, %%ltid, %d;", q.c_str(), (hslot % nw) * 32 + hslot / nw);
      e("@%s bra %s;", q.c_str(), skip.c_str());
      dtab_factor(o, c);
      const std::string a = r();
      e("mov.u32 %s, lfqs_dtabc;", a.c_str());
      sts(a, c, hslot * ES);
      label(skip);
    } else if (hoist) {
      dtab_factor(o, c);
    }
    for (int k = 0; k * NT < (1 << nb); ++k) {
      const std::string skip = L(), q = p(), eid = r();
      e("add.u32 %s, %%ltid, %d;", eid.c_str(), k * NT);
      e("setp.ge.u32 %s, %s, %u;", q.c_str(), eid.c_str(), 1u << nb);
      e("@%s bra %s;", q.c_str(), skip.c_str());
      const std::string ie = r();
      e("mov.u32 %s, %u;", ie.c_str(), cp);
      uint32_t u = U;
      for (int b = 0; b < nb; ++b) {
        const int pos = __builtin_ctz(u);
        u &= u - 1;
        const std::string t = r();
        e("bfe.u32 %s, %s, %d, 1;", t.c_str(), eid.c_str(), b);
        e("bfi.b32 %s, %s, %s, %d, 1;", ie.c_str(), t.c_str(), ie.c_str(), pos);
      }
      Cx t{f(), f()};
      e("mov.%s %s, %s;", FT, t.x.c_str(), c64 ? "0f3F800000" : "0d3FF0000000000000");
      e("mov.%s %s, %s;", FT, t.y.c_str(), zero().c_str());
      for (int j = 1; j <= nm; ++j)
        if (!hoist || !hoisted_member(P.h[o + j], cm)) dtab_member(P.h[o + j], ie, t);
      if (hoist && hslot < 0) assign(t.x, t.y, cmulf(c, t));
      const std::string a = r();
      e("mad.lo.u32 %s, %s, %d, %%dtab;", a.c_str(), eid.c_str(), ES);
      sts(a, t, off * ES);
      label(skip);
    }
  }
  // After the barrier that follows the prologue builds: entries of the prebuilt tables
  // with hoisted members times their C (each thread its own entries).
  void dtab_finalize(int o, int off, int hslot) {
    const FHdr& h = P.h[o];
    const int nb = __builtin_popcount(h.mlo);
    const std::string ca = r();
    e("mov.u32 %s, lfqs_dtabc;", ca.c_str());
    const Cx c = lds(ca, hslot * ES);
    for (int k = 0; k * NT < (1 << nb); ++k) {
      const std::string skip = L(), q = p(), eid = r();
      e("add.u32 %s, %%ltid, %d;", eid.c_str(), k * NT);
      e("setp.ge.u32 %s, %s, %u;", q.c_str(), eid.c_str(), 1u << nb);
      e("@%s bra %s;", q.c_str(), skip.c_str());
      const std::string a = r();
      e("mad.lo.u32 %s, %s, %d, %%dtab;", a.c_str(), eid.c_str(), ES);
      const Cx t = lds(a, off * ES);
      sts(a, cmulf(c, t), off * ES);
      label(skip);
    }
  }

  void op_dtab(int o) {
    const FHdr& h = P.h[o];
    const int nm = h.m;
    const uint32_t U = h.mlo, cm = h.plo & 0xffffu, cp = h.plo >> 16;
    const auto pre = dtab_off.find(o);
    const int toff = pre != dtab_off.end() ? pre->second : dtab_pre;
    if (pre != dtab_off.end()) {
      ensure_regs(o + nm + 1);
    } else {
      sync();
      dtab_build(o, toff);
      if (!in_regs) {
        if (greedy && nreg >= 1) {
          place(plan_set(o + nm + 1), o + nm + 1);
          emit_taddr();
        }
        tile_to_regs();
        in_regs = true;
      }
      sync();
    }
    const std::string end = L();
    skip_unless(thread_pred(cm, cp), end);
    // e(i) = pext(i, U): table-index bit k is tile bit u_k, held by a thread bit
    // (runtime, et) or a slot bit (compile time, w[j]).
    const std::string et = r();
    e("mov.u32 %s, 0;", et.c_str());
    uint32_t w[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    uint32_t u = U;
    for (int k = 0; u; ++k) {
      const int pos = __builtin_ctz(u);
      u &= u - 1;
      if (tbit(pos) >= 0) {
        const std::string t = r();
        e("bfe.u32 %s, %%ltid, %d, 1;", t.c_str(), tbit(pos));
        e("bfi.b32 %s, %s, %s, %d, 1;", et.c_str(), t.c_str(), et.c_str(), k);
      } else {
        w[reg_of(pos)] = 1u << k;
      }
    }
    const std::string ebase = r();
    e("mad.lo.u32 %s, %s, %d, %%dtab;", ebase.c_str(), et.c_str(), ES);
    if (toff) e("add.u32 %s, %s, %d;", ebase.c_str(), ebase.c_str(), toff * ES);
    uint32_t ctm, ctv, crm, crp;
    split(cm, cp, ctm, ctv, crm, crp);
    for (int r_ = 0; r_ < R; ++r_) {
      if (((uint32_t)r_ & crm) != crp) continue;
      uint32_t off = 0;
      for (int b = 0; b < nreg; ++b)
        if ((r_ >> b) & 1) off += w[b];
      const Cx d = lds(ebase, (int)off * ES);
      set(r_, cmulf(d, {vx(r_), vy(r_)}));
    }
    label(end);
  }

  // Tile -> registers after the tile was last written in shared memory (smem ops,
  // phase-table builds): the placement may change for free here, so with greedy
  // placement the register positions are chosen for the ops from `o` on.
  void ensure_regs(int o) {
    if (!in_regs) {
      sync();
      if (greedy && nreg >= 1) {
        place(plan_set(o), o);
        emit_taddr();
      }
      tile_to_regs();
      in_regs = true;
    }
  }
  // Register-position requirement of op o: 0 none (diagonal, fixed-lane shuffle),
  // 1 its targets in `bits`, 2 it runs as a shared-memory op.
  int op_need(int o, uint32_t& bits) const {
    const FHdr& h = P.h[o];
    bits = 0;
    if (h.type == F_DTAB || h.type == F_DIAG1 || h.type == F_DIAGN) return 0;
    int ts[3];
    const int m = op_targets(h, ts);
    bool anyl = false;
    for (int s_ = 0; s_ < m; ++s_) anyl |= fixed_lane(ts[s_]);
    if (m == 1) {
      if (anyl) return 0;
      if (nreg < 1) return 2;
      bits = 1u << ts[0];
      return 1;
    }
    if (lane_reg2 && m == 2 && nreg >= 1 && (h.type == F_U4 || h.type == F_SWAP) &&
        fixed_lane(ts[0]) != fixed_lane(ts[1])) {
      bits = 1u << (fixed_lane(ts[0]) ? ts[1] : ts[0]);
      return 1;
    }
    if (lane_reg2 && m == 2 && (h.type == F_U4 || h.type == F_SWAP) && fixed_lane(ts[0]) &&
        fixed_lane(ts[1]))
      return 0;  // op_lanelane2: shuffles only
    if (anyl || m > nreg) return 2;
    for (int s_ = 0; s_ < m; ++s_) bits |= 1u << ts[s_];
    return 1;
  }
  // Greedy placement (LFQS_OPT_JIT_GREEDY_PLACE): one tile round trip costs the same
  // whatever number of bits it moves, so a remap takes into register positions the
  // targets of the longest run of upcoming ops whose register requirements fit
  // nreg positions together (interval covering: the fewest round trips).
  uint32_t plan_set(int o) const {
    if (pool) return plan_pool(o);
    uint32_t S = 0;
    for (int q = o; q < P.nops; ++q) {
      if (P.h[q].type == F_DTAB) {
        q += P.h[q].m;
        continue;
      }
      uint32_t b;
      const int k = op_need(q, b);
      if (k == 0) continue;
      if (k == 2 || __builtin_popcount(S | b) > nreg) break;
      S |= b;
    }
    return S;
  }
  // Placement change (no code): every bit of S not register-held takes the register
  // position of a bit outside S, the one with the furthest next use first.
  // Lane-pool requirement / plan: 1-target gates and SWAP / U4 need their non-fixed-lane
  // targets at cheap positions (registers or movable lanes); an 8x8 gate ends the run.
  uint32_t plan_pool(int o) const {
    const int npool = nreg + (5 - FL);
    uint32_t S = 0;
    for (int q = o; q < P.nops; ++q) {
      const FHdr& h = P.h[q];
      if (h.type == F_DTAB) {
        q += h.m;
        continue;
      }
      if (h.type == F_DIAG1 || h.type == F_DIAGN) continue;
      if (h.type == F_U8) break;
      int ts[3];
      const int m = op_targets(h, ts);
      uint32_t b = 0;
      for (int s_ = 0; s_ < m; ++s_)
        if (!fixed_lane(ts[s_])) b |= 1u << ts[s_];
      if (__builtin_popcount(S | b) > npool) break;
      S |= b;
    }
    return S;
  }
  void place_pool(uint32_t S, int o) {
    for (int b = 0; b < K; ++b) {
      if (!((S >> b) & 1) || cheap(b)) continue;
      // victim: a cheap position holding a bit outside S, furthest next use (ties: register)
      int best_r = -1, best_l = -1, bd = -1;
      for (int j = 0; j < nreg; ++j) {
        if ((S >> rpos[j]) & 1) continue;
        const int d = next_use(rpos[j], o);
        if (d > bd) { bd = d; best_r = j; best_l = -1; }
      }
      for (int j = FL; j < 5; ++j) {
        if ((S >> tpos[j]) & 1) continue;
        const int d = next_use(tpos[j], o);
        if (d > bd) { bd = d; best_l = j; best_r = -1; }
      }
      const int tb = tbit(b);
      if (best_r >= 0) {
        tpos[tb] = rpos[best_r];
        rpos[best_r] = b;
      } else {
        tpos[tb] = tpos[best_l];
        tpos[best_l] = b;
      }
    }
  }
  void place(uint32_t S, int o) {
    if (pool) {
      place_pool(S, o);
      return;
    }
    for (int b = 0; b < K; ++b) {
      if (!((S >> b) & 1) || reg_of(b) >= 0) continue;
      int best = -1, bd = -1;
      for (int j = 0; j < nreg; ++j) {
        if ((S >> rpos[j]) & 1) continue;
        const int d = next_use(rpos[j], o);
        if (d > bd) {
          bd = d;
          best = j;
        }
      }
      tpos[tbit(b)] = rpos[best];
      rpos[best] = b;
    }
  }
  static int op_targets(const FHdr& h, int* ts) {
    ts[0] = h.t0;
    ts[1] = h.t1;
    ts[2] = h.t2;
    switch (h.type) {
      case F_SWAP: case F_U4: return 2;
      case F_U8: return 3;
      default: return 1;
    }
  }
  // Ops until tile bit b is next a target of a non-diagonal op (Belady distance).
  int next_use(int b, int from) const {
    for (int o = from; o < P.nops; ++o) {
      const FHdr& h = P.h[o];
      if (h.type == F_DTAB) {
        o += h.m;
        continue;
      }
      if (h.type == F_DIAG1 || h.type == F_DIAGN) continue;
      int ts[3];
      const int m = op_targets(h, ts);
      for (int s_ = 0; s_ < m; ++s_)
        if (ts[s_] == b) return o - from;
    }
    return 1 << 30;
  }
  // Moves the warp-held tile bits `need` into register positions (evicting, by
  // furthest next use, register-held bits that are not targets of op o) with one
  // round trip through the shared-memory tile.
  void remap(const std::vector<int>& need, const int* ts, int m, int o) {
    body += "  // remap\n";
    int ot[9], orp[8];
    std::memcpy(ot, tpos, sizeof ot);
    std::memcpy(orp, rpos, sizeof orp);
    const bool partial = partial_rt && in_regs;
    if (in_regs && !partial) regs_to_tile();  // under the old placement
    if (greedy) {
      place(plan_set(o), o);
    } else for (int b : need) {
      int best = -1, bd = -1;
      for (int j = 0; j < nreg; ++j) {
        bool tgt = false;
        for (int s_ = 0; s_ < m; ++s_) tgt |= rpos[j] == ts[s_];
        if (tgt) continue;
        const int d = next_use(rpos[j], o + 1);
        if (d > bd) {
          bd = d;
          best = j;
        }
      }
      tpos[tbit(b)] = rpos[best];
      rpos[best] = b;
    }
    if (partial) {
      partial_roundtrip(ot, orp);
      return;
    }
    sync();
    emit_taddr();
    tile_to_regs();
    in_regs = true;
  }

  // SWAP / U4 with one target at a fixed lane position (a) and the other register-held
  // (b): the partner lane (lane ^ 2^tbit(a)) holds the other half of every group, fetched
  // by shuffles, so the gate needs no shared-memory round trip.  The group values are
  // put in local-index order and each output is the interpreter's sum over q ascending
  // (F_U4) or its move (F_SWAP): bit-identical.
  void op_lanereg2(const FHdr& h) {
    const std::string end = L();
    tile_pred(h.mhi, h.phi, end);
    const bool a_is_t0 = at_lane(h.t0) && reg_of(h.t1) >= 0;
    const int ta = a_is_t0 ? h.t0 : h.t1, tb = a_is_t0 ? h.t1 : h.t0;
    const int tl = tbit(ta), rb = reg_of(tb);
    // local index j = 2 bit(t0) + bit(t1)
    auto jidx = [&](int av, int bv) { return a_is_t0 ? (av << 1) | bv : (bv << 1) | av; };
    uint32_t tm_, tv_, mr, pr;
    split(h.mlo, h.plo, tm_, tv_, mr, pr);
    const std::string bt = thread_pred(h.mlo, h.plo);
    const std::string x = p(), xa = r();
    e("and.b32 %s, %%ltid, %u;", xa.c_str(), 1u << tl);
    e("setp.ne.b32 %s, %s, 0;", x.c_str(), xa.c_str());
    // Coefficient rows of this thread's two outputs (a = x, b = 0 / 1), selected once.
    std::vector<Cx> row[2], nrow[2];
    if (h.type == F_U4) {
      std::vector<Cx> c, nc;
      for (int k = 0; k < 16; ++k) {
        c.push_back(coef(h.coef + k));
        nc.push_back({c.back().zy() ? std::string() : neg(c.back().y), ""});
      }
      for (int bv = 0; bv < 2; ++bv)
        for (int q = 0; q < 4; ++q) {
          const int j1 = jidx(1, bv), j0 = jidx(0, bv);
          row[bv].push_back(sel_c(c[j1 * 4 + q], c[j0 * 4 + q], x));
          const Cx& n1 = nc[j1 * 4 + q];
          const Cx& n0 = nc[j0 * 4 + q];
          if (row[bv].back().zy())
            nrow[bv].push_back({std::string(), ""});
          else
            nrow[bv].push_back({sel(n1.x.empty() ? zero() : n1.x, n0.x.empty() ? zero() : n0.x, x), ""});
        }
    }
    for (int r_ = 0; r_ < R; ++r_) {
      if ((r_ >> rb) & 1) continue;
      if (((uint32_t)r_ & mr) != pr) continue;
      const int r1 = r_ | (1 << rb);
      const Cx A0 = copy({vx(r_), vy(r_)}), A1 = copy({vx(r1), vy(r1)});
      const Cx P0 = shfl(A0, tl), P1 = shfl(A1, tl);
      Cx o0, o1;
      if (h.type == F_SWAP) {
        // new(a, b) = old(b, a): (x, 0) <- old(0, x); (x, 1) <- old(1, x)
        o0 = {sel(P1.x, A0.x, x), sel(P1.y, A0.y, x)};
        o1 = {sel(A1.x, P0.x, x), sel(A1.y, P0.y, x)};
      } else {
        // group values by local index: (a = x) own, (a = 1 - x) partner
        Cx v[4];
        for (int bv = 0; bv < 2; ++bv) {
          const Cx& own = bv ? A1 : A0;
          const Cx& par = bv ? P1 : P0;
          v[jidx(0, bv)] = {sel(par.x, own.x, x), sel(par.y, own.y, x)};
          v[jidx(1, bv)] = {sel(own.x, par.x, x), sel(own.y, par.y, x)};
        }
        for (int q = 0; q < 4; ++q) cfma(o0, row[0][q], nrow[0][q], v[q], q == 0);
        for (int q = 0; q < 4; ++q) cfma(o1, row[1][q], nrow[1][q], v[q], q == 0);
      }
      if (bt.empty()) {
        set(r_, o0);
        set(r1, o1);
      } else {
        e("selp.%s %s, %s, %s, %s;", FT, vx(r_).c_str(), o0.x.c_str(), vx(r_).c_str(), bt.c_str());
        e("selp.%s %s, %s, %s, %s;", FT, vy(r_).c_str(), o0.y.c_str(), vy(r_).c_str(), bt.c_str());
        e("selp.%s %s, %s, %s, %s;", FT, vx(r1).c_str(), o1.x.c_str(), vx(r1).c_str(), bt.c_str());
        e("selp.%s %s, %s, %s, %s;", FT, vy(r1).c_str(), o1.y.c_str(), vy(r1).c_str(), bt.c_str());
      }
    }
    label(end);
  }

  // Shuffle by source lane (idx mode).
  Cx shfl_idx(const Cx& v, const std::string& src) {
    Cx o{f(), f()};
    for (int c = 0; c < 2; ++c) {
      const std::string& sv = c ? v.y : v.x;
      const std::string& dv = c ? o.y : o.x;
      if (!c64) {
        const std::string lo = r(), hi = r(), lo2 = r(), hi2 = r();
        e("mov.b64 {%s, %s}, %s;", lo.c_str(), hi.c_str(), sv.c_str());
        e("shfl.sync.idx.b32 %s, %s, %s, 31, -1;", lo2.c_str(), lo.c_str(), src.c_str());
        e("shfl.sync.idx.b32 %s, %s, %s, 31, -1;", hi2.c_str(), hi.c_str(), src.c_str());
        e("mov.b64 %s, {%s, %s};", dv.c_str(), lo2.c_str(), hi2.c_str());
      } else {
        const std::string a = r(), b = r();
        e("mov.b32 %s, %s;", a.c_str(), sv.c_str());
        e("shfl.sync.idx.b32 %s, %s, %s, 31, -1;", b.c_str(), a.c_str(), src.c_str());
        e("mov.b32 %s, %s;", dv.c_str(), b.c_str());
      }
    }
    return o;
  }

  // SWAP / U4 with both targets at fixed lane positions: the four lanes that differ
  // only in the two target bits hold a group (one amplitude per slot each); every lane
  // gathers the group in local-index order by idx shuffles and computes its own output
  // with the interpreter's sum (F_U4) or move (F_SWAP) -- bit-identical, no tile round
  // trip and no strided shared-memory items.
  void op_lanelane2(const FHdr& h) {
    const std::string end = L();
    tile_pred(h.mhi, h.phi, end);
    const int l0 = tbit(h.t0), l1 = tbit(h.t1);  // lane bits of the local index MSB / LSB
    uint32_t tm_, tv_, mr, pr;
    split(h.mlo, h.plo, tm_, tv_, mr, pr);
    const std::string bt = thread_pred(h.mlo, h.plo);
    const std::string b0 = p(), b1 = p(), a0 = r(), a1 = r();
    e("and.b32 %s, %%ltid, %u;", a0.c_str(), 1u << l0);
    e("setp.ne.b32 %s, %s, 0;", b0.c_str(), a0.c_str());
    e("and.b32 %s, %%ltid, %u;", a1.c_str(), 1u << l1);
    e("setp.ne.b32 %s, %s, 0;", b1.c_str(), a1.c_str());
    const std::string base = r();
    e("and.b32 %s, %%ltid, %u;", base.c_str(), 31u & ~((1u << l0) | (1u << l1)));
    if (h.type == F_SWAP) {
      // new(x0, x1) = old(x1, x0): source lane with the two bits exchanged
      const std::string src = r(), t = r(), u = r();
      e("shr.u32 %s, %s, %d;", t.c_str(), a0.c_str(), l0);
      e("shl.b32 %s, %s, %d;", t.c_str(), t.c_str(), l1);
      e("shr.u32 %s, %s, %d;", u.c_str(), a1.c_str(), l1);
      e("shl.b32 %s, %s, %d;", u.c_str(), u.c_str(), l0);
      e("or.b32 %s, %s, %s;", src.c_str(), base.c_str(), t.c_str());
      e("or.b32 %s, %s, %s;", src.c_str(), src.c_str(), u.c_str());
      for (int r_ = 0; r_ < R; ++r_) {
        if (((uint32_t)r_ & mr) != pr) continue;
        const Cx o = shfl_idx({vx(r_), vy(r_)}, src);
        if (bt.empty()) {
          set(r_, o);
        } else {
          e("selp.%s %s, %s, %s, %s;", FT, vx(r_).c_str(), o.x.c_str(), vx(r_).c_str(), bt.c_str());
          e("selp.%s %s, %s, %s, %s;", FT, vy(r_).c_str(), o.y.c_str(), vy(r_).c_str(), bt.c_str());
        }
      }
      label(end);
      return;
    }
    std::string src[4];
    for (int q = 0; q < 4; ++q) {
      src[q] = r();
      e("or.b32 %s, %s, %u;", src[q].c_str(), base.c_str(),
        (uint32_t)(((q >> 1) & 1) << l0) | (uint32_t)((q & 1) << l1));
    }
    // coefficient row of this lane's local index j = 2 b0 + b1, selected once
    std::vector<Cx> c, nc;
    for (int k = 0; k < 16; ++k) {
      c.push_back(coef(h.coef + k));
      nc.push_back({c.back().zy() ? zero() : neg(c.back().y), ""});
    }
    std::vector<Cx> row, nrow;
    for (int q = 0; q < 4; ++q) {
      const Cx lo = sel_c(c[1 * 4 + q], c[0 * 4 + q], b1);   // j = 0 / 1
      const Cx hi = sel_c(c[3 * 4 + q], c[2 * 4 + q], b1);   // j = 2 / 3
      row.push_back(sel_c(hi, lo, b0));
      const std::string nlo = sel(nc[1 * 4 + q].x, nc[0 * 4 + q].x, b1);
      const std::string nhi = sel(nc[3 * 4 + q].x, nc[2 * 4 + q].x, b1);
      nrow.push_back({sel(nhi, nlo, b0), ""});
    }
    for (int r_ = 0; r_ < R; ++r_) {
      if (((uint32_t)r_ & mr) != pr) continue;
      Cx v[4];
      for (int q = 0; q < 4; ++q) v[q] = shfl_idx({vx(r_), vy(r_)}, src[q]);
      Cx o;
      for (int q = 0; q < 4; ++q) cfma(o, row[q], nrow[q], v[q], q == 0);
      if (bt.empty()) {
        set(r_, o);
      } else {
        e("selp.%s %s, %s, %s, %s;", FT, vx(r_).c_str(), o.x.c_str(), vx(r_).c_str(), bt.c_str());
        e("selp.%s %s, %s, %s, %s;", FT, vy(r_).c_str(), o.y.c_str(), vy(r_).c_str(), bt.c_str());
      }
    }
    label(end);
  }

  // SWAP / U4 / U8 with every target register-held.
  void op_regmulti(const FHdr& h) {
    const std::string end = L();
    tile_pred(h.mhi, h.phi, end);
    skip_unless(thread_pred(h.mlo, h.plo), end);
    uint32_t tm_, tv_, mr, pr;
    split(h.mlo, h.plo, tm_, tv_, mr, pr);
    if (h.type == F_SWAP) {
      const int j0 = reg_of(h.t0), j1 = reg_of(h.t1);
      for (int r_ = 0; r_ < R; ++r_) {
        if (((r_ >> j0) & 1) || ((r_ >> j1) & 1)) continue;
        if (((uint32_t)r_ & mr) != pr) continue;
        const int x = r_ | (1 << j0), y = r_ | (1 << j1);
        const Cx a = copy({vx(x), vy(x)}), b = copy({vx(y), vy(y)});
        set(x, b);
        set(y, a);
      }
      label(end);
      return;
    }
    const int Lm = h.type == F_U4 ? 4 : 8;
    std::vector<Cx> c, nc;
    for (int j = 0; j < Lm * Lm; ++j) {
      c.push_back(coef(h.coef + j));
      nc.push_back({c.back().zy() ? std::string() : neg(c.back().y), ""});
    }
    int sb[3] = {reg_of(h.t0), reg_of(h.t1), Lm == 8 ? reg_of(h.t2) : -1};
    for (int r_ = 0; r_ < R; ++r_) {
      bool clear = true;
      for (int q = 0; q < (Lm == 4 ? 2 : 3); ++q) clear &= !((r_ >> sb[q]) & 1);
      if (!clear || ((uint32_t)r_ & mr) != pr) continue;
      int idx[8];
      for (int j = 0; j < Lm; ++j) {
        idx[j] = r_;
        if (Lm == 4) {
          if ((j >> 1) & 1) idx[j] |= 1 << sb[0];
          if (j & 1) idx[j] |= 1 << sb[1];
        } else {
          if ((j >> 2) & 1) idx[j] |= 1 << sb[0];
          if ((j >> 1) & 1) idx[j] |= 1 << sb[1];
          if (j & 1) idx[j] |= 1 << sb[2];
        }
      }
      std::vector<Cx> v, w(Lm);
      for (int j = 0; j < Lm; ++j) v.push_back({vx(idx[j]), vy(idx[j])});
      for (int j = 0; j < Lm; ++j)
        for (int q = 0; q < Lm; ++q) cfma(w[j], c[j * Lm + q], nc[j * Lm + q], v[q], q == 0);
      for (int j = 0; j < Lm; ++j) set(idx[j], w[j]);
    }
    label(end);
  }

  // Lane-pool dispatch: every target of a 1-target gate or SWAP / U4 at a cheap
  // position (register or lane) after at most one greedy round trip; 1-target gates at a
  // lane run by shuffle, 2-target gates by registers / shuffles (regmulti, lanereg2,
  // lanelane2); 8x8 gates in registers when all three targets are there, else as a
  // shared-memory op.
  void dispatch_pool(int o, const FHdr& h, const int* ts, int m) {
    if (h.type == F_U8) {
      if (reg_of(ts[0]) >= 0 && reg_of(ts[1]) >= 0 && reg_of(ts[2]) >= 0) {
        ensure_regs(o);
        op_regmulti(h);
      } else {
        if (in_regs) {
          regs_to_tile();
          in_regs = false;
        }
        sync();
        op_smem(h);
      }
      return;
    }
    bool ok = true;
    for (int s_ = 0; s_ < m; ++s_) ok &= fixed_lane(ts[s_]) || cheap(ts[s_]);
    if (!ok) {
      body += "  // remap\n";
      int ot[9], orp[8];
      std::memcpy(ot, tpos, sizeof ot);
      std::memcpy(orp, rpos, sizeof orp);
      const bool partial = partial_rt && in_regs;
      if (in_regs && !partial) regs_to_tile();
      place_pool(plan_pool(o), o);
      if (partial) {
        partial_roundtrip(ot, orp);
      } else {
        sync();
        emit_taddr();
        tile_to_regs();
        in_regs = true;
      }
    }
    ensure_regs(o);
    if (m == 1) {
      op_reg1q(h);
      return;
    }
    const bool r0 = reg_of(ts[0]) >= 0, r1 = reg_of(ts[1]) >= 0;
    if (r0 && r1)
      op_regmulti(h);
    else if (!r0 && !r1)
      op_lanelane2(h);
    else
      op_lanereg2(h);
  }

  // ---- whole kernel -------------------------------------------------------------
  std::string build() {
    const FTile& tg = P.tile;
    const uint32_t T = 1u << K;
    const uint32_t bytes = T * ES, chunk_bytes = (uint32_t)ES << tg.lc;
    const int nch = 1 << tg.nh;
    plan_prebuild();
    // prologue: base, TMA load
    e("ld.param.u64 %%ga, [pa];");
    e("cvta.to.global.u64 %%ga, %%ga;");
    e("mov.u32 %%ltid, %%tid.x;");
    e("mov.u32 %%bid, %%ctaid.x;");
    e("cvt.u64.u32 %%base, %%bid;");
    // tile-index insertions (kNoTileIns: none): the fixed bits of a block of the state
    e("ld.param.u64 %%toff, [poff];");
    for (int i = 0; i < 3; ++i) {
      const std::string x = rd(), b = r(), pp = r(), vv = r(), m = rd(), lo = rd(), v64 = rd();
      e("shr.u64 %s, %%toff, %d;", x.c_str(), 8 * i);
      e("cvt.u32.u64 %s, %s;", b.c_str(), x.c_str());
      e("and.b32 %s, %s, 63;", pp.c_str(), b.c_str());
      e("bfe.u32 %s, %s, 6, 1;", vv.c_str(), b.c_str());
      e("mov.b64 %s, 1;", m.c_str());
      e("shl.b64 %s, %s, %s;", m.c_str(), m.c_str(), pp.c_str());
      e("sub.u64 %s, %s, 1;", m.c_str(), m.c_str());
      e("and.b64 %s, %%base, %s;", lo.c_str(), m.c_str());
      e("sub.u64 %%base, %%base, %s;", lo.c_str());
      e("shl.b64 %%base, %%base, 1;");
      e("or.b64 %%base, %%base, %s;", lo.c_str());
      e("cvt.u64.u32 %s, %s;", v64.c_str(), vv.c_str());
      e("shl.b64 %s, %s, %s;", v64.c_str(), v64.c_str(), pp.c_str());
      e("or.b64 %%base, %%base, %s;", v64.c_str());
    }
    e("shl.b64 %%base, %%base, %d;", tg.lc);
    for (int i = 0; i < tg.nh; ++i) {
      const int pp = tg.hpos[i];
      const std::string lo = rd();
      e("and.b64 %s, %%base, %llu;", lo.c_str(), (unsigned long long)((1ull << pp) - 1));
      e("sub.u64 %%base, %%base, %s;", lo.c_str());
      e("shl.b64 %%base, %%base, 1;");
      e("or.b64 %%base, %%base, %s;", lo.c_str());
    }
    e("mov.u32 %%tile, lfqs_tile;");
    e("mov.u32 %%dtab, lfqs_dtab;");
    e("mov.u32 %%bar, lfqs_bar;");
    // The first tile -> registers transfer is free to choose the placement too.
    if (greedy && nreg >= 1) place(plan_set(0), 0);
    emit_taddr();
    {
      const std::string w0 = L(), q = p(), q0 = p();
      e("setp.ge.u32 %s, %%ltid, 32;", q.c_str());
      e("@%s bra %s;", q.c_str(), w0.c_str());
      e("setp.eq.u32 %s, %%ltid, 0;", q0.c_str());
      const std::string s0 = L();
      e("@!%s bra %s;", q0.c_str(), s0.c_str());
      e("mbarrier.init.shared::cta.b64 [%%bar], 1;");
      e("fence.mbarrier_init.release.cluster;");
      e("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%%bar], %u;", bytes);
      label(s0);
      e("bar.warp.sync -1;");
      chunk_loop(nch, chunk_bytes, true);
      label(w0);
    }
    // while the tile loads; tables with hoisted members: partial entries here, C by one
    // thread each, multiplied in after the barrier
    std::vector<std::pair<int, int>> fin;  // (table op, slot)
    for (const auto& t : dtab_off) {
      const int hs = n_hoisted(t.first) >= 2 && (int)fin.size() < NT ? (int)fin.size() : -1;
      if (hs >= 0) fin.emplace_back(t.first, hs);
      dtab_build(t.first, t.second, hs);
    }
    sync();
    if (!fin.empty()) {
      for (const auto& t : fin) dtab_finalize(t.first, dtab_off[t.first], t.second);
      sync();
    }
    n_dtabc = (int)fin.size();
    {
      const std::string wt = L(), q = p();
      label(wt);
      e("mbarrier.try_wait.parity.shared::cta.b64 %s, [%%bar], 0;", q.c_str());
      e("@!%s bra %s;", q.c_str(), wt.c_str());
    }
    tile_to_regs();
    in_regs = true;
    for (int o = 0; o < P.nops; ++o) {
      const FHdr& h = P.h[o];
      const int type = h.type;
      body += "  // op " + std::to_string(o) + " type " + std::to_string(type) + " t " +
              std::to_string(h.t0) + "," + std::to_string(h.t1) + "," + std::to_string(h.t2) +
              " m " + std::to_string(h.m) + " regs";
      for (int j = 0; j < nreg; ++j) body += " " + std::to_string(rpos[j]);
      body += "\n";
      if (type == F_DTAB) {
        op_dtab(o);
        o += h.m;
        continue;
      }
      if (type == F_DIAG1 || type == F_DIAGN) {
        ensure_regs(o);
        if (type == F_DIAG1)
          op_diag1(h);
        else
          op_diagn(h);
        continue;
      }
      int ts[3];
      const int m = op_targets(h, ts);
      if (pool) {
        dispatch_pool(o, h, ts, m);
        continue;
      }
      bool any_lane = false;
      for (int s_ = 0; s_ < m; ++s_) any_lane |= fixed_lane(ts[s_]);
      // 1-target gates: fixed lane bits by shuffle, everything else in registers (a
      // warp or movable lane bit is first moved into a register position).
      // Multi-target gates: in registers when no target is at a fixed lane position
      // and they fit the register positions.
      const bool in_reg_path = m == 1 ? (any_lane || nreg >= 1) : (!any_lane && m <= nreg);
      // SWAP / U4 with exactly one fixed-lane target: shuffles + registers.
      const bool lanereg = lane_reg2 && !in_reg_path && m == 2 && nreg >= 1 &&
                           (h.type == F_U4 || h.type == F_SWAP) &&
                           (fixed_lane(ts[0]) != fixed_lane(ts[1]));
      const bool lanelane = lane_reg2 && !in_reg_path && m == 2 &&
                            (h.type == F_U4 || h.type == F_SWAP) && fixed_lane(ts[0]) &&
                            fixed_lane(ts[1]);
      if (lanelane) {
        ensure_regs(o);
        op_lanelane2(h);
      } else if (lanereg) {
        const int tb = fixed_lane(ts[0]) ? ts[1] : ts[0];
        if (reg_of(tb) < 0) {
          std::vector<int> need{tb};
          remap(need, ts, m, o);
        }
        ensure_regs(o);
        op_lanereg2(h);
      } else if (in_reg_path) {
        std::vector<int> need;
        for (int s_ = 0; s_ < m; ++s_)
          if (!fixed_lane(ts[s_]) && reg_of(ts[s_]) < 0) need.push_back(ts[s_]);
        if (!need.empty()) remap(need, ts, m, o);
        ensure_regs(o);
        if (m == 1)
          op_reg1q(h);
        else
          op_regmulti(h);
      } else {
        if (in_regs) {
          regs_to_tile();
          in_regs = false;
        }
        sync();
        op_smem(h);
      }
    }
    if (in_regs) regs_to_tile();
    e("fence.proxy.async.shared::cta;");
    sync();
    {
      const std::string w0 = L(), q = p();
      e("setp.ge.u32 %s, %%ltid, 32;", q.c_str());
      e("@%s bra %s;", q.c_str(), w0.c_str());
      chunk_loop(nch, chunk_bytes, false);
      e("cp.async.bulk.commit_group;");
      e("cp.async.bulk.wait_group.read 0;");
      label(w0);
    }
    e("ret;");

    std::string out;
    out += ".version 8.7\n.target sm_100a\n.address_size 64\n\n";
    out += ".extern .shared .align 128 .b8 lfqs_tile[];\n";
    out += ".shared .align 8 .b64 lfqs_bar;\n";
    out += ".shared .align 16 .b8 lfqs_dtab[" + std::to_string(dtab_entries() * ES) + "];\n";
    out += ".shared .align 16 .b8 lfqs_dtabc[" + std::to_string(std::max(n_dtabc, 1) * ES) + "];\n\n";
    const int nc = P.ncoef > 0 ? P.ncoef : 1;
    out += ".visible .entry lfqs_jit(.param .u64 pa, .param .u64 poff, .param .align 16 .b8 pc[" +
           std::to_string(nc * 16) + "])\n";
    out += ".maxntid " + std::to_string(NT) + ", 1, 1\n.minnctapersm " +
           std::to_string(min_ctas()) + "\n{\n";
    out += "  .reg .pred %p<" + std::to_string(np + 1) + ">;\n";
    out += "  .reg .b32 %r<" + std::to_string(nr + 1) + ">;\n";
    out += "  .reg .b64 %rd<" + std::to_string(nrd + 1) + ">;\n";
    out += "  .reg .f64 %dd<" + std::to_string(nrd + 1) + ">;\n";
    out += std::string("  .reg .") + FT + " %f<" + std::to_string(nf + 1) + ">;\n";
    out += std::string("  .reg .") + FT + " %vx<" + std::to_string(R) + ">;\n";
    out += std::string("  .reg .") + FT + " %vy<" + std::to_string(R) + ">;\n";
    out += "  .reg .b64 %ga, %base, %toff;\n  .reg .b32 %ltid, %bid, %tile, %dtab, %bar, %taddr;\n";
    out += body;
    out += "}\n";
    return out;
  }

  // Chunk copies by the lanes of warp 0: chunk ch = lane + 32 k.
  void chunk_loop(int nch, uint32_t chunk_bytes, bool load) {
    const FTile& tg = P.tile;
    for (int k = 0; k * 32 < nch; ++k) {
      const std::string skip = L();
      const std::string ch = r();
      e("add.u32 %s, %%ltid, %d;", ch.c_str(), 32 * k);
      if (nch < 32 * (k + 1)) {
        const std::string q = p();
        e("setp.ge.u32 %s, %s, %d;", q.c_str(), ch.c_str(), nch);
        e("@%s bra %s;", q.c_str(), skip.c_str());
      }
      // off = base | deposit(ch) at hpos
      const std::string off = rd();
      e("mov.b64 %s, %%base;", off.c_str());
      for (int i = 0; i < tg.nh; ++i) {
        const std::string b = r(), b64 = rd();
        e("bfe.u32 %s, %s, %d, 1;", b.c_str(), ch.c_str(), i);
        e("cvt.u64.u32 %s, %s;", b64.c_str(), b.c_str());
        e("shl.b64 %s, %s, %d;", b64.c_str(), b64.c_str(), tg.hpos[i]);
        e("or.b64 %s, %s, %s;", off.c_str(), off.c_str(), b64.c_str());
      }
      const std::string ga = rd(), sa = r();
      e("mad.lo.u64 %s, %s, %d, %%ga;", ga.c_str(), off.c_str(), ES);
      e("mad.lo.u32 %s, %s, %u, %%tile;", sa.c_str(), ch.c_str(), chunk_bytes);
      if (load)
        e("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%s], [%s], %u, [%%bar];",
          sa.c_str(), ga.c_str(), chunk_bytes);
      else
        e("cp.async.bulk.global.shared::cta.bulk_group [%s], [%s], %u;", ga.c_str(), sa.c_str(),
          chunk_bytes);
      label(skip);
    }
  }
};

// ---------------------------------------------------------------------------
// Compilation cache
// ---------------------------------------------------------------------------
// An entry is published in g_cache as soon as one thread starts compiling it; `done`
// (guarded by g_mu, signalled on g_cv) says its cubin / error are final.  Any other
// thread that finds the entry waits for `done` before reading the cubin, so a
// concurrent jit_launch never loads a half-written image.  The dynamic shared-memory
// attribute is a per-device property of the kernel, so it is tracked per device.
struct Entry {
  std::vector<char> cubin;
  std::string error;
  bool done = false;
  cudaLibrary_t lib = nullptr;
  cudaKernel_t kern = nullptr;
  std::map<int, int> smem_set;  // device -> dynamic smem bytes already allowed
};

std::mutex g_mu;
std::condition_variable g_cv;
std::unordered_map<std::string, std::shared_ptr<Entry>> g_cache;

void compile_entry(const std::string& ptx, Entry& en) {
  nvPTXCompilerHandle h = nullptr;
  if (nvPTXCompilerCreate(&h, ptx.size(), ptx.c_str()) != NVPTXCOMPILE_SUCCESS) {
    en.error = "nvPTXCompilerCreate failed";
    return;
  }
  const char* opts[] = {"--gpu-name=sm_100a", "-O3"};
  const nvPTXCompileResult rc = nvPTXCompilerCompile(h, 2, opts);
  if (rc != NVPTXCOMPILE_SUCCESS) {
    size_t n = 0;
    nvPTXCompilerGetErrorLogSize(h, &n);
    std::string log(n, '\0');
    if (n) nvPTXCompilerGetErrorLog(h, &log[0]);
    en.error = "nvPTXCompiler: " + log.substr(0, 600);
  } else {
    size_t n = 0;
    nvPTXCompilerGetCompiledProgramSize(h, &n);
    en.cubin.resize(n);
    nvPTXCompilerGetCompiledProgram(h, en.cubin.data());
  }
  nvPTXCompilerDestroy(&h);
}

}  // namespace

std::string jit_ptx(const FProg& P, int K, bool c64, int jc) {
  Gen g(P, K, c64, jc);
  return g.build();
}

// Cache key: everything the generator reads -- geometry, op headers, and per
// coefficient component its class (0, +1, -1, other; the generator specialises
// exact zeros and ones) -- but not the coefficient values, which are a kernel
// parameter.  Building the key costs O(program), not a PTX generation.
std::string jit_key(const FProg& P, int K, bool c64, int jc) {
  std::string k;
  k.reserve(64 + P.nops * sizeof(FHdr) + P.ncoef);
  const int head[5] = {K, c64 ? 1 : 0, P.nops, P.ncoef, jc};
  k.append(reinterpret_cast<const char*>(head), sizeof head);
  k.append(reinterpret_cast<const char*>(&P.tile), sizeof P.tile);
  k.append(reinterpret_cast<const char*>(P.h), sizeof(FHdr) * P.nops);
  for (int j = 0; j < P.ncoef; ++j) {
    char cls = 0;
    const double v[2] = {P.c[j].x, P.c[j].y};
    for (int q = 0; q < 2; ++q) {
      const double x = c64 ? (double)(float)v[q] : v[q];
      const int c = x == 0.0 ? 0 : x == 1.0 ? 1 : x == -1.0 ? 2 : 3;
      cls = (char)(cls | (c << (2 * q)));
    }
    k.push_back(cls);
  }
  return k;
}

void jit_compile(const std::vector<std::pair<std::string, const FProg*>>& items, int K, bool c64,
                 int jc) {
  struct Todo {
    const std::string* key;
    const FProg* prog;
    std::shared_ptr<Entry> en;
  };
  std::vector<Todo> todo;
  std::vector<std::shared_ptr<Entry>> others;  // being compiled by another thread
  {
    std::lock_guard<std::mutex> lk(g_mu);
    for (const auto& it : items) {
      auto f = g_cache.find(it.first);
      if (f != g_cache.end()) {
        if (!f->second->done) others.push_back(f->second);
        continue;
      }
      auto en = std::make_shared<Entry>();
      g_cache.emplace(it.first, en);
      todo.push_back({&it.first, it.second, en});
    }
  }
  auto wait_others = [&] {
    std::unique_lock<std::mutex> lk(g_mu);
    for (const auto& en : others) {
      g_cv.wait(lk, [&] { return en->done; });
      if (!en->error.empty()) throw Error(LFQS_ERR_CUDA, "JIT pass compile failed: " + en->error);
    }
  };
  if (todo.empty()) {
    wait_others();
    return;
  }
  unsigned nth = std::thread::hardware_concurrency();
  if (nth == 0) nth = 4;
  if (nth > todo.size()) nth = (unsigned)todo.size();
  std::atomic<size_t> next{0};
  const char* dump = std::getenv("LFQS_JIT_DUMP");  // debugging aid: write the PTX
  auto work = [&] {
    for (size_t i; (i = next.fetch_add(1)) < todo.size();) {
      const std::string ptx = jit_ptx(*todo[i].prog, K, c64, jc);
      if (dump) {
        const std::string fn = std::string(dump) + "/pass_" +
                               std::to_string(std::hash<std::string>()(ptx)) + ".ptx";
        if (FILE* fp = std::fopen(fn.c_str(), "w")) {
          std::fwrite(ptx.data(), 1, ptx.size(), fp);
          std::fclose(fp);
        }
      }
      compile_entry(ptx, *todo[i].en);
    }
  };
  std::vector<std::thread> th;
  for (unsigned t = 1; t < nth; ++t) th.emplace_back(work);
  work();
  for (auto& t : th) t.join();
  std::string err;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    for (auto& t : todo) {
      t.en->done = true;  // waiters read cubin / error only after this
      if (!t.en->error.empty()) {
        if (err.empty()) err = t.en->error;
        g_cache.erase(*t.key);  // a later call retries
      }
    }
  }
  g_cv.notify_all();
  if (!err.empty()) throw Error(LFQS_ERR_CUDA, "JIT pass compile failed: " + err);
  wait_others();
}

// FP64 operations per amplitude a pass issues (static estimate from its program): dense
// 1-target types 4 (H, real / imaginary-off-diagonal) or 8 (general), a 4x4 / 8x8 matrix 2 per
// nonzero real or imaginary coefficient part per row, one-entry diagonals 4 per affected
// amplitude; each scaled by the fraction of amplitudes its predicates select.
double pass_fp64_per_amp(const FProg& P, double* table_work) {
  double ops = 0.0;
  *table_work = 0.0;
  for (int o = 0; o < P.nops; ++o) {
    const FHdr& h = P.h[o];
    const double frac =
        std::ldexp(1.0, -__builtin_popcount(h.mlo) - __builtin_popcountll(h.mhi));
    const double2* c = P.c + h.coef;
    auto parts = [&](int n) {
      int k = 0;
      for (int i = 0; i < n; ++i) k += 2 * (c[i].x != 0.0) + 2 * (c[i].y != 0.0);
      return k;
    };
    switch (h.type) {
      case F_DTAB:  // entries x members evaluated per tile
        *table_work += std::ldexp((double)h.m, __builtin_popcount(h.mlo));
        o += h.m;
        break;
      case F_DIAG1: ops += 4.0 * frac; break;
      case F_DIAGN: ops += 4.0 * frac; break;
      case F_H: ops += (c[0].x == 1.0 ? 2.0 : 4.0) * frac; break;
      case F_UR: case F_UI: ops += 4.0 * frac; break;
      case F_U2: ops += 8.0 * frac; break;
      case F_U4: ops += parts(16) / 4.0 * frac; break;
      case F_U8: ops += parts(64) / 8.0 * frac; break;
      default: break;  // moves
    }
  }
  return ops;
}

// LFQS_OPT_JIT_THREADS = 0 (auto): 128 threads per CTA (3 CTAs per SM, one more
// register-held tile bit: fewer tile round trips) for passes whose FP64 work is below ~0.9 of
// their HBM time and that build no large phase tables; 256 otherwise -- heavy FP64 passes and
// table-heavy (QFT) passes need 256's 16 warps per SM to hide latency.  Calibrated on the
// per-pass ncu A/B of profiles/r02_heavy_passes.md (light passes 1.6 -> 1.25 ms with 128,
// heavy ones 5.5 -> 9.9 ms, QFT table passes 2.3 -> 3.2 ms).  The same rule for complex64
// (fp32 arithmetic at twice the rate on half the bytes: about the same ratio): random
// layered(31) 347 -> 333 ms, Grover 121 -> 116, the others unchanged.
int auto_threads(const FProg& P, bool c64, int K) {
  if (K < 9) return 256;
  double table_work = 0.0;
  const double ops = pass_fp64_per_amp(P, &table_work);
  // FP64 time / HBM time of the pass = ops x 2^n / 1.7e13 per s  /  (32 x 2^n B / 6.5e12 B/s)
  const double rho = ops * 6.5e12 / (1.7e13 * 32.0);
  return (table_work < 2048.0 && rho <= 0.9) ? 128 : 256;
}

int jit_config(const LaunchCtx& ctx, int K, const FProg* P) {
  int t = ctx.opt->jit_threads;
  if (t == 0) t = P ? auto_threads(*P, ctx.c64, K) : 256;
  return ((t == 512 && K >= 9) ? 512 : (t == 128 && K >= 8) ? 128 : 256) |
         (ctx.opt->jit_lane_move ? JIT_LANE_MOVE : 0) |
         (ctx.opt->jit_greedy_place ? JIT_GREEDY_PLACE : 0) |
         (ctx.opt->jit_lane_reg2 ? JIT_LANE_REG2 : 0) |
         (ctx.opt->jit_lane_pool ? JIT_LANE_POOL : 0) |
         (ctx.opt->jit_partial_rt ? JIT_PARTIAL_RT : 0);
}

size_t jit_cache_size() {
  std::lock_guard<std::mutex> lk(g_mu);
  return g_cache.size();
}

void jit_launch(const LaunchCtx& ctx, const FProg& P, int K, const std::string& key, int jc,
                uint64_t tile_ins) {
  const int nt = jc & JIT_THREADS_MASK;
  std::shared_ptr<Entry> en;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_cache.find(key);
    if (it != g_cache.end() && it->second->done) en = it->second;
  }
  if (!en) {
    jit_compile({{key, &P}}, K, ctx.c64, jc);  // compiles, or waits for another thread's compile
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_cache.find(key);
    require(it != g_cache.end() && it->second->done, "internal: JIT entry missing after compile");
    en = it->second;
  }
  const int es = ctx.c64 ? 8 : 16;
  const int smem = es << K;
  int dev = 0;
  LFQS_CUDA_CHECK(cudaGetDevice(&dev));
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto ss = en->smem_set.find(dev);
    if (en->lib == nullptr || ss == en->smem_set.end() || ss->second < smem) {
      // Module loading is not a stream operation: allowed while this thread
      // captures a CUDA graph (lfqs_circuit_compile) under relaxed mode.
      cudaStreamCaptureMode mode = cudaStreamCaptureModeRelaxed;
      LFQS_CUDA_CHECK(cudaThreadExchangeStreamCaptureMode(&mode));
      cudaError_t err = cudaSuccess;
      if (en->lib == nullptr) {
        err = cudaLibraryLoadData(&en->lib, en->cubin.data(), nullptr, nullptr, 0, nullptr,
                                  nullptr, 0);
        if (err == cudaSuccess) err = cudaLibraryGetKernel(&en->kern, en->lib, "lfqs_jit");
      }
      if (err == cudaSuccess)
        err = cudaFuncSetAttribute((const void*)en->kern,
                                   cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      cudaThreadExchangeStreamCaptureMode(&mode);
      LFQS_CUDA_CHECK(err);
      en->smem_set[dev] = smem;
    }
  }
  void* a = ctx.amps;
  void* args[3] = {&a, &tile_ins, (void*)P.c};
  const uint64_t tiles = 1ull << (ctx.n_local - K);
  LFQS_CUDA_CHECK(cudaLaunchKernel((const void*)en->kern, dim3((unsigned)tiles), dim3(nt),
                                   args, (size_t)smem, ctx.stream));
}

}  // namespace lfqs
