// jit.h -- pass compiler for fused passes (LFQS_FUSE_JIT, jit.cpp).
#pragma once
#include <string>
#include <utility>
#include <vector>

#include "fused_prog.h"
#include "lfqs_internal.h"

namespace lfqs {

// Generator configuration `jc` of a compiled pass: threads per CTA (low bits) and
// variant flags.
constexpr int JIT_THREADS_MASK = 0xffff;
constexpr int JIT_LANE_MOVE = 1 << 16;  // lane bits >= 3 (c64: >= 4) movable (LFQS_OPT_JIT_LANE_MOVE)
constexpr int JIT_GREEDY_PLACE = 1 << 17;  // multi-bit remaps (LFQS_OPT_JIT_GREEDY_PLACE)
constexpr int JIT_LANE_REG2 = 1 << 18;     // lane/register 2-target gates (LFQS_OPT_JIT_LANE_REG2)
constexpr int JIT_LANE_POOL = 1 << 19;     // movable lanes as cheap positions (LFQS_OPT_JIT_LANE_POOL)
constexpr int JIT_PARTIAL_RT = 1 << 20;    // round trips move only re-placed amplitudes

// PTX of one fused pass: structure baked in, coefficients a kernel parameter.
std::string jit_ptx(const FProg& P, int K, bool c64, int jc);
// Cache key of a pass (its structure and coefficient classes, not values).
std::string jit_key(const FProg& P, int K, bool c64, int jc);
// Generates and compiles (in parallel, nvPTXCompiler) every pass not yet cached.
void jit_compile(const std::vector<std::pair<std::string, const FProg*>>& items, int K, bool c64,
                 int jc);
// Launches the pass (compiling it first if needed) on ctx.stream: 2^(ctx.n_local - K) tiles,
// with the tile-index insertions tile_ins (fused_prog.h; a block of the state).
void jit_launch(const LaunchCtx& ctx, const FProg& P, int K, const std::string& key, int jc,
                uint64_t tile_ins = kNoTileIns);
// Generator configuration of pass P for tile size K (LFQS_OPT_JIT_THREADS -- 0: chosen per
// pass from P -- LFQS_OPT_JIT_LANE_MOVE, ...).
int jit_config(const LaunchCtx& ctx, int K, const FProg* P = nullptr);
size_t jit_cache_size();

}  // namespace lfqs
