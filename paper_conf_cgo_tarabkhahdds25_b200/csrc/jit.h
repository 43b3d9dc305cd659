// jit.h -- pass compiler for fused passes (LFQS_FUSE_JIT, jit.cpp).
#pragma once
#include <string>
#include <utility>
#include <vector>

#include "fused_prog.h"
#include "lfqs_internal.h"

namespace lfqs {

// PTX of one fused pass: structure baked in, coefficients a kernel parameter.
std::string jit_ptx(const FProg& P, int K, bool c64, int nt);
// Cache key of a pass (its structure and coefficient classes, not values).
std::string jit_key(const FProg& P, int K, bool c64, int nt);
// Generates and compiles (in parallel, nvPTXCompiler) every pass not yet cached.
void jit_compile(const std::vector<std::pair<std::string, const FProg*>>& items, int K, bool c64,
                 int nt);
// Launches the pass (compiling it first if needed) on ctx.stream.
void jit_launch(const LaunchCtx& ctx, const FProg& P, int K, const std::string& key, int nt);
// Threads per CTA of a compiled pass for tile size K (LFQS_OPT_JIT_THREADS).
int jit_threads(const LaunchCtx& ctx, int K);
size_t jit_cache_size();

}  // namespace lfqs
