// fused_prog.h -- the gate program of one fused pass, shared by
// the interpreting kernel (fused_kernels.cu) and the pass compiler (jit.cpp).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace lfqs {

// 1-target dense types are specialised by matrix values (static matrix
// specialisation): F_UR real matrix (Ry), F_UI real diagonal with
// imaginary off-diagonal (Rx) -- 4 FP ops per amplitude instead of 8.
// F_DTAB (LFQS_FUSE_PHASE): a phase table over <= 8 tile bits standing for the
// m diagonal ops that follow it (its members).
enum FType : uint8_t {
  F_DIAG1 = 0, F_DIAGN, F_X, F_Y, F_H, F_UR, F_UI, F_U2, F_SWAP, F_U4, F_U8, F_DTAB
};

struct FHdr {       // 32 bytes
  uint8_t type, m, t0, t1, t2, pad0;
  uint16_t coef;    // offset into the coefficient pool
  uint32_t mlo, plo;  // per-amplitude predicate (i & mlo) == plo   (tile bits)
  uint64_t mhi, phi;  // per-tile predicate     (base & mhi) == phi (qubits outside the tile)
  // F_DTAB: m = member count, mlo = table bits U (tile bits), plo = common
  // predicate cm | cp << 16 (every member requires (i & cm) == cp); mhi = phi = 0.
};
constexpr int kMaxOps = 192;
constexpr int kMaxCoef = 1580;
constexpr int kMaxHigh = 8;
// Tile geometry: tile bits [0, lc) are qubits [0, lc) (one contiguous chunk of
// 2^lc amplitudes); tile bits lc + i are the "high" qubits hpos[i] (ascending).
// The tile is 2^(K - lc) chunks, each moved by one TMA bulk copy.
struct FTile {
  int lc;
  int nh;
  uint8_t hpos[kMaxHigh];
};
struct FProg {
  int nops;
  int ncoef;
  FTile tile;
  FHdr h[kMaxOps];
  double2 c[kMaxCoef];
};
static_assert(sizeof(FProg) + 8 <= 32764, "kernel parameter limit");

// Tile-index insertions of a launch (k_fused / compiled passes): byte i (i = 0..2, by
// ascending position) = position p (bits 0-5, in tile-index space) | value << 6 of a bit
// inserted into the block index before it becomes the tile base; p = 63 inserts nothing.
// A launch with insertions covers the tiles of one block of the state (the amplitudes
// whose chunk qubits hold fixed values -- overlapped exchanges, state.cu).
constexpr uint64_t kNoTileIns = 0x3f3f3full;

constexpr int kFThreads = 256;
constexpr int kMinK = 8, kMaxK = 12;

}  // namespace lfqs
