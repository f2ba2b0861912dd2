// Dynamic kernel generator of the fusion strategy:
// one CUDA kernel per network, built from the building blocks of
// blocks.cuh -- per-element calls for simple primitives (L101), direct
// memory access for the gradient (L102), constants inserted as source
// literals (L103), vector results as per-lane registers (L104) and
// decompose as a register selection (L105).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "lang.hpp"

namespace dfg {

struct FusedLayout {
  std::vector<int> stencil_inputs;  // input indices read by some grad3d (+ centre)
  std::vector<int> point_inputs;    // input indices read only at the cell
  int outw = 1;                     // 1 or 4
  bool has_grad = false;
};

struct FusedConfig {
  int div_mode = 1;    // 0 ieee, 1 exact (Markstein), 2 fast; see blocks.cuh
  int div2 = 0;        // div_mode 1, fp32: bit a = axis a uses the verified two-op quotient
  bool fold = true;    // power-of-two scale folding in the body (off for div_mode 0, "ieee")
  int ncw = 15;        // consumer warps per CTA (tile rows); +1 producer = 512 threads
  int stages = 0;      // smem ring depth (0: choose)
  int ctas = 1;        // resident CTAs per SM the TMA kernel is sized for
  int rpw = 1;         // tile rows per consumer warp (1, 2, 4): tile = (32*VEC/rpw) x (ncw*rpw)
  bool has_tma = false;
  int rstages = 0;     // row-class kernel: ring depth (0: it does not fit)
};

struct FusedSource {
  std::string source;
  FusedLayout layout;
  FusedConfig cfg;
};

FusedLayout fused_layout(const Dag& dag);
// nx/ny/nz: global mesh dims (axis degeneracy n == 1 is baked in).
// ref > 0: use the hand-written reference body `ref` (reference_bodies.cuh)
// instead of generating one from the network.
FusedSource generate_fused(const Dag& dag, int64_t nx, int64_t ny, int64_t nz, FusedConfig cfg, int ref = 0);

// Reference kernels: the paper program of a quantity
// ("velmag", "vortmag", "qcrit") and its body id, or nullptr / 0.
const char* reference_program(const std::string& which, int* id);

// Dynamic shared memory the TMA kernel needs for a config (bytes).
size_t fused_tma_smem_bytes(DType dt, int nsf, int ncw, int stages, int rpw = 1);
// the row-class kernel (fused_tma.cuh "rows"): a ring of `stages` stages of
// class boxes (box width = halo'd tile row + one chunk) + its barriers
size_t fused_rows_smem_bytes(DType dt, int nsf, int ncw, int rpw, int stages);

// TMA kernel tile: tile_w cells along x, tile_h rows along y (fused_tma.cuh).
inline int tma_tile_w(DType dt, int rpw) { return 32 * (dt == DType::F32 ? 4 : 2) / rpw; }
inline int tma_tile_h(int ncw, int rpw) { return ncw * rpw; }

// Rows per consumer warp for a mesh of nx x ny x nz cells on `slots`
// persistent CTAs: the candidate (1, 2, 4) whose best z-chunking needs the
// fewest plane-steps, weighted by the halo'd tile it loads per computed cell.
int choose_rpw(DType dt, int64_t nx, int64_t ny, int64_t nz, int ncw, int64_t slots, double* cost = nullptr);
// Tile shape of the fused kernel for a mesh: consumer warps (15, or 12 when the
// plane-step model -- steps per CTA x halo'd tile area -- is >= 5 % cheaper,
// e.g. 192 rows = 8 tiles of 24) and rows per warp.
void choose_tile(DType dt, int64_t nx, int64_t ny, int64_t nz, int64_t slots, int* ncw, int* rpw);
// the same for layouts only the row-class kernel takes (packed ghost shells,
// rows that are not 16-byte multiples): 14 or 12 consumer warps (the kernel
// adds a producer and a fixup warp: 16 warps keep 128 registers), 12 when
// 14 leave more of a ragged last y-tile idle (its two-plane ring makes the
// rows, not the halo, the cost: 192-row blocks 260 -> 288 Gcells/s with 12 x 2)
void choose_rows_tile(DType dt, int64_t nx, int64_t ny, int64_t nz, int64_t slots, int* ncw, int* rpw);

// z-chunk length for `tiles` x-y tiles over `range` planes: whole rounds of
// items over the persistent CTAs against the two halo planes (and the
// pipeline fill) each chunk costs.  Returns the chunk length; *cost gets the
// plane-steps of the slowest CTA.
int64_t choose_kz(int64_t tiles, int64_t range, int64_t slots, int64_t* cost = nullptr);

}  // namespace dfg
