// NVRTC compilation of generated fused kernels for sm_100a, with an
// in-process cache keyed by the source text (compile once per network,
// re-execute per time step: PAPER.md L122).
#pragma once

#include <cuda.h>

#include <string>
#include <vector>

namespace dfg {

struct Cubin {
  std::vector<char> image;
  std::string log;
  int regs = -1;   // ptxas "Used N registers" of the TMA kernel (or the first kernel)
  int spill = -1;  // ptxas spill stores (bytes)
};

// Compile (or fetch from cache).  Throws DfgError(DFG_E_NVRTC) with the log.
const Cubin& nvrtc_compile(const std::string& source, const std::string& name);

struct LoadedModule {
  CUmodule mod = nullptr;
  CUfunction pointwise = nullptr, general = nullptr, tma = nullptr;
  CUfunction tma_multi = nullptr;  // several meshes per launch (dfg_execute_blocks)
  CUfunction tile = nullptr;       // same ring, filled by cp.async (layouts TMA cannot describe)
  CUfunction tile_multi = nullptr; // several meshes per launch on the cp.async ring
  CUfunction rows = nullptr;       // same ring, one bulk copy per tile row (packed / unaligned rows)
  CUfunction rows_multi = nullptr; // several meshes per launch on the row-copy ring
};

// Load into the current context (requires a device).
LoadedModule load_module(const Cubin& c, bool has_stencil, bool has_tma, bool rows = false);

}  // namespace dfg
