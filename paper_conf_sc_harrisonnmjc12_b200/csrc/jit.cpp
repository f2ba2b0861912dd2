// NVRTC -> sm_100a cubin -> CUmodule.  See jit.hpp.
#include "jit.hpp"

#include <dlfcn.h>
#include <nvrtc.h>

#include <algorithm>

#include <cstdlib>
#include <functional>
#include <map>
#include <memory>
#include <mutex>
#include <sstream>

#include "common.hpp"
#include "driver.hpp"

namespace dfg {

namespace {

// NVRTC is loaded by absolute path with RTLD_LOCAL, not linked: a process
// that already holds another libnvrtc.so.12 (torch ships its own) would
// otherwise bind libdfg to that compiler and the generated kernels would
// depend on import order.
struct NvrtcApi {
  void* h = nullptr;
  nvrtcResult (*CreateProgram)(nvrtcProgram*, const char*, const char*, int, const char* const*,
                               const char* const*) = nullptr;
  nvrtcResult (*CompileProgram)(nvrtcProgram, int, const char* const*) = nullptr;
  nvrtcResult (*GetProgramLogSize)(nvrtcProgram, size_t*) = nullptr;
  nvrtcResult (*GetProgramLog)(nvrtcProgram, char*) = nullptr;
  nvrtcResult (*GetCUBINSize)(nvrtcProgram, size_t*) = nullptr;
  nvrtcResult (*GetCUBIN)(nvrtcProgram, char*) = nullptr;
  nvrtcResult (*DestroyProgram)(nvrtcProgram*) = nullptr;
  const char* (*GetErrorString)(nvrtcResult) = nullptr;
  nvrtcResult (*Version)(int*, int*) = nullptr;
};

NvrtcApi& nvrtc() {
  static NvrtcApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* env = std::getenv("DFG_NVRTC_LIB");
    const char* cands[] = {env, "/usr/local/cuda/lib64/libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so",
                           "libnvrtc.so.12"};
    for (const char* c : cands) {
      if (!c) continue;
      api.h = dlopen(c, RTLD_NOW | RTLD_LOCAL);
      if (api.h) break;
    }
    if (!api.h) return;
#define DFG_SYM(field, name) api.field = reinterpret_cast<decltype(api.field)>(dlsym(api.h, name))
    DFG_SYM(CreateProgram, "nvrtcCreateProgram");
    DFG_SYM(CompileProgram, "nvrtcCompileProgram");
    DFG_SYM(GetProgramLogSize, "nvrtcGetProgramLogSize");
    DFG_SYM(GetProgramLog, "nvrtcGetProgramLog");
    DFG_SYM(GetCUBINSize, "nvrtcGetCUBINSize");
    DFG_SYM(GetCUBIN, "nvrtcGetCUBIN");
    DFG_SYM(DestroyProgram, "nvrtcDestroyProgram");
    DFG_SYM(GetErrorString, "nvrtcGetErrorString");
    DFG_SYM(Version, "nvrtcVersion");
#undef DFG_SYM
  });
  if (!api.h || !api.CreateProgram || !api.CompileProgram || !api.GetCUBIN || !api.GetCUBINSize)
    fail(DFG_E_NVRTC, "NVRTC (libnvrtc.so.12) could not be loaded");
  return api;
}

std::mutex g_mu;
std::map<std::string, std::unique_ptr<Cubin>> g_cache;

void parse_ptxas(const std::string& log, Cubin& c) {
  std::istringstream in(log);
  std::string line, fn;
  int best = -1;  // priority: tma 2, general/pointwise 1
  while (std::getline(in, line)) {
    auto p = line.find("entry function '");
    if (p != std::string::npos) {
      auto q = line.find('\'', p + 16);
      fn = line.substr(p + 16, q - p - 16);
      continue;
    }
    int prio = fn == "dfg_fused_tma" ? 2 : 1;
    p = line.find("Used ");
    if (p != std::string::npos && line.find("registers") != std::string::npos && prio >= best) {
      c.regs = std::atoi(line.c_str() + p + 5);
      best = prio;
    }
    // spills: the worst of ALL kernels in the module (any spilling kernel counts)
    p = line.find("bytes spill stores");
    if (p != std::string::npos) {
      auto q = line.rfind(',', p);
      size_t start = q == std::string::npos ? 0 : q + 1;
      c.spill = std::max(c.spill, std::atoi(line.c_str() + start));
    }
  }
}

}  // namespace

const Cubin& nvrtc_compile(const std::string& source, const std::string& name) {
  std::lock_guard<std::mutex> lk(g_mu);
  // developer hook: extra -D options for kernel experiments (part of the cache key)
  const char* xdef = std::getenv("DFG_NVRTC_DEFINES");
  std::vector<std::string> xopts;
  if (xdef) {
    std::istringstream is(xdef);
    for (std::string t; is >> t;) xopts.push_back(t);
  }
  const std::string key = xdef ? source + "\n//" + xdef : source;
  auto it = g_cache.find(key);
  if (it != g_cache.end()) return *it->second;

  NvrtcApi& api = nvrtc();
  nvrtcProgram prog;
  if (api.CreateProgram(&prog, source.c_str(), name.c_str(), 0, nullptr, nullptr) != NVRTC_SUCCESS)
    fail(DFG_E_NVRTC, "nvrtcCreateProgram failed");
  // Reading R6: no contraction across blocks, IEEE division/sqrt, denormals kept.
  const char* opts[] = {"--gpu-architecture=sm_100a", "--std=c++17",        "--fmad=false",
                        "--ftz=false",                "--prec-div=true",    "--prec-sqrt=true",
                        "--device-as-default-execution-space", "--generate-line-info",
                        "--ptxas-options=-v",         "-DNDEBUG"};
  std::vector<const char*> all(opts, opts + sizeof(opts) / sizeof(opts[0]));
  for (const auto& t : xopts) all.push_back(t.c_str());
  nvrtcResult rc = api.CompileProgram(prog, int(all.size()), all.data());
  size_t log_size = 0;
  api.GetProgramLogSize(prog, &log_size);
  std::string log(log_size, '\0');
  if (log_size) api.GetProgramLog(prog, &log[0]);
  if (rc != NVRTC_SUCCESS) {
    api.DestroyProgram(&prog);
    fail(DFG_E_NVRTC, std::string("NVRTC: ") + api.GetErrorString(rc) + "\n" + log);
  }
  auto c = std::make_unique<Cubin>();
  size_t n = 0;
  if (api.GetCUBINSize(prog, &n) != NVRTC_SUCCESS || n == 0) {
    api.DestroyProgram(&prog);
    fail(DFG_E_NVRTC, "NVRTC produced no cubin\n" + log);
  }
  c->image.resize(n);
  api.GetCUBIN(prog, c->image.data());
  api.DestroyProgram(&prog);
  c->log = log;
  parse_ptxas(log, *c);
  const Cubin& ref = *c;
  g_cache.emplace(key, std::move(c));
  return ref;
}

LoadedModule load_module(const Cubin& c, bool has_stencil, bool has_tma, bool rows) {
  LoadedModule m;
  DFG_CU(drv().ModuleLoadData(&m.mod, c.image.data()));
  // look up exactly the kernels skeleton.cuh / fused_tma.cuh emit for this layout
  if (!has_stencil) {
    DFG_CU(drv().ModuleGetFunction(&m.pointwise, m.mod, "dfg_fused_pointwise"));
  } else {
    DFG_CU(drv().ModuleGetFunction(&m.general, m.mod, "dfg_fused_general"));
    if (has_tma) {
      DFG_CU(drv().ModuleGetFunction(&m.tma, m.mod, "dfg_fused_tma"));
      DFG_CU(drv().ModuleGetFunction(&m.tma_multi, m.mod, "dfg_fused_tma_multi"));
      DFG_CU(drv().ModuleGetFunction(&m.tile, m.mod, "dfg_fused_tile"));
      DFG_CU(drv().ModuleGetFunction(&m.tile_multi, m.mod, "dfg_fused_tile_multi"));
      if (rows) {
        DFG_CU(drv().ModuleGetFunction(&m.rows, m.mod, "dfg_fused_rows"));
        DFG_CU(drv().ModuleGetFunction(&m.rows_multi, m.mod, "dfg_fused_rows_multi"));
      }
    }
  }
  return m;
}

}  // namespace dfg
