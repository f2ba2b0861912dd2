// NVRTC -> sm_100a cubin -> CUmodule.  See jit.hpp.
#include "jit.hpp"

#include <nvrtc.h>

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
    p = line.find("bytes spill stores");
    if (p != std::string::npos && prio >= best) {
      auto q = line.rfind(',', p);
      size_t start = q == std::string::npos ? 0 : q + 1;
      c.spill = std::atoi(line.c_str() + start);
    }
  }
}

}  // namespace

const Cubin& nvrtc_compile(const std::string& source, const std::string& name) {
  std::lock_guard<std::mutex> lk(g_mu);
  auto it = g_cache.find(source);
  if (it != g_cache.end()) return *it->second;

  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, source.c_str(), name.c_str(), 0, nullptr, nullptr) != NVRTC_SUCCESS)
    fail(DFG_E_NVRTC, "nvrtcCreateProgram failed");
  // Reading R6: no contraction across blocks, IEEE division/sqrt, denormals kept.
  const char* opts[] = {"--gpu-architecture=sm_100a", "--std=c++17",        "--fmad=false",
                        "--ftz=false",                "--prec-div=true",    "--prec-sqrt=true",
                        "--device-as-default-execution-space", "--generate-line-info",
                        "--ptxas-options=-v",         "-DNDEBUG"};
  nvrtcResult rc = nvrtcCompileProgram(prog, int(sizeof(opts) / sizeof(opts[0])), opts);
  size_t log_size = 0;
  nvrtcGetProgramLogSize(prog, &log_size);
  std::string log(log_size, '\0');
  if (log_size) nvrtcGetProgramLog(prog, &log[0]);
  if (rc != NVRTC_SUCCESS) {
    nvrtcDestroyProgram(&prog);
    fail(DFG_E_NVRTC, std::string("NVRTC: ") + nvrtcGetErrorString(rc) + "\n" + log);
  }
  auto c = std::make_unique<Cubin>();
  size_t n = 0;
  if (nvrtcGetCUBINSize(prog, &n) != NVRTC_SUCCESS || n == 0) {
    nvrtcDestroyProgram(&prog);
    fail(DFG_E_NVRTC, "NVRTC produced no cubin\n" + log);
  }
  c->image.resize(n);
  nvrtcGetCUBIN(prog, c->image.data());
  nvrtcDestroyProgram(&prog);
  c->log = log;
  parse_ptxas(log, *c);
  const Cubin& ref = *c;
  g_cache.emplace(source, std::move(c));
  return ref;
}

LoadedModule load_module(const Cubin& c, bool has_stencil, bool has_tma) {
  LoadedModule m;
  DFG_CU(drv().ModuleLoadData(&m.mod, c.image.data()));
  // look up exactly the kernels skeleton.cuh / fused_tma.cuh emit for this layout
  if (!has_stencil) {
    DFG_CU(drv().ModuleGetFunction(&m.pointwise, m.mod, "dfg_fused_pointwise"));
  } else {
    DFG_CU(drv().ModuleGetFunction(&m.general, m.mod, "dfg_fused_general"));
    if (has_tma) DFG_CU(drv().ModuleGetFunction(&m.tma, m.mod, "dfg_fused_tma"));
  }
  return m;
}

}  // namespace dfg
