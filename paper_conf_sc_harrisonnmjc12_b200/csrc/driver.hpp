// CUDA driver-API entry points, resolved at run time through the runtime's
// cudaGetDriverEntryPoint, so libdfg.so loads on machines without a driver
// (build / CPU test hosts) and fails with DFG_E_CUDA only when used there.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <mutex>
#include <string>

#include "common.hpp"

namespace dfg {

struct DriverApi {
  CUresult (*GetErrorString)(CUresult, const char**) = nullptr;
  CUresult (*ModuleLoadData)(CUmodule*, const void*) = nullptr;
  CUresult (*ModuleUnload)(CUmodule) = nullptr;
  CUresult (*ModuleGetFunction)(CUfunction*, CUmodule, const char*) = nullptr;
  CUresult (*FuncSetAttribute)(CUfunction, CUfunction_attribute, int) = nullptr;
  CUresult (*FuncGetAttribute)(int*, CUfunction_attribute, CUfunction) = nullptr;
  CUresult (*LaunchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                           CUstream, void**, void**) = nullptr;
  CUresult (*OccupancyMaxActiveBlocksPerMultiprocessor)(int*, CUfunction, int, size_t) = nullptr;
  CUresult (*TensorMapEncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion,
                                   CUtensorMapFloatOOBfill) = nullptr;
  // peer-memory halo (z-slabs): allocation ranges for IPC export, stream
  // memory operations for the ready / done flags
  CUresult (*MemGetAddressRange)(CUdeviceptr*, size_t*, CUdeviceptr) = nullptr;
  CUresult (*StreamWriteValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned) = nullptr;
  CUresult (*StreamWaitValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned) = nullptr;
};

inline DriverApi& drv() {
  static DriverApi api;
  static std::once_flag once;
  static bool ok = false;
  std::call_once(once, [] {
    auto get = [](const char* name, void** fn) {
      cudaDriverEntryPointQueryResult q;
      return cudaGetDriverEntryPoint(name, fn, cudaEnableDefault, &q) == cudaSuccess &&
             q == cudaDriverEntryPointSuccess && *fn;
    };
    ok = get("cuGetErrorString", reinterpret_cast<void**>(&api.GetErrorString)) &&
         get("cuModuleLoadData", reinterpret_cast<void**>(&api.ModuleLoadData)) &&
         get("cuModuleUnload", reinterpret_cast<void**>(&api.ModuleUnload)) &&
         get("cuModuleGetFunction", reinterpret_cast<void**>(&api.ModuleGetFunction)) &&
         get("cuFuncSetAttribute", reinterpret_cast<void**>(&api.FuncSetAttribute)) &&
         get("cuFuncGetAttribute", reinterpret_cast<void**>(&api.FuncGetAttribute)) &&
         get("cuLaunchKernel", reinterpret_cast<void**>(&api.LaunchKernel)) &&
         get("cuOccupancyMaxActiveBlocksPerMultiprocessor",
             reinterpret_cast<void**>(&api.OccupancyMaxActiveBlocksPerMultiprocessor)) &&
         get("cuTensorMapEncodeTiled", reinterpret_cast<void**>(&api.TensorMapEncodeTiled)) &&
         get("cuMemGetAddressRange", reinterpret_cast<void**>(&api.MemGetAddressRange)) &&
         get("cuStreamWriteValue32", reinterpret_cast<void**>(&api.StreamWriteValue32)) &&
         get("cuStreamWaitValue32", reinterpret_cast<void**>(&api.StreamWaitValue32));
    if (!ok) cudaGetLastError();
  });
  if (!ok) fail(DFG_E_CUDA, "CUDA driver API unavailable (no driver / no device); libdfg has no CPU fallback");
  return api;
}

}  // namespace dfg

#undef DFG_CU
#define DFG_CU(call)                                                                     \
  do {                                                                                   \
    CUresult r_ = (call);                                                                \
    if (r_ != CUDA_SUCCESS) {                                                            \
      const char* s_ = nullptr;                                                          \
      ::dfg::drv().GetErrorString(r_, &s_);                                              \
      ::dfg::fail(r_ == CUDA_ERROR_OUT_OF_MEMORY ? DFG_E_NOMEM : DFG_E_CUDA,            \
                  std::string(#call) + ": " + (s_ ? s_ : "unknown"));                    \
    }                                                                                    \
  } while (0)
