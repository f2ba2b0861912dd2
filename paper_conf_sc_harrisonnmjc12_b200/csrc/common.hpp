// Shared host-side plumbing of libdfg: status codes as exceptions, the
// thread-local last-error message, CUDA error checks.
#pragma once

#include <cstdint>
#include <stdexcept>
#include <string>

#include "dfg.h"

namespace dfg {

// Every internal failure is a DfgError carrying the C-ABI status; the C
// entry points catch it, store the message and return the status.
struct DfgError : std::runtime_error {
  int status;
  DfgError(int s, const std::string& m) : std::runtime_error(m), status(s) {}
};

[[noreturn]] inline void fail(int status, const std::string& msg) { throw DfgError(status, msg); }

void set_last_error(const std::string& msg);
void clear_last_error();

enum class DType { F32 = 0, F64 = 1 };
inline size_t dsize(DType t) { return t == DType::F32 ? 4 : 8; }

}  // namespace dfg

#define DFG_CUDA(call)                                                                   \
  do {                                                                                   \
    cudaError_t e_ = (call);                                                             \
    if (e_ != cudaSuccess) {                                                             \
      int st_ = (e_ == cudaErrorMemoryAllocation) ? DFG_E_NOMEM : DFG_E_CUDA;            \
      ::dfg::fail(st_, std::string(#call) + ": " + cudaGetErrorString(e_));              \
    }                                                                                    \
  } while (0)
