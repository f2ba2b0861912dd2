// Internal helpers shared by the libdfg runtime translation units (mesh.cpp,
// model.cpp, runtime.cpp, exec_staged.cpp).  Not part of the C ABI.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "common.hpp"
#include "runtime.hpp"

namespace dfg {
namespace detail {

// NVTX range around a host-side step (header-only NVTX3: a no-op unless a
// tool such as nsys injects itself), so a timeline shows every execute, each
// staged filter, the halo exchange and each fused launch by name
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
  ~NvtxRange() { nvtxRangePop(); }
};

// ---- mesh.cpp
cudaMemPool_t pool_for(int dev);  // per-device pool, memory kept across executes
int sm_count(int dev);

// NCCL, loaded with dlopen (the process's copy first: torch's)
struct NcclApi {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi& nccl();
void nccl_check(ncclResult_t r, const char* what);

// ---- model.cpp
struct Sources {
  std::vector<int> inputs;  // first-use order (+ bare result)
  bool mesh = false;
};
Sources sources(const Dag& dag);                // bound inputs in first-use order, mesh use
int64_t units(const Dag& dag, const Ref& r);     // problem-array units: scalar 1, vector 4
bool host_side(Op op);                           // roundtrip runs it on the host

// ---- runtime.cpp
// device-memory ledger of one execute (dev_mem_cap, Fig. 2 high-water)
struct Ledger {
  size_t cap, live = 0, high = 0;
  explicit Ledger(size_t c) : cap(c) {}
  void add(size_t b) {
    if (cap && live + b > cap)
      fail(DFG_E_NOMEM, "device memory cap exceeded: " + std::to_string(live + b) + " > " + std::to_string(cap) +
                            " bytes");
    live += b;
    high = std::max(high, live);
  }
  void sub(size_t b) { live -= std::min(live, b); }
};
void* dev_alloc(size_t bytes, int dev, cudaStream_t s);  // stream-ordered, from pool_for(dev)
bool aligned16(const void* p);
// pinned host buffers shared by the plans of the process (guard: g_host_mu)
struct HostPool {
  std::multimap<size_t, void*> free_;
  std::vector<void*> all;
  void* get(size_t b) {
    auto it = free_.lower_bound(b);
    if (it != free_.end() && it->first < 2 * b + 4096) {
      void* p = it->second;
      free_.erase(it);
      return p;
    }
    void* p = nullptr;
    DFG_CUDA(cudaHostAlloc(&p, b ? b : 16, cudaHostAllocDefault));
    all.push_back(p);
    sizes[p] = b;
    return p;
  }
  void put(void* p) { free_.emplace(sizes[p], p); }
  std::map<void*, size_t> sizes;
  ~HostPool() {
    for (void* p : all) cudaFreeHost(p);
  }
};
HostPool& host_pool();

// Host loops of the roundtrip strategy (constant fills, decompose on the host,
// L289) over problem-sized arrays: split [0, n) over the host cores.  Element
// order does not matter (each index is written once from its own inputs).
template <class F>
void parallel_for(int64_t n, F f) {
  static const int64_t cap = [] {
    const char* e = std::getenv("DFG_HOST_THREADS");
    return e ? std::max<int64_t>(1, std::atoll(e)) : int64_t(32);
  }();
  const int64_t hw = int64_t(std::max(1u, std::thread::hardware_concurrency()));
  const int64_t T = std::max<int64_t>(1, std::min<int64_t>({hw, cap, n / (1 << 16)}));
  if (T == 1) {
    f(int64_t(0), n);
    return;
  }
  std::vector<std::thread> th;
  for (int64_t t = 1; t < T; ++t) th.emplace_back(f, n * t / T, n * (t + 1) / T);
  f(int64_t(0), n / T);
  for (auto& x : th) x.join();
}
extern std::mutex g_host_mu;

}  // namespace detail
}  // namespace dfg
