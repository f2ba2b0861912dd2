// libdfg runtime.  See runtime.hpp; DESIGN.md sections 2, 5 and 6.
#include "runtime.hpp"

#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <set>

#include "driver.hpp"
#include "kernels.hpp"

namespace dfg {

// ====================================================================== mesh
namespace {

template <typename T>
void build_axis(const T* p, int64_t n, std::vector<char>& tab, bool& safe) {
  // Reading R1: centres c_i = (p_i + p_{i+1}) * 0.5 in T; for each cell the
  // clamped neighbour-centre distance d_i = c[ip] - c[im] and r_i = RN(1/d_i).
  for (int64_t i = 0; i <= n; ++i)
    if (!std::isfinite(double(p[i]))) fail(DFG_E_INVALID, "coordinates must be finite");
  for (int64_t i = 0; i < n; ++i)
    if (!(p[i] < p[i + 1])) fail(DFG_E_INVALID, "coordinates must be strictly increasing");
  std::vector<T> c(n);
  for (int64_t i = 0; i < n; ++i) c[i] = (p[i] + p[i + 1]) * T(0.5);
  tab.assign(size_t(4 * n) * sizeof(T), 0);
  T* d = reinterpret_cast<T*>(tab.data());
  T* r = d + n;
  T* nd = r + n;  // exact negation: the fused kernels form num - q0*d with one FFMA2
  T* yl = nd + n; // low part of 1/d for the two-operation quotient (fp32 only)
  for (int64_t i = 0; i < n; ++i) {
    if (n == 1) {  // derivative is 0 by definition; the kernels never read these
      d[i] = T(1);
      r[i] = T(1);
      nd[i] = T(-1);
      continue;
    }
    int64_t ip = std::min(i + 1, n - 1), im = std::max<int64_t>(i - 1, 0);
    d[i] = c[ip] - c[im];
    if (!(d[i] > T(0))) fail(DFG_E_INVALID, "cell centres coincide (coordinates too close for T)");
    r[i] = T(1) / d[i];
    nd[i] = -d[i];
    // yl = RN(1/d - r): 1/d in double is within 2^-53 of the real quotient and
    // the subtraction is exact (Sterbenz); the kernels only use yl on axes whose
    // every divisor passed the exhaustive check (verify_div2 below), so its last
    // bit needs no argument.
    if (sizeof(T) == 4) yl[i] = T(1.0 / double(d[i]) - double(r[i]));
    // Markstein's exact-quotient argument needs d and r well inside the normal range.
    double ad = double(d[i]);
    if (!(ad > 0x1p-60 && ad < 0x1p60) || !std::isfinite(double(r[i]))) safe = false;
  }
}

// Two-operation quotient: an fp32 axis uses
// q = RN(num*r + RN(num*yl)) in the fused kernels only if every divisor of
// its table passed the exhaustive device check.  Verdicts are cached per
// (d, yl) bit pattern (r is a function of d).
std::mutex g_div2_mu;
std::map<uint64_t, bool> g_div2_ok;  // key: d bits << 32 | yl bits

uint64_t div2_key(float d, float yl) {
  uint32_t a, b;
  std::memcpy(&a, &d, 4);
  std::memcpy(&b, &yl, 4);
  return uint64_t(a) << 32 | b;
}

bool axis_div2(const std::vector<char>& tab, int64_t n) {
  const float* d = reinterpret_cast<const float*>(tab.data());
  const float* r = d + n;
  const float* yl = d + 3 * n;
  if (n == 1) return true;  // no division on a degenerate axis
  std::lock_guard<std::mutex> lk(g_div2_mu);
  std::vector<float> qd, qr, ql;
  std::set<uint64_t> seen;
  for (int64_t i = 0; i < n; ++i) {
    const uint64_t b = div2_key(d[i], yl[i]);
    if (g_div2_ok.count(b) || !seen.insert(b).second) continue;
    qd.push_back(d[i]);
    qr.push_back(r[i]);
    ql.push_back(yl[i]);
  }
  if (!qd.empty()) {
    const int m = int(qd.size());
    float* buf = nullptr;
    unsigned* bad = nullptr;
    DFG_CUDA(cudaMalloc(&buf, 3 * size_t(m) * sizeof(float)));
    DFG_CUDA(cudaMalloc(&bad, size_t(m) * sizeof(unsigned)));
    DFG_CUDA(cudaMemcpy(buf, qd.data(), m * sizeof(float), cudaMemcpyHostToDevice));
    DFG_CUDA(cudaMemcpy(buf + m, qr.data(), m * sizeof(float), cudaMemcpyHostToDevice));
    DFG_CUDA(cudaMemcpy(buf + 2 * m, ql.data(), m * sizeof(float), cudaMemcpyHostToDevice));
    DFG_CUDA(cudaMemset(bad, 0, size_t(m) * sizeof(unsigned)));
    kern::verify_div2(buf, buf + m, buf + 2 * m, m, bad, nullptr);
    std::vector<unsigned> hb(m);
    cudaError_t e = cudaMemcpy(hb.data(), bad, m * sizeof(unsigned), cudaMemcpyDeviceToHost);
    cudaFree(buf);
    cudaFree(bad);
    DFG_CUDA(e);
    for (int k = 0; k < m; ++k) g_div2_ok[div2_key(qd[k], ql[k])] = hb[k] == 0;
  }
  for (int64_t i = 0; i < n; ++i)
    if (!g_div2_ok[div2_key(d[i], yl[i])]) return false;
  return true;
}

std::mutex g_pool_mu;
std::map<int, cudaMemPool_t> g_pools;

cudaMemPool_t pool_for(int dev) {
  std::lock_guard<std::mutex> lk(g_pool_mu);
  auto it = g_pools.find(dev);
  if (it != g_pools.end()) return it->second;
  cudaMemPoolProps props{};
  props.allocType = cudaMemAllocationTypePinned;
  props.location.type = cudaMemLocationTypeDevice;
  props.location.id = dev;
  cudaMemPool_t pool;
  DFG_CUDA(cudaMemPoolCreate(&pool, &props));
  uint64_t thr = UINT64_MAX;
  DFG_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
  g_pools[dev] = pool;
  return pool;
}

int sm_count(int dev) {
  static std::map<int, int> cache;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(dev);
  if (it != cache.end()) return it->second;
  int n = 0;
  DFG_CUDA(cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev));
  cache[dev] = n;
  return n;
}

}  // namespace

MeshImpl::~MeshImpl() {
  int cur = -1;
  cudaGetDevice(&cur);
  cudaSetDevice(device);
  for (auto& p : dev_tab)
    if (p) cudaFree(p);
  if (nccl) {
    using destroy_fn = ncclResult_t (*)(ncclComm_t);
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (h) {
      auto f = reinterpret_cast<destroy_fn>(dlsym(h, "ncclCommDestroy"));
      if (f) f(static_cast<ncclComm_t>(nccl));
    }
  }
  if (cur >= 0) cudaSetDevice(cur);
}

std::shared_ptr<MeshImpl> create_mesh(DType dt, int64_t nx, int64_t ny, int64_t nzl, const void* x, const void* y,
                                      const void* z, int64_t NZ, int64_t k0, int ghost) {
  if (nx < 1 || ny < 1 || nzl < 1 || NZ < 1) fail(DFG_E_INVALID, "mesh sizes must be >= 1");
  if (k0 < 0 || k0 + nzl > NZ) fail(DFG_E_INVALID, "z slab outside the global mesh");
  if (ghost != 0 && ghost != 1) fail(DFG_E_INVALID, "ghost must be 0 or 1");
  if (nzl != NZ && ghost != 1) fail(DFG_E_INVALID, "a z slab of a larger mesh needs ghost = 1");
  if (!x || !y || !z) fail(DFG_E_INVALID, "null coordinate pointer");
  return create_block_impl(dt, nx, ny, nzl, x, y, z, nx, ny, NZ, 0, 0, k0, ghost, 0);
}

std::shared_ptr<MeshImpl> create_block(DType dt, int64_t nx, int64_t ny, int64_t nz, const void* x, const void* y,
                                       const void* z, int64_t NX, int64_t NY, int64_t NZ, int64_t i0, int64_t j0,
                                       int64_t k0, int ghost, int64_t pitch, int64_t xoff) {
  if (nx < 1 || ny < 1 || nz < 1 || NX < 1 || NY < 1 || NZ < 1) fail(DFG_E_INVALID, "block sizes must be >= 1");
  if (i0 < 0 || j0 < 0 || k0 < 0 || i0 + nx > NX || j0 + ny > NY || k0 + nz > NZ)
    fail(DFG_E_INVALID, "block outside the global mesh");
  if (ghost != 0 && ghost != 1) fail(DFG_E_INVALID, "ghost must be 0 or 1");
  if (ghost == 0 && (nx != NX || ny != NY || nz != NZ))
    fail(DFG_E_INVALID, "a block of a larger mesh needs its one-cell ghost shell");
  if (!x || !y || !z) fail(DFG_E_INVALID, "null coordinate pointer");
  if (xoff == 0) xoff = ghost;
  if (pitch == 0) pitch = xoff + nx + ghost;
  if (xoff < ghost || xoff + nx + ghost > pitch)
    fail(DFG_E_INVALID, "need ghost <= x_offset and x_offset + nx + ghost <= row_pitch");
  auto m = create_block_impl(dt, nx, ny, nz, x, y, z, NX, NY, NZ, i0, j0, k0, ghost, ghost);
  m->ghosts_supplied = ghost == 1;
  m->pitch = pitch;
  m->xoff = xoff;
  return m;
}

std::shared_ptr<MeshImpl> create_block_impl(DType dt, int64_t nx, int64_t ny, int64_t nzl, const void* x,
                                            const void* y, const void* z, int64_t NX, int64_t NY, int64_t NZ,
                                            int64_t i0, int64_t j0, int64_t k0, int ghost, int gxy) {
  auto m = std::make_shared<MeshImpl>();
  m->dt = dt;
  m->nx = nx;
  m->ny = ny;
  m->nzl = nzl;
  m->NZ = NZ;
  m->k0 = k0;
  m->NX = NX;
  m->NY = NY;
  m->i0 = i0;
  m->j0 = j0;
  m->ghost = ghost;
  m->gxy = gxy;
  const void* P[3] = {x, y, z};
  int64_t N[3] = {NX, NY, NZ};
  for (int a = 0; a < 3; ++a) {
    if (dt == DType::F32) build_axis(static_cast<const float*>(P[a]), N[a], m->host_tab[a], m->markstein_safe);
    else build_axis(static_cast<const double*>(P[a]), N[a], m->host_tab[a], m->markstein_safe);
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) {
    cudaGetLastError();
    fail(DFG_E_CUDA, "no CUDA device available (libdfg has no CPU fallback)");
  }
  DFG_CUDA(cudaGetDevice(&m->device));
  // DFG_DIV2=0: never use the two-operation quotient; DFG_DIV2=test-1op (tests
  // only): yl = 0, i.e. the one-operation RN(num*r), which the check must reject
  // unless every divisor is a power of two
  const char* d2 = std::getenv("DFG_DIV2");
  const bool div2_off = d2 && !std::strcmp(d2, "0");
  if (dt == DType::F32 && d2 && !std::strcmp(d2, "test-1op"))
    for (int a = 0; a < 3; ++a)
      std::fill_n(reinterpret_cast<float*>(m->host_tab[a].data()) + 3 * N[a], N[a], 0.0f);
  for (int a = 0; a < 3; ++a) {
    DFG_CUDA(cudaMalloc(&m->dev_tab[a], m->host_tab[a].size()));
    DFG_CUDA(cudaMemcpy(m->dev_tab[a], m->host_tab[a].data(), m->host_tab[a].size(), cudaMemcpyHostToDevice));
  }
  if (dt == DType::F32 && m->markstein_safe && !div2_off)
    for (int a = 0; a < 3; ++a)
      if (axis_div2(m->host_tab[a], N[a])) m->div2_mask |= 1 << a;
  return m;
}

// ===================================================================== NCCL
namespace {
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

NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    // Prefer the NCCL the process already loaded (torch's), else the system one.
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    api.h = h;
    api.GetUniqueId = reinterpret_cast<decltype(api.GetUniqueId)>(dlsym(h, "ncclGetUniqueId"));
    api.CommInitRank = reinterpret_cast<decltype(api.CommInitRank)>(dlsym(h, "ncclCommInitRank"));
    api.Send = reinterpret_cast<decltype(api.Send)>(dlsym(h, "ncclSend"));
    api.Recv = reinterpret_cast<decltype(api.Recv)>(dlsym(h, "ncclRecv"));
    api.GroupStart = reinterpret_cast<decltype(api.GroupStart)>(dlsym(h, "ncclGroupStart"));
    api.GroupEnd = reinterpret_cast<decltype(api.GroupEnd)>(dlsym(h, "ncclGroupEnd"));
    api.GetErrorString = reinterpret_cast<decltype(api.GetErrorString)>(dlsym(h, "ncclGetErrorString"));
  });
  if (!api.h || !api.GetUniqueId || !api.CommInitRank || !api.Send || !api.Recv || !api.GroupStart ||
      !api.GroupEnd)
    fail(DFG_E_NCCL, "NCCL (libnccl.so.2) could not be loaded");
  return api;
}

void nccl_check(ncclResult_t r, const char* what) {
  if (r != ncclSuccess) {
    const char* s = nccl().GetErrorString ? nccl().GetErrorString(r) : "?";
    fail(DFG_E_NCCL, std::string(what) + ": " + s);
  }
}
}  // namespace

void nccl_unique_id(void* out128) {
  ncclUniqueId id;
  nccl_check(nccl().GetUniqueId(&id), "ncclGetUniqueId");
  static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(out128, &id, 128);
}

void mesh_init_comm(MeshImpl& m, const void* id128, int rank, int nranks) {
  if (nranks < 1 || rank < 0 || rank >= nranks) fail(DFG_E_INVALID, "bad rank/nranks");
  if (nranks == 1) {
    m.rank = 0;
    m.nranks = 1;
    return;
  }
  ncclUniqueId id;
  std::memcpy(&id, id128, 128);
  DFG_CUDA(cudaSetDevice(m.device));
  ncclComm_t comm;
  nccl_check(nccl().CommInitRank(&comm, nranks, id, rank), "ncclCommInitRank");
  m.nccl = comm;
  m.rank = rank;
  m.nranks = nranks;
}

// ==================================================================== model
namespace {
struct Sources {
  std::vector<int> inputs;  // first-use order (+ bare result)
  bool mesh = false;
};
Sources sources(const Dag& dag) {
  Sources s;
  auto note = [&](const Ref& r) {
    if (r.kind == Ref::Mesh) s.mesh = true;
    else if (r.kind == Ref::Input && std::find(s.inputs.begin(), s.inputs.end(), r.id) == s.inputs.end())
      s.inputs.push_back(r.id);
  };
  for (auto& f : dag.filters)
    for (auto& r : f.in) note(r);
  if (dag.result.kind == Ref::Input) note(dag.result);
  return s;
}
int64_t units(const Dag& dag, const Ref& r) { return dag.width(r) == 1 ? 1 : 4; }
bool host_side(Op op) { return op == Op::Decompose || op == Op::Const; }  // roundtrip: no kernel
}  // namespace

Model model(const Dag& dag, dfg_strategy s, bool host) {
  // the streamed strategy is fusion per z-chunk: its network-level numbers
  // are fusion's (per-chunk transfers and the ring footprint are physical);
  // a reference kernel has fusion's I/O; without a cap hybrid is staged
  if (s == DFG_STREAMED || s == DFG_REFERENCE) s = DFG_FUSED;
  if (s == DFG_HYBRID) s = DFG_STAGED;
  Model m;
  Sources src = sources(dag);
  const int64_t F = int64_t(dag.filters.size());
  const bool bare = dag.result.kind != Ref::Filter;
  const int64_t out_u = units(dag, dag.result);
  int64_t in_u = 0;
  for (int i : src.inputs) (void)i, in_u += 1;
  // ---- counts (Table II rules, R11-R13)
  if (s == DFG_FUSED) {
    m.kernels = 1;
    if (host) { m.h2d = int64_t(src.inputs.size()) + (src.mesh ? 4 : 0); m.d2h = 1; }
  } else if (s == DFG_STAGED) {
    m.kernels = F;
    if (host) { m.h2d = int64_t(src.inputs.size()) + (src.mesh ? 4 : 0); m.d2h = 1; }
  } else {
    for (auto& f : dag.filters) {
      if (host_side(f.op)) continue;
      m.kernels += 1;
      m.d2h += 1;
      for (auto& r : f.in) {
        if (host) m.h2d += 1;                    // every argument of every kernel
        else if (r.kind == Ref::Filter) m.h2d += 1;  // only host-resident values
      }
    }
    if (!host && !bare) m.h2d += 1;              // final result to the device output
  }
  // ---- footprint (Fig. 2 rules)
  if (s == DFG_FUSED) {
    m.units = in_u + out_u;
  } else if (s == DFG_ROUNDTRIP) {
    int64_t base = host ? 0 : in_u + out_u, high = base;
    for (size_t k = 0; k < dag.filters.size(); ++k) {
      const Filter& f = dag.filters[k];
      if (host_side(f.op)) continue;
      int64_t args = 0;
      for (auto& r : f.in) {
        if (r.kind == Ref::Mesh) continue;
        if (!host && r.kind == Ref::Input) continue;
        args += units(dag, r);
      }
      high = std::max(high, base + args + units(dag, Ref{Ref::Filter, int(k)}));
    }
    m.units = high;
  } else {
    std::vector<int> order(dag.filters.size());
    for (size_t k = 0; k < order.size(); ++k) order[k] = int(k);
    m.units = staged_units(dag, order, host);
  }
  return m;
}

// Staged footprint of a given execution order: lazy upload of host inputs,
// free at reference count zero (L85), Fig. 2 accounting.
int64_t staged_units(const Dag& dag, const std::vector<int>& order, bool host) {
  Sources src = sources(dag);
  std::map<std::pair<int, int>, int64_t> rc;
  auto key = [](const Ref& r) { return std::make_pair(int(r.kind), r.id); };
  for (auto& f : dag.filters)
    for (auto& r : f.in)
      if (r.kind != Ref::Mesh) rc[key(r)] += 1;
  rc[key(dag.result)] += 1;
  std::set<int> resident;
  int64_t live = 0, high = 0;
  if (!host) {
    live = int64_t(src.inputs.size()) + units(dag, dag.result);
    for (int i : src.inputs) resident.insert(i);
    high = live;
  }
  for (size_t pos = 0; pos < order.size(); ++pos) {
    const int k = order[pos];
    const Filter& f = dag.filters[k];
    for (auto& r : f.in)
      if (r.kind == Ref::Input && !resident.count(r.id)) {
        resident.insert(r.id);
        live += 1;
      }
    bool into_out = !host && dag.result.kind == Ref::Filter && dag.result.id == k && pos + 1 == order.size();
    if (!into_out) live += f.width == 1 ? 1 : 4;
    high = std::max(high, live);
    for (auto& r : f.in) {
      if (r.kind == Ref::Mesh) continue;
      if (--rc[key(r)] == 0 && (host || r.kind == Ref::Filter)) live -= units(dag, r);
    }
  }
  if (dag.result.kind == Ref::Input && !resident.count(dag.result.id)) {
    live += 1;
    high = std::max(high, live);
  }
  return high;
}

// Memory-aware staged schedule: repeatedly run the ready
// filter whose execution changes the live device memory the least
// (allocation minus arrays it frees; ties to the lowest id).
std::vector<int> greedy_staged_order(const Dag& dag) {
  const size_t n = dag.filters.size();
  std::map<int, int64_t> rc;  // remaining uses of each filter result
  for (auto& f : dag.filters)
    for (auto& r : f.in)
      if (r.kind == Ref::Filter) rc[r.id] += 1;
  if (dag.result.kind == Ref::Filter) rc[dag.result.id] += 1;
  std::vector<char> done(n, 0);
  std::vector<int> order;
  while (order.size() < n) {
    int best = -1;
    int64_t best_delta = 0;
    for (size_t k = 0; k < n; ++k) {
      if (done[k]) continue;
      const Filter& f = dag.filters[k];
      bool ready = true;
      for (auto& r : f.in)
        if (r.kind == Ref::Filter && !done[r.id]) ready = false;
      if (!ready) continue;
      int64_t delta = f.width == 1 ? 1 : 4;
      std::map<int, int64_t> uses;
      for (auto& r : f.in)
        if (r.kind == Ref::Filter) uses[r.id] += 1;
      for (auto& u : uses)
        if (rc[u.first] == u.second) delta -= dag.filters[u.first].width == 1 ? 1 : 4;
      if (best < 0 || delta < best_delta) {
        best = int(k);
        best_delta = delta;
      }
    }
    done[best] = 1;
    order.push_back(best);
    for (auto& r : dag.filters[best].in)
      if (r.kind == Ref::Filter) rc[r.id] -= 1;
  }
  return order;
}

// Staged execution holding at most cap units on the device:
// before each array that does not fit, evict the resident array read
// furthest in the future (ties: larger, filter before input, higher id),
// never an operand of the running filter; an intermediate is copied to the
// host the first time it is evicted, an uploaded input is dropped.
HybridPlan plan_hybrid(const Dag& dag, const std::vector<int>& order, int64_t cap, bool host) {
  using Key = std::pair<int, int>;  // (kind, id): Ref::Filter = 0, Ref::Input = 1
  auto key = [](const Ref& r) { return Key(int(r.kind), r.id); };
  auto ref_of = [](const Key& k) { return Ref{Ref::Kind(k.first), k.second}; };
  HybridPlan hp;
  const int n = int(order.size());
  Sources src = sources(dag);
  std::map<Key, std::vector<int>> uses;  // positions reading each value; the sink reads the result at n
  std::map<Key, int64_t> rc;
  for (int p = 0; p < n; ++p)
    for (auto& r : dag.filters[size_t(order[p])].in)
      if (r.kind != Ref::Mesh) {
        uses[key(r)].push_back(p);
        rc[key(r)] += 1;
      }
  uses[key(dag.result)].push_back(n);
  rc[key(dag.result)] += 1;
  auto next_use = [&](const Key& k, int pos) {
    for (int p : uses[k])
      if (p >= pos) return p;
    return n + 1;
  };
  std::map<Key, int64_t> resident;  // evictable device arrays -> units
  std::set<Key> host_copy;
  const int64_t base = host ? 0 : int64_t(src.inputs.size()) + units(dag, dag.result);
  if (base > cap)
    fail(DFG_E_NOMEM, "dev_mem_cap of " + std::to_string(cap) + " problem arrays is below the resident inputs and " +
                          "output (" + std::to_string(base) + ")");
  auto live = [&] {
    int64_t l = base;
    for (auto& kv : resident) l += kv.second;
    return l;
  };
  auto note = [&](HybridEvent::Kind k, const Key& v) { hp.ev.push_back(HybridEvent{k, ref_of(v)}); };
  auto make_room = [&](int64_t u, const std::set<Key>& protect, int pos) {
    while (live() + u > cap) {
      const Key* victim = nullptr;
      std::tuple<int, int64_t, int, int> best{};
      for (auto& kv : resident) {
        if (protect.count(kv.first)) continue;
        std::tuple<int, int64_t, int, int> t{next_use(kv.first, pos), kv.second,
                                             kv.first.first == int(Ref::Filter) ? 1 : 0, kv.first.second};
        if (!victim || t > best) {
          victim = &kv.first;
          best = t;
        }
      }
      if (!victim)
        fail(DFG_E_NOMEM, "dev_mem_cap of " + std::to_string(cap) + " problem arrays is below the working set of " +
                              "the filter at position " + std::to_string(pos));
      const Key v = *victim;
      if (v.first == int(Ref::Filter)) {
        if (!host_copy.count(v)) {
          note(HybridEvent::Spill, v);
          host_copy.insert(v);
          hp.d2h += 1;
          hp.d2h_units += resident[v];
        } else {
          note(HybridEvent::Discard, v);
        }
      } else {
        note(HybridEvent::Drop, v);
      }
      resident.erase(v);
    }
  };
  auto bring = [&](const Ref& r, const std::set<Key>& protect, int pos) {
    const Key k = key(r);
    if (resident.count(k) || (!host && r.kind == Ref::Input)) return;
    const int64_t u = units(dag, r);
    make_room(u, protect, pos);
    note(r.kind == Ref::Filter ? HybridEvent::Reload : HybridEvent::Upload, k);
    hp.h2d += 1;
    hp.h2d_units += u;
    resident[k] = u;
  };
  int64_t high = base;
  bool mesh_up = false;
  for (int pos = 0; pos < n; ++pos) {
    const int k = order[size_t(pos)];
    const Filter& f = dag.filters[size_t(k)];
    std::vector<Ref> need;
    std::set<Key> protect;
    for (auto& r : f.in) {
      if (r.kind == Ref::Mesh) {
        if (host && !mesh_up) mesh_up = true, hp.h2d += 4;  // dims, x, y, z (R13)
        continue;
      }
      if (protect.insert(key(r)).second) need.push_back(r);
    }
    for (auto& r : need) bring(r, protect, pos);
    const Ref out{Ref::Filter, k};
    const bool writes_out = !host && dag.result == out && pos == n - 1;
    if (!writes_out) {
      make_room(units(dag, out), protect, pos);
      resident[key(out)] = units(dag, out);
    }
    high = std::max(high, live());
    note(HybridEvent::Run, key(out));
    for (auto& r : f.in) {
      if (r.kind == Ref::Mesh) continue;
      if (--rc[key(r)] == 0) {
        resident.erase(key(r));
        host_copy.erase(key(r));
      }
    }
  }
  const Ref& res = dag.result;
  const Key rk = key(res);
  if (host) {
    if (resident.count(rk)) {
      note(HybridEvent::SinkD2H, rk);
    } else if (host_copy.count(rk)) {
      note(HybridEvent::SinkHost, rk);
    } else {  // a bare input result
      bring(res, {rk}, n);
      high = std::max(high, live());
      note(HybridEvent::SinkD2H, rk);
    }
    if (hp.ev.back().kind == HybridEvent::SinkD2H) {
      hp.d2h += 1;
      hp.d2h_units += units(dag, res);
    }
  } else if (res.kind == Ref::Filter && !resident.count(rk) && !(n > 0 && order[size_t(n - 1)] == res.id)) {
    note(HybridEvent::SinkH2D, rk);
    hp.h2d += 1;
    hp.h2d_units += units(dag, res);
  }
  hp.high = high;
  return hp;
}

int64_t predicted_device_bytes(const Dag& dag, dfg_strategy s, int64_t cells, size_t ts) {
  // Algorithmic device-memory bytes of one execute:
  // fused reads every input once and writes the result once; staged and
  // roundtrip read every kernel argument and write every kernel result.
  Sources src = sources(dag);
  int64_t u = 0;
  if (s == DFG_FUSED || s == DFG_STREAMED || s == DFG_REFERENCE) {
    u = int64_t(src.inputs.size()) + units(dag, dag.result);
  } else {
    for (size_t k = 0; k < dag.filters.size(); ++k) {
      const Filter& f = dag.filters[k];
      if (s == DFG_ROUNDTRIP && host_side(f.op)) continue;
      for (auto& r : f.in)
        if (r.kind != Ref::Mesh) u += units(dag, r);
      u += f.width == 1 ? 1 : 4;
    }
  }
  return u * cells * int64_t(ts);
}

int64_t predicted_pcie_bytes(const Dag& dag, dfg_strategy s, int64_t cells, size_t ts, bool host) {
  Sources src = sources(dag);
  int64_t u = 0;
  if (s != DFG_ROUNDTRIP) {
    if (host) u = int64_t(src.inputs.size()) + units(dag, dag.result);
  } else {
    for (auto& f : dag.filters) {
      if (host_side(f.op)) continue;
      for (auto& r : f.in)
        if (r.kind != Ref::Mesh && (host || r.kind == Ref::Filter)) u += units(dag, r);
      u += f.width == 1 ? 1 : 4;
    }
  }
  return u * cells * int64_t(ts);
}

// ==================================================================== plans
namespace {

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

struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  bool owned = false;     // allocated by this execute
  bool counted = false;   // problem-sized: tracked by the ledger
};

void* dev_alloc(size_t bytes, int dev, cudaStream_t s) {
  void* p = nullptr;
  cudaError_t e = cudaMallocFromPoolAsync(&p, bytes ? bytes : 16, pool_for(dev), s);
  if (e != cudaSuccess) {
    cudaGetLastError();
    fail(e == cudaErrorMemoryAllocation ? DFG_E_NOMEM : DFG_E_CUDA,
         std::string("device allocation of ") + std::to_string(bytes) + " bytes failed: " + cudaGetErrorString(e));
  }
  return p;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

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

// one pool per plan would pin memory per plan; share per process instead
HostPool& host_pool() {
  static HostPool* pool = new HostPool();  // leaked on purpose: outlives plans at exit
  return *pool;
}
std::mutex g_host_mu;

}  // namespace

PlanImpl::~PlanImpl() {
  int cur = -1;
  cudaGetDevice(&cur);
  if (mesh) cudaSetDevice(mesh->device);
  if (ev0) cudaEventDestroy(ev0);
  if (ev1) cudaEventDestroy(ev1);
  for (auto* v : {&kev_free, &kev_pending})
    for (auto& e : *v) {
      cudaEventDestroy(e.first);
      cudaEventDestroy(e.second);
    }
  if (mod.mod) drv().ModuleUnload(mod.mod);
  release_stream_buffers();
  if (sH2D) cudaStreamDestroy(sH2D);
  if (sD2H) cudaStreamDestroy(sD2H);
  if (sHalo) cudaStreamDestroy(sHalo);
  if (evHaloIn) cudaEventDestroy(evHaloIn);
  if (evHaloOut) cudaEventDestroy(evHaloOut);
  if (cur >= 0) cudaSetDevice(cur);
}

std::unique_ptr<PlanImpl> compile_plan(std::shared_ptr<MeshImpl> mesh, const std::string& expr, dfg_strategy s,
                                       size_t cap) {
  if (s != DFG_ROUNDTRIP && s != DFG_STAGED && s != DFG_FUSED && s != DFG_STREAMED && s != DFG_REFERENCE &&
      s != DFG_HYBRID)
    fail(DFG_E_INVALID, "bad strategy");
  std::vector<std::string> names;
  for (auto& kv : mesh->fields) names.push_back(kv.first);
  auto plan = std::make_unique<PlanImpl>();
  plan->mesh = mesh;
  plan->strategy = s;
  plan->cap = cap;
  int ref = 0;
  if (s == DFG_REFERENCE) {
    const char* prog = reference_program(expr, &ref);
    if (!prog) fail(DFG_E_INVALID, "reference kernels exist for \"velmag\", \"vortmag\" and \"qcrit\"");
    plan->dag = build_dag(prog, names, mesh->dt);
  } else {
    plan->dag = build_dag(expr, names, mesh->dt);
  }
  const Dag& dag = plan->dag;
  const bool multi = mesh->nzl != mesh->NZ || mesh->nx != mesh->NX || mesh->ny != mesh->NY || mesh->gxy;
  if (multi && s != DFG_FUSED && s != DFG_REFERENCE)
    fail(DFG_E_UNSUPPORTED, "staged/hybrid/roundtrip/streamed run on a whole mesh; slabs and blocks use fusion");

  // Footprint check against the cap for the binding modes at compile time
  // (the streamed ring is bounded by construction; its ledger checks at run time)
  bool any_host = false;
  for (int i : sources(dag).inputs)
    if (!mesh->fields[dag.inputs[i]].on_device) any_host = true;
  Model mdl = model(dag, s, any_host);
  const size_t unit_bytes = size_t(mesh->cells()) * dsize(mesh->dt);
  size_t need = size_t(mdl.units) * unit_bytes;
  plan->order.resize(dag.filters.size());
  for (size_t k = 0; k < plan->order.size(); ++k) plan->order[k] = int(k);
  if (s == DFG_STAGED || s == DFG_HYBRID) {
    // the paper's list order, unless a cap rejects it and the memory-aware
    // order fits (or DFG_STAGED_ORDER=greedy asks for it); hybrid plans take
    // the memory-aware order whenever the list order does not fit
    const char* env = std::getenv("DFG_STAGED_ORDER");
    const bool force = env && !std::strcmp(env, "greedy");
    if (force || (cap && need > cap)) {
      std::vector<int> g = greedy_staged_order(dag);
      size_t gneed = size_t(staged_units(dag, g, any_host)) * unit_bytes;
      if (force || gneed <= cap || s == DFG_HYBRID) {
        plan->order = g;
        need = gneed;
      }
    }
  }
  if (s == DFG_HYBRID) plan->plan_hybrid_for(any_host);  // DFG_E_NOMEM below a filter's working set
  if (cap && need > cap && s != DFG_STREAMED && s != DFG_HYBRID)
    fail(DFG_E_NOMEM, "predicted device footprint " + std::to_string(need) + " bytes exceeds the cap " +
                          std::to_string(cap));

  DFG_CUDA(cudaSetDevice(mesh->device));
  DFG_CUDA(cudaEventCreate(&plan->ev0));
  DFG_CUDA(cudaEventCreate(&plan->ev1));
  plan->st.last_ms = -1;

  if (s == DFG_FUSED || s == DFG_STREAMED || s == DFG_REFERENCE) {
    FusedConfig cfg;
    const char* var = std::getenv("DFG_FUSED_VARIANT");
    if (var && !std::strcmp(var, "ieee")) cfg.div_mode = 0;
    else if (var && !std::strcmp(var, "fast")) cfg.div_mode = 2;
    if (!mesh->markstein_safe && cfg.div_mode == 1) cfg.div_mode = 0;  // keep results exact
    // exact quotient with two operations on the axes whose divisors all verified;
    // DFG_FUSED_VARIANT=markstein keeps the three-operation correction everywhere
    const bool markstein_only = var && !std::strcmp(var, "markstein");
    if (cfg.div_mode == 1 && mesh->dt == DType::F32 && !markstein_only) cfg.div2 = mesh->div2_mask;
    // scale folding is exact in the normal range only; "ieee" keeps every op
    const char* fold = std::getenv("DFG_SCALE_FOLD");
    cfg.fold = cfg.div_mode != 0 && !(fold && !std::strcmp(fold, "0"));
    const char* ncw = std::getenv("DFG_NCW");
    if (ncw) cfg.ncw = std::max(1, std::min(30, std::atoi(ncw)));
    const char* ctas = std::getenv("DFG_CTAS");
    if (ctas) cfg.ctas = std::max(1, std::min(4, std::atoi(ctas)));
    const char* st = std::getenv("DFG_STAGES");
    if (st) cfg.stages = std::max(2, std::min(16, std::atoi(st)));
    // axis degeneracy (n == 1) is a property of the GLOBAL mesh
    plan->fsrc = generate_fused(dag, mesh->NX, mesh->NY, mesh->NZ, cfg, ref);
    static const std::string kUnit = "dfg_fused.cu";
    const Cubin& cb = nvrtc_compile(plan->fsrc.source, kUnit);  // cached for the process lifetime
    plan->regs = cb.regs;
    plan->spill = cb.spill;
    // the runtime API owns the primary context; make it current for the driver API
    DFG_CUDA(cudaFree(0));
    plan->mod = load_module(cb, !plan->fsrc.layout.stencil_inputs.empty(), plan->fsrc.cfg.has_tma);
    // registers / local memory of the main kernel from the loaded module (the
    // NVRTC log can be empty when the compile is served from a cache)
    CUfunction main_fn = plan->mod.tma ? plan->mod.tma : plan->mod.general ? plan->mod.general : plan->mod.pointwise;
    int nregs = 0, local = 0;
    DFG_CU(drv().FuncGetAttribute(&nregs, CU_FUNC_ATTRIBUTE_NUM_REGS, main_fn));
    DFG_CU(drv().FuncGetAttribute(&local, CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, main_fn));
    plan->regs = nregs;
    plan->spill = local;
    if (plan->mod.tma) {
      size_t smem = fused_tma_smem_bytes(mesh->dt, int(plan->fsrc.layout.stencil_inputs.size() + plan->fsrc.layout.point_inputs.size()), plan->fsrc.cfg.ncw,
                                         plan->fsrc.cfg.stages);
      DFG_CU(drv().FuncSetAttribute(plan->mod.tma, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(smem)));
      DFG_CU(drv().FuncSetAttribute(plan->mod.tma_multi, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(smem)));
    }
  }
  return plan;
}

std::pair<cudaEvent_t, cudaEvent_t> PlanImpl::kernel_events() {
  std::pair<cudaEvent_t, cudaEvent_t> e;
  if (!kev_free.empty()) {
    e = kev_free.back();
    kev_free.pop_back();
  } else {
    DFG_CUDA(cudaEventCreate(&e.first));
    DFG_CUDA(cudaEventCreate(&e.second));
  }
  kev_pending.push_back(e);
  return e;
}

void PlanImpl::resolve_kernel_times() {
  for (auto& e : kev_pending) {
    DFG_CUDA(cudaEventSynchronize(e.second));
    float ms = 0;
    DFG_CUDA(cudaEventElapsedTime(&ms, e.first, e.second));
    st.kernel_ms_sum += ms;
    st.kernel_launches_timed += 1;
    kev_free.push_back(e);
  }
  kev_pending.clear();
}

// -------------------------------------------------------------- halo
void PlanImpl::halo_exchange(const std::vector<int>& inputs, cudaStream_t s) {
  MeshImpl& m = *mesh;
  const bool has_lo = m.k0 > 0, has_hi = m.k0 + m.nzl < m.NZ;
  if ((!has_lo && !has_hi) || m.ghosts_supplied) return;  // blocks: the caller filled the ghosts
  const size_t ts = dsize(m.dt);
  const size_t pb = size_t(m.plane()) * ts;
  auto lo = m.link_lo.lock(), hi = m.link_hi.lock();
  if (m.nccl) {
    auto& api = nccl();
    ncclComm_t comm = static_cast<ncclComm_t>(m.nccl);
    ncclDataType_t t = m.dt == DType::F32 ? ncclFloat32 : ncclFloat64;
    nccl_check(api.GroupStart(), "ncclGroupStart");
    for (int in : inputs) {
      char* base = static_cast<char*>(m.fields[dag.inputs[in]].ptr);
      if (has_lo) {
        nccl_check(api.Send(base + 1 * pb, size_t(m.plane()), t, m.rank - 1, comm, s), "ncclSend");
        nccl_check(api.Recv(base + 0 * pb, size_t(m.plane()), t, m.rank - 1, comm, s), "ncclRecv");
      }
      if (has_hi) {
        nccl_check(api.Send(base + size_t(m.nzl) * pb, size_t(m.plane()), t, m.rank + 1, comm, s), "ncclSend");
        nccl_check(api.Recv(base + size_t(m.nzl + 1) * pb, size_t(m.plane()), t, m.rank + 1, comm, s), "ncclRecv");
      }
    }
    nccl_check(api.GroupEnd(), "ncclGroupEnd");
  } else if (lo || hi || (has_lo && !lo) || (has_hi && !hi)) {
    if ((has_lo && !lo) || (has_hi && !hi))
      fail(DFG_E_INVALID, "slab has neighbours but no halo transport (dfg_mesh_init_comm / dfg_mesh_link_local)");
    for (int in : inputs) {
      const std::string& name = dag.inputs[in];
      char* base = static_cast<char*>(m.fields[name].ptr);
      if (has_lo) {
        auto it = lo->fields.find(name);
        if (it == lo->fields.end() || !it->second.ptr || !it->second.on_device)
          fail(DFG_E_UNBOUND, "linked slab below has no device field '" + name + "'");
        DFG_CUDA(cudaMemcpyPeerAsync(base, m.device, static_cast<char*>(it->second.ptr) + size_t(lo->nzl) * pb,
                                     lo->device, pb, s));
      }
      if (has_hi) {
        auto it = hi->fields.find(name);
        if (it == hi->fields.end() || !it->second.ptr || !it->second.on_device)
          fail(DFG_E_UNBOUND, "linked slab above has no device field '" + name + "'");
        DFG_CUDA(cudaMemcpyPeerAsync(base + size_t(m.nzl + 1) * pb, m.device, static_cast<char*>(it->second.ptr) + pb,
                                     hi->device, pb, s));
      }
    }
  }
  st.halo_bytes += int64_t(inputs.size()) * int64_t((has_lo ? 1 : 0) + (has_hi ? 1 : 0)) * int64_t(pb);
}

// -------------------------------------------------------------- execute
void PlanImpl::execute(void* out, bool out_dev, cudaStream_t s) {
  if (!out) fail(DFG_E_INVALID, "null output pointer");
  MeshImpl& m = *mesh;
  DFG_CUDA(cudaSetDevice(m.device));
  for (int i : sources(dag).inputs) {
    auto it = m.fields.find(dag.inputs[i]);
    if (it == m.fields.end() || !it->second.ptr) fail(DFG_E_UNBOUND, "input '" + dag.inputs[i] + "' is not bound");
  }
  DFG_CUDA(cudaEventRecord(ev0, s));
  switch (strategy) {
    case DFG_FUSED: exec_fused(out, out_dev, s); break;
    case DFG_STREAMED: exec_streamed(out, out_dev, s); break;
    case DFG_REFERENCE: exec_fused(out, out_dev, s); break;
    case DFG_STAGED: exec_staged(out, out_dev, s); break;
    case DFG_HYBRID: exec_hybrid(out, out_dev, s); break;
    case DFG_ROUNDTRIP: exec_roundtrip(out, out_dev, s); break;
  }
  DFG_CUDA(cudaEventRecord(ev1, s));
  DFG_CUDA(cudaGetLastError());
  timed = true;
  st.executes += 1;
  bool any_host = !out_dev;
  for (int i : sources(dag).inputs)
    if (!m.fields[dag.inputs[i]].on_device) any_host = true;
  const int64_t unit_b = m.cells() * int64_t(dsize(m.dt));
  const int64_t units = strategy == DFG_HYBRID   ? hyb.high
                        : strategy == DFG_STAGED ? staged_units(dag, order, any_host)
                                                 : model(dag, strategy, any_host).units;
  st.predicted_highwater_bytes = units * unit_b;
  st.predicted_hbm_bytes = predicted_device_bytes(dag, strategy, m.cells(), dsize(m.dt));
  st.predicted_pcie_bytes = strategy == DFG_HYBRID ? (hyb.h2d_units + hyb.d2h_units) * unit_b
                                                   : predicted_pcie_bytes(dag, strategy, m.cells(), dsize(m.dt), any_host);
}

namespace {
// CUtensorMap for one stencil field: dims {nx, ny, nzl + 2g}, box
// {32*VEC + 2*VEC, NCW + 2, 1}, OOB fill zero (never read: clamped in smem).
void encode_map(CUtensorMap* map, const SlabView& m, void* base, int ncw) {
  const size_t ts = dsize(m.dt);
  const int vec = int(16 / ts);
  cuuint64_t gdim[3] = {cuuint64_t(m.px()), cuuint64_t(m.py()), cuuint64_t(m.nzl + 2 * m.ghost)};
  cuuint64_t gstride[2] = {cuuint64_t(m.px()) * ts, cuuint64_t(m.px() * m.py()) * ts};
  cuuint32_t box[3] = {cuuint32_t(32 * vec + 2 * vec), cuuint32_t(ncw + 2), 1};
  cuuint32_t estr[3] = {1, 1, 1};
  DFG_CU(drv().TensorMapEncodeTiled(map, m.dt == DType::F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64,
                                3, base, gdim, gstride, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE));
}

// Host mirror of DfgParams in skeleton.cuh (same field order and widths).
std::vector<uint64_t> pack_params(const std::vector<const void*>& f, void* out, const void* tx, const void* ty,
                                  const void* tz, const SlabView& m, int64_t kbeg, int64_t kend, int64_t items,
                                  int tiles_x, int tiles_y, int kz, int vec_ok) {
  std::vector<uint64_t> w;
  for (auto p : f) w.push_back(reinterpret_cast<uint64_t>(p));
  if (f.empty()) w.push_back(0);
  w.push_back(reinterpret_cast<uint64_t>(out));
  w.push_back(reinterpret_cast<uint64_t>(tx));
  w.push_back(reinterpret_cast<uint64_t>(ty));
  w.push_back(reinterpret_cast<uint64_t>(tz));
  for (int64_t v : {m.nx, m.ny, m.nzl, m.NZ, m.k0, int64_t(m.ghost), kbeg, kend, items, m.NX, m.NY, m.i0, m.j0,
                    m.px(), m.py(), m.gx(), int64_t(m.gxy)})
    w.push_back(uint64_t(v));
  w.push_back(uint64_t(uint32_t(tiles_x)) | (uint64_t(uint32_t(tiles_y)) << 32));
  w.push_back(uint64_t(uint32_t(kz)) | (uint64_t(uint32_t(vec_ok)) << 32));
  // nzero = -0.0 in T (the contraction guard of the paired blocks)
  w.push_back(m.dt == DType::F32 ? uint64_t(0x80000000u) : uint64_t(0x8000000000000000ull));
  return w;
}
}  // namespace

void PlanImpl::exec_fused(void* out, bool out_dev, cudaStream_t s) {
  MeshImpl& m = *mesh;
  const size_t ts = dsize(m.dt);
  const FusedLayout& L = fsrc.layout;
  const int64_t N = m.cells();
  Ledger led(cap);
  std::vector<void*> scratch;
  struct Free {
    std::vector<void*>& v;
    cudaStream_t s;
    ~Free() {
      for (void* p : v) cudaFreeAsync(p, s);
    }
  } guard{scratch, s};

  bool any_host = false;
  for (int i : L.stencil_inputs) any_host |= !m.fields[dag.inputs[i]].on_device;
  for (int i : L.point_inputs) any_host |= !m.fields[dag.inputs[i]].on_device;
  if (any_host && m.nzl != m.NZ && !m.ghosts_supplied)
    fail(DFG_E_UNSUPPORTED, "host-pointer fields are single-slab only");

  // inputs: resident (in situ) or uploaded once (host interface, Table II "Dev-W")
  auto input_ptr = [&](int in) -> const void* {
    Binding& b = m.fields[dag.inputs[in]];
    size_t bytes = m.field_bytes();
    led.add(bytes);
    if (b.on_device) return b.ptr;
    void* d = dev_alloc(bytes, m.device, s);
    scratch.push_back(d);
    DFG_CUDA(cudaMemcpyAsync(d, b.ptr, bytes, cudaMemcpyHostToDevice, s));
    st.h2d_count += 1;
    st.h2d_bytes += int64_t(bytes);
    return d;
  };
  std::vector<const void*> fptr;
  std::vector<int> order;  // first-use order for the upload sequence
  for (int i : sources(dag).inputs) order.push_back(i);
  std::map<int, const void*> got;
  for (int i : order) got[i] = input_ptr(i);
  for (int i : L.stencil_inputs) fptr.push_back(got[i]);
  for (int i : L.point_inputs) fptr.push_back(got[i]);

  // z-slab of a multi-GPU mesh: the ghost planes arrive while the interior
  // planes (which read only owned planes) compute; the one or two planes next
  // to a ghost plane run after the exchange.  DFG_HALO_OVERLAP=0: serial.
  const bool need_lo = m.k0 > 0, need_hi = m.k0 + m.nzl < m.NZ;
  const bool halo = !any_host && !L.stencil_inputs.empty() && (need_lo || need_hi) && !m.ghosts_supplied;
  const char* ov = std::getenv("DFG_HALO_OVERLAP");
  const bool overlap = halo && m.nzl >= 3 && !(ov && !std::strcmp(ov, "0"));
  if (halo && !overlap) halo_exchange(L.stencil_inputs, s);
  if (overlap) {
    if (!sHalo) DFG_CUDA(cudaStreamCreateWithFlags(&sHalo, cudaStreamNonBlocking));
    if (!evHaloIn) DFG_CUDA(cudaEventCreateWithFlags(&evHaloIn, cudaEventDisableTiming));
    if (!evHaloOut) DFG_CUDA(cudaEventCreateWithFlags(&evHaloOut, cudaEventDisableTiming));
    DFG_CUDA(cudaEventRecord(evHaloIn, s));
    DFG_CUDA(cudaStreamWaitEvent(sHalo, evHaloIn, 0));
    halo_exchange(L.stencil_inputs, sHalo);
    DFG_CUDA(cudaEventRecord(evHaloOut, sHalo));
  }

  // mesh arrays: resident, or uploaded like the paper's dims/x/y/z (L225)
  const void* tab[3] = {m.dev_tab[0], m.dev_tab[1], m.dev_tab[2]};
  if (L.has_grad && any_host) {
    int64_t dims[4] = {m.nx, m.ny, m.NZ, m.k0};
    void* dd = dev_alloc(sizeof(dims), m.device, s);
    scratch.push_back(dd);
    DFG_CUDA(cudaMemcpyAsync(dd, dims, sizeof(dims), cudaMemcpyHostToDevice, s));
    st.h2d_count += 1;
    st.h2d_bytes += sizeof(dims);
    for (int a = 0; a < 3; ++a) {
      void* d = dev_alloc(m.host_tab[a].size(), m.device, s);
      scratch.push_back(d);
      DFG_CUDA(cudaMemcpyAsync(d, m.host_tab[a].data(), m.host_tab[a].size(), cudaMemcpyHostToDevice, s));
      st.h2d_count += 1;
      st.h2d_bytes += int64_t(m.host_tab[a].size());
      tab[a] = d;
    }
  }

  const size_t out_bytes = size_t(N) * size_t(L.outw) * ts;
  led.add(out_bytes);
  void* dout = out;
  if (!out_dev) {
    dout = dev_alloc(out_bytes, m.device, s);
    scratch.push_back(dout);
  }

  if (overlap) {
    const int64_t a = m.k0 + (need_lo ? 1 : 0), b = m.k0 + m.nzl - (need_hi ? 1 : 0);
    launch_fused(fptr, dout, tab, SlabView::of(m), s, a, b);
    DFG_CUDA(cudaStreamWaitEvent(s, evHaloOut, 0));
    if (need_lo) launch_fused(fptr, dout, tab, SlabView::of(m), s, m.k0, m.k0 + 1);
    if (need_hi) launch_fused(fptr, dout, tab, SlabView::of(m), s, b, b + 1);
  } else {
    launch_fused(fptr, dout, tab, SlabView::of(m), s);
  }
  if (!out_dev) {
    DFG_CUDA(cudaMemcpyAsync(out, dout, out_bytes, cudaMemcpyDeviceToHost, s));
    st.d2h_count += 1;
    st.d2h_bytes += int64_t(out_bytes);
    DFG_CUDA(cudaStreamSynchronize(s));
  }
  st.dev_highwater_bytes = std::max<int64_t>(st.dev_highwater_bytes, int64_t(led.high));
}

// One launch of the generated kernel over the owned planes of a slab view
// (the mesh itself, or one z-chunk of the streamed strategy).
void PlanImpl::launch_fused(const std::vector<const void*>& fptr, void* dout, const void* const tab[3],
                            const SlabView& m, cudaStream_t s, int64_t kb, int64_t ke) {
  const size_t ts = dsize(m.dt);
  const FusedLayout& L = fsrc.layout;
  const int64_t kbeg = kb < 0 ? m.k0 : kb, kend = ke < 0 ? m.k0 + m.nzl : ke;
  const int64_t N = m.nx * m.ny * (kend - kbeg);
  const int vec = int(16 / ts);
  bool vec_ok = aligned16(dout) && (N % vec == 0) && m.gxy == 0 && m.px() == m.nx && m.gx() == 0;
  for (auto p : fptr) vec_ok = vec_ok && aligned16(p);
  const char* force = std::getenv("DFG_FUSED_KERNEL");
  bool want_general = force && !std::strcmp(force, "general");
  const int sms = sm_count(mesh->device);

  if (L.stencil_inputs.empty()) {
    auto w = pack_params(fptr, dout, tab[0], tab[1], tab[2], m, kbeg, kend, 0, 0, 0, 0, vec_ok ? 1 : 0);
    void* args[] = {w.data()};
    long long work = vec_ok ? N / vec : N;
    unsigned grid = unsigned(std::max<long long>(1, std::min<long long>((work + 255) / 256, sms * 8LL)));
    auto ke = kernel_events();
    DFG_CUDA(cudaEventRecord(ke.first, s));
    DFG_CU(drv().LaunchKernel(mod.pointwise, grid, 1, 1, 256, 1, 1, 0, s, args, nullptr));
    DFG_CUDA(cudaEventRecord(ke.second, s));
    last_variant = 3;
  } else if (mod.tma && !want_general && m.nx % vec == 0 && m.px() % vec == 0 && m.gx() % vec == 0 &&
             aligned16(dout) &&
             std::all_of(fptr.begin(), fptr.end(), [](const void* p) { return aligned16(p); })) {
    const int ncw = fsrc.cfg.ncw;
    const int nsf = int(L.stencil_inputs.size() + L.point_inputs.size());  // TMA tiles per stage
    const int tiles_x = int((m.nx + 32 * vec - 1) / (32 * vec));
    const int tiles_y = int((m.ny + ncw - 1) / ncw);
    const int64_t range = kend - kbeg;
    size_t smem = fused_tma_smem_bytes(m.dt, nsf, ncw, fsrc.cfg.stages);
    int occ = 1;
    DFG_CU(drv().OccupancyMaxActiveBlocksPerMultiprocessor(&occ, mod.tma, (ncw + 1) * 32, smem));
    occ = std::max(occ, 1);
    const int64_t slots = int64_t(sms) * occ;
    // z-chunk length: balance whole rounds of items over the persistent CTAs
    // against the two extra (z-halo) planes each chunk loads.
    int64_t best_kz = range, best_cost = INT64_MAX;
    const char* kzenv = std::getenv("DFG_KZ");
    if (kzenv) {
      best_kz = std::max<int64_t>(1, std::min<int64_t>(range, std::atoll(kzenv)));
    } else {
      for (int64_t kz = 1; kz <= range; kz = kz < 8 ? kz + 1 : kz + std::max<int64_t>(1, kz / 8)) {
        int64_t items = int64_t(tiles_x) * tiles_y * ((range + kz - 1) / kz);
        int64_t rounds = (items + slots - 1) / slots;
        int64_t cost = rounds * (std::min(kz, range) + 2 + 4);  // +4: pipeline fill per item
        if (cost < best_cost) {
          best_cost = cost;
          best_kz = kz;
        }
      }
    }
    const int64_t items = int64_t(tiles_x) * tiles_y * ((range + best_kz - 1) / best_kz);
    const unsigned grid = unsigned(std::min<int64_t>(items, slots));
    // parameter blob: DfgTmap map[NSF_] (128 B each, 64-aligned) then DfgParams
    auto w = pack_params(fptr, dout, tab[0], tab[1], tab[2], m, kbeg, kend, items, tiles_x, tiles_y, int(best_kz),
                         vec_ok ? 1 : 0);
    size_t pbytes = size_t(nsf) * 128 + w.size() * 8;
    pbytes = (pbytes + 63) / 64 * 64;
    alignas(64) unsigned char blob[8 * 128 + 512];
    if (pbytes > sizeof(blob)) fail(DFG_E_UNSUPPORTED, "too many stencil fields for the TMA kernel");
    std::memset(blob, 0, sizeof(blob));
    for (int f = 0; f < nsf; ++f)
      encode_map(reinterpret_cast<CUtensorMap*>(blob + 128 * f), m, const_cast<void*>(fptr[f]), ncw);
    std::memcpy(blob + 128 * nsf, w.data(), w.size() * 8);
    void* args[] = {blob};
    auto ke = kernel_events();
    DFG_CUDA(cudaEventRecord(ke.first, s));
    DFG_CU(drv().LaunchKernel(mod.tma, grid, 1, 1, (ncw + 1) * 32, 1, 1, unsigned(smem), s, args, nullptr));
    DFG_CUDA(cudaEventRecord(ke.second, s));
    last_variant = 1;
  } else {
    // z-marching columns: enough (column, z-chunk) units to fill the device
    // (~2048 threads per SM), each chunk as long as that allows
    const int64_t cols = m.nx * m.ny, range = kend - kbeg;
    const int64_t chunks = std::max<int64_t>(1, std::min<int64_t>(range, (int64_t(sms) * 2048 + cols - 1) / cols));
    const int64_t kz = (range + chunks - 1) / chunks;
    const int64_t units = cols * ((range + kz - 1) / kz);
    auto w = pack_params(fptr, dout, tab[0], tab[1], tab[2], m, kbeg, kend, 0, 0, 0, int(kz), 0);
    void* args[] = {w.data()};
    unsigned grid = unsigned(std::max<long long>(1, std::min<long long>((units + 255) / 256, sms * 8LL)));
    auto ke = kernel_events();
    DFG_CUDA(cudaEventRecord(ke.first, s));
    DFG_CU(drv().LaunchKernel(mod.general, grid, 1, 1, 256, 1, 1, 0, s, args, nullptr));
    DFG_CUDA(cudaEventRecord(ke.second, s));
    last_variant = 2;
  }
  st.kernel_count += 1;
}

// Several fused plans of one network (one generated module) in a single
// launch of dfg_fused_tma_multi: per-block parameter blobs (tensor maps +
// DfgParams, the layout of DfgTmaParams) go to device memory, the persistent
// CTAs walk the concatenated item space.  Plans that cannot share the launch
// run one by one (same results).
void execute_blocks(const std::vector<PlanImpl*>& plans, const std::vector<void*>& outs, cudaStream_t s) {
  if (plans.empty()) return;
  PlanImpl& p0 = *plans[0];
  const MeshImpl& m0 = *p0.mesh;
  const size_t ts = dsize(m0.dt);
  const int vec = int(16 / ts);
  const FusedLayout& L = p0.fsrc.layout;
  const char* force = std::getenv("DFG_FUSED_KERNEL");
  bool batch = plans.size() > 1 && p0.strategy == DFG_FUSED && p0.mod.tma_multi && p0.fsrc.cfg.has_tma &&
               !(force && !std::strcmp(force, "general"));
  std::vector<std::vector<const void*>> fptrs(plans.size());
  for (size_t b = 0; b < plans.size() && batch; ++b) {
    PlanImpl& p = *plans[b];
    const MeshImpl& m = *p.mesh;
    const bool halo = (m.k0 > 0 || m.k0 + m.nzl < m.NZ) && !m.ghosts_supplied;
    batch = p.strategy == DFG_FUSED && p.fsrc.source == p0.fsrc.source && m.device == m0.device && !halo &&
            m.nx % vec == 0 && m.px() % vec == 0 && m.gx() % vec == 0 && aligned16(outs[b]);
    std::vector<int> ins = L.stencil_inputs;
    ins.insert(ins.end(), L.point_inputs.begin(), L.point_inputs.end());
    for (int i : ins) {
      auto it = m.fields.find(p.dag.inputs[size_t(i)]);
      if (it == m.fields.end() || !it->second.ptr) fail(DFG_E_UNBOUND, "input '" + p.dag.inputs[size_t(i)] + "' is not bound");
      batch = batch && it->second.on_device && aligned16(it->second.ptr);
      fptrs[b].push_back(it->second.ptr);
    }
  }
  if (!batch) {
    for (size_t b = 0; b < plans.size(); ++b) plans[b]->execute(outs[b], true, s);
    return;
  }
  DFG_CUDA(cudaSetDevice(m0.device));
  const int ncw = p0.fsrc.cfg.ncw;
  const int nsf = int(L.stencil_inputs.size() + L.point_inputs.size());
  const size_t smem = fused_tma_smem_bytes(m0.dt, nsf, ncw, p0.fsrc.cfg.stages);
  int occ = 1;
  DFG_CU(drv().OccupancyMaxActiveBlocksPerMultiprocessor(&occ, p0.mod.tma_multi, (ncw + 1) * 32, smem));
  const int64_t slots = int64_t(sm_count(m0.device)) * std::max(occ, 1);
  // one z-chunk length for the batch: whole rounds of the concatenated items
  // against the two halo planes per chunk (as launch_fused)
  int64_t max_range = 1;
  for (auto* p : plans) max_range = std::max(max_range, p->mesh->nzl);
  auto items_for = [&](int64_t kz) {
    int64_t t = 0;
    for (auto* p : plans) {
      const MeshImpl& m = *p->mesh;
      t += int64_t((m.nx + 32 * vec - 1) / (32 * vec)) * ((m.ny + ncw - 1) / ncw) * ((m.nzl + kz - 1) / kz);
    }
    return t;
  };
  int64_t best_kz = max_range, best_cost = INT64_MAX;
  for (int64_t kz = 1; kz <= max_range; kz = kz < 8 ? kz + 1 : kz + std::max<int64_t>(1, kz / 8)) {
    const int64_t cost = (items_for(kz) + slots - 1) / slots * (kz + 2 + 4);
    if (cost < best_cost) best_cost = cost, best_kz = kz;
  }
  // blobs: DfgTmaParams per block, 64-byte aligned stride
  std::vector<std::vector<uint64_t>> words;
  std::vector<int64_t> first{0};
  size_t wmax = 0;
  for (size_t b = 0; b < plans.size(); ++b) {
    const MeshImpl& m = *plans[b]->mesh;
    const SlabView v = SlabView::of(m);
    const int tx = int((m.nx + 32 * vec - 1) / (32 * vec)), ty = int((m.ny + ncw - 1) / ncw);
    const int64_t items = int64_t(tx) * ty * ((m.nzl + best_kz - 1) / best_kz);
    words.push_back(pack_params(fptrs[b], outs[b], m.dev_tab[0], m.dev_tab[1], m.dev_tab[2], v, m.k0, m.k0 + m.nzl,
                                items, tx, ty, int(best_kz), 0));
    wmax = std::max(wmax, words.back().size());
    first.push_back(first.back() + items);
  }
  const size_t stride = (size_t(nsf) * 128 + wmax * 8 + 63) / 64 * 64;
  std::vector<unsigned char> host(stride * plans.size() + sizeof(int64_t) * first.size(), 0);
  for (size_t b = 0; b < plans.size(); ++b) {
    unsigned char* blob = host.data() + stride * b;
    const SlabView v = SlabView::of(*plans[b]->mesh);
    for (int f = 0; f < nsf; ++f) encode_map(reinterpret_cast<CUtensorMap*>(blob + 128 * f), v, const_cast<void*>(fptrs[b][size_t(f)]), ncw);
    std::memcpy(blob + 128 * nsf, words[b].data(), words[b].size() * 8);
  }
  std::memcpy(host.data() + stride * plans.size(), first.data(), sizeof(int64_t) * first.size());
  void* dev = dev_alloc(host.size(), m0.device, s);
  DFG_CUDA(cudaMemcpyAsync(dev, host.data(), host.size(), cudaMemcpyHostToDevice, s));  // pageable: staged now
  struct {
    const void* blocks;
    const void* first;
    int nb;
  } arg{dev, static_cast<char*>(dev) + stride * plans.size(), int(plans.size())};
  void* args[] = {&arg};
  DFG_CUDA(cudaEventRecord(p0.ev0, s));
  auto ke = p0.kernel_events();
  DFG_CUDA(cudaEventRecord(ke.first, s));
  const unsigned grid = unsigned(std::max<int64_t>(1, std::min(first.back(), slots)));
  DFG_CU(drv().LaunchKernel(p0.mod.tma_multi, grid, 1, 1, (ncw + 1) * 32, 1, 1, unsigned(smem), s, args, nullptr));
  DFG_CUDA(cudaEventRecord(ke.second, s));
  DFG_CUDA(cudaEventRecord(p0.ev1, s));
  DFG_CUDA(cudaFreeAsync(dev, s));
  DFG_CUDA(cudaGetLastError());
  p0.timed = true;
  p0.st.kernel_count += 1;
  for (auto* p : plans) {
    p->st.executes += 1;
    p->last_variant = 4;
  }
}

// ----------------------------------------------------------- streamed
// The paper's future-work streaming strategy (L344, L245): host-resident
// fields flow through a ring of DFG_STREAM_SLOTS z-chunk slabs.  Chunk c
// (planes [a, b)) is uploaded with one ghost plane on each side (the
// neighbour planes inside the mesh), computed by the fused kernel exactly as
// a z-slab with ghost = 1, and downloaded -- upload, compute and download of
// different chunks overlap on three streams.  Device memory is bounded by the
// ring, so meshes larger than HBM run too.
void PlanImpl::exec_streamed(void* out, bool out_dev, cudaStream_t s) {
  MeshImpl& m = *mesh;
  const FusedLayout& L = fsrc.layout;
  bool all_dev = out_dev;
  for (int i : sources(dag).inputs) all_dev = all_dev && m.fields[dag.inputs[i]].on_device;
  if (all_dev) return exec_fused(out, out_dev, s);  // nothing to stream: in situ
  if (m.nzl != m.NZ) fail(DFG_E_UNSUPPORTED, "the streamed strategy runs on a single slab");
  const size_t ts = dsize(m.dt);
  const int64_t plane = m.plane();
  const int64_t pb = plane * int64_t(ts);
  const int nf = int(L.stencil_inputs.size() + L.point_inputs.size());
  std::vector<int> fin;  // input index per kernel field slot
  for (int i : L.stencil_inputs) fin.push_back(i);
  for (int i : L.point_inputs) fin.push_back(i);

  // chunk height: ~512 MiB of input per chunk, at least 4 planes (balances the
  // pipeline fill / drain against per-chunk overheads)
  int64_t C = std::max<int64_t>(4, (512ll << 20) / std::max<int64_t>(1, pb * std::max(nf, 1)));
  if (const char* e = std::getenv("DFG_STREAM_PLANES")) C = std::max<int64_t>(1, std::atoll(e));
  C = std::min<int64_t>(C, m.nzl);
  const int64_t nchunks = (m.nzl + C - 1) / C;
  const int R = int(std::min<int64_t>(kStreamSlots, nchunks));

  // ring buffers (cached in the plan; the ledger counts them)
  const size_t in_bytes = size_t(C + 2) * size_t(pb), out_bytes = size_t(C) * size_t(pb) * size_t(L.outw);
  if (!stream_ready || stream_C != C || stream_R != R) {
    release_stream_buffers();
    for (int r = 0; r < R; ++r) {
      for (int f = 0; f < nf; ++f) {
        void* p = nullptr;
        DFG_CUDA(cudaMalloc(&p, in_bytes));
        stream_in.push_back(p);
      }
      void* p = nullptr;
      DFG_CUDA(cudaMalloc(&p, out_bytes));
      stream_out.push_back(p);
    }
    for (auto* x : {&sH2D, &sD2H})
      if (!*x) DFG_CUDA(cudaStreamCreateWithFlags(x, cudaStreamNonBlocking));
    stream_C = C;
    stream_R = R;
    stream_ready = true;
  }
  Ledger led(cap);
  led.add(size_t(R) * (size_t(nf) * in_bytes + out_bytes));

  std::vector<cudaEvent_t> ev;
  auto new_event = [&]() {
    cudaEvent_t e;
    DFG_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    ev.push_back(e);
    return e;
  };
  struct Destroy {
    std::vector<cudaEvent_t>& v;
    ~Destroy() {
      for (auto e : v) cudaEventDestroy(e);
    }
  } guard{ev};
  cudaEvent_t start = new_event();
  DFG_CUDA(cudaEventRecord(start, s));
  DFG_CUDA(cudaStreamWaitEvent(sH2D, start, 0));
  DFG_CUDA(cudaStreamWaitEvent(sD2H, start, 0));
  std::vector<cudaEvent_t> computed(nchunks), downloaded(nchunks);
  const void* tab[3] = {m.dev_tab[0], m.dev_tab[1], m.dev_tab[2]};
  for (int64_t c = 0; c < nchunks; ++c) {
    const int r = int(c % R);
    const int64_t a = c * C, b = std::min(m.nzl, a + C);
    const int64_t lo = std::max<int64_t>(a - 1, 0), hi = std::min<int64_t>(b + 1, m.NZ);
    // slot r is free once chunk c-R was computed (inputs) and downloaded (output)
    if (c >= R) {
      DFG_CUDA(cudaStreamWaitEvent(sH2D, computed[c - R], 0));
      DFG_CUDA(cudaStreamWaitEvent(s, downloaded[c - R], 0));
    }
    std::vector<const void*> fptr;
    for (int f = 0; f < nf; ++f) {
      char* dst = static_cast<char*>(stream_in[size_t(r) * nf + f]);
      const Binding& bd = m.fields[dag.inputs[fin[f]]];
      // local plane index of global plane g is g - a + 1 (ghost plane 0)
      int64_t from = lo;
      if (c > 0) {
        // planes a-1 and a already sit in the previous slot (its local C, C+1)
        const char* prev = static_cast<const char*>(stream_in[size_t((c - 1) % R) * nf + f]);
        DFG_CUDA(cudaMemcpyAsync(dst, prev + C * pb, size_t(2 * pb), cudaMemcpyDeviceToDevice, sH2D));
        from = a + 1;
      }
      if (hi > from) {
        const char* src = static_cast<const char*>(bd.ptr) + (from + m.ghost) * pb;
        DFG_CUDA(cudaMemcpyAsync(dst + (from - a + 1) * pb, src, size_t(hi - from) * size_t(pb),
                                 bd.on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, sH2D));
        if (!bd.on_device) {
          st.h2d_count += 1;
          st.h2d_bytes += (hi - from) * pb;
        }
      }
      fptr.push_back(dst);
    }
    cudaEvent_t up = new_event();
    DFG_CUDA(cudaEventRecord(up, sH2D));
    DFG_CUDA(cudaStreamWaitEvent(s, up, 0));
    SlabView v = SlabView::of(m);
    v.nzl = b - a;
    v.k0 = a;
    v.ghost = 1;
    launch_fused(fptr, stream_out[r], tab, v, s);
    computed[c] = new_event();
    DFG_CUDA(cudaEventRecord(computed[c], s));
    DFG_CUDA(cudaStreamWaitEvent(sD2H, computed[c], 0));
    char* dsto = static_cast<char*>(out) + a * pb * int64_t(L.outw);
    DFG_CUDA(cudaMemcpyAsync(dsto, stream_out[r], size_t(b - a) * size_t(pb) * size_t(L.outw),
                             out_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, sD2H));
    if (!out_dev) {
      st.d2h_count += 1;
      st.d2h_bytes += (b - a) * pb * int64_t(L.outw);
    }
    downloaded[c] = new_event();
    DFG_CUDA(cudaEventRecord(downloaded[c], sD2H));
  }
  // join: the caller's stream waits for the last download and upload
  cudaEvent_t up_done = new_event();
  DFG_CUDA(cudaEventRecord(up_done, sH2D));
  DFG_CUDA(cudaStreamWaitEvent(s, up_done, 0));
  DFG_CUDA(cudaStreamWaitEvent(s, downloaded[nchunks - 1], 0));
  if (!out_dev) DFG_CUDA(cudaStreamSynchronize(s));
  st.dev_highwater_bytes = std::max<int64_t>(st.dev_highwater_bytes, int64_t(led.high));
}

void PlanImpl::release_stream_buffers() {
  for (void* p : stream_in) cudaFree(p);
  for (void* p : stream_out) cudaFree(p);
  stream_in.clear();
  stream_out.clear();
  stream_ready = false;
}

// ------------------------------------------------------------- staged
namespace {
// One primitive kernel over the owned cells of a whole mesh: o = f(args)
// (args: operand values, mesh references skipped); grad3d reads `gsrc`, its
// field's buffer from local plane 0, which has `gghost` ghost planes.
void launch_primitive(const MeshImpl& m, const Filter& f, void* o, const std::vector<const void*>& a,
                      const void* gsrc, int64_t gghost, const void* const tab[3], cudaStream_t s) {
  const int64_t N = m.cells();
  switch (f.op) {
    case Op::Const: kern::fill(m.dt, f.cval, o, N, s); break;
    case Op::Add: case Op::Sub: case Op::Mult: case Op::Div:
    case Op::Gt: case Op::Lt: case Op::Ge: case Op::Le: case Op::Eq: case Op::Ne:
      kern::binary(f.op, m.dt, a[0], a[1], o, N, s);
      break;
    case Op::Neg: case Op::Sqrt: kern::unary(f.op, m.dt, a[0], o, N, s); break;
    case Op::Select: kern::select(m.dt, a[0], a[1], a[2], o, N, s); break;
    case Op::Decompose: kern::decompose(m.dt, a[0], f.k, o, N, s); break;
    case Op::Compose: kern::compose(m.dt, a.data(), int(a.size()), o, N, s); break;
    case Op::Grad3d:
      kern::grad3d(m.dt, gsrc, o, tab[0], tab[1], tab[2], m.nx, m.ny, m.nzl, m.NZ, m.k0, gghost, s);
      break;
  }
}
}  // namespace

void PlanImpl::plan_hybrid_for(bool host) {
  const int64_t unit_b = mesh->cells() * int64_t(dsize(mesh->dt));
  const int64_t cap_units = cap ? int64_t(cap) / unit_b : (int64_t(1) << 40);
  hyb = plan_hybrid(dag, order, cap_units, host);
  hyb_host = host ? 1 : 0;
}

// ------------------------------------------------------------- hybrid
// Replays the compile-time transfer schedule (plan_hybrid): the same
// primitive kernels as staged, plus spills of intermediates to pinned host
// buffers and their reloads.  One stream orders everything; host copies live
// until the end of the execute.
void PlanImpl::exec_hybrid(void* out, bool out_dev, cudaStream_t s) {
  MeshImpl& m = *mesh;
  const size_t ts = dsize(m.dt);
  const size_t sb = size_t(m.cells()) * ts;
  Sources src = sources(dag);
  bool all_host = !out_dev, all_dev = out_dev;
  for (int i : src.inputs) {
    const bool d = m.fields[dag.inputs[i]].on_device;
    all_host = all_host && !d;
    all_dev = all_dev && d;
  }
  if (!all_host && !all_dev)
    fail(DFG_E_UNSUPPORTED, "hybrid: inputs and output must all be in host memory or all on the device");
  const bool host = all_host;
  if (hyb_host != (host ? 1 : 0)) plan_hybrid_for(host);

  Ledger led(cap);
  std::lock_guard<std::mutex> lk(g_host_mu);
  HostPool& hp = host_pool();
  using Key = std::pair<int, int>;
  auto key = [](const Ref& r) { return Key(int(r.kind), r.id); };
  auto bytes_of = [&](const Ref& r) { return sb * size_t(units(dag, r)); };
  std::map<Key, void*> dev, hcopy;
  std::vector<void*> host_bufs;
  struct Cleanup {
    std::map<Key, void*>& dev;
    cudaStream_t s;
    ~Cleanup() {
      for (auto& kv : dev) cudaFreeAsync(kv.second, s);
    }
  } cleanup{dev, s};
  if (!host) {
    for (size_t i = 0; i < src.inputs.size(); ++i) led.add(m.field_bytes());
    led.add(bytes_of(dag.result));  // the caller's output buffer
  }
  std::map<Key, int64_t> rc;
  for (auto& f : dag.filters)
    for (auto& r : f.in)
      if (r.kind != Ref::Mesh) rc[key(r)] += 1;
  rc[key(dag.result)] += 1;

  const void* tab[3] = {m.dev_tab[0], m.dev_tab[1], m.dev_tab[2]};
  std::vector<void*> mesh_bufs;
  auto ensure_mesh = [&] {
    if (!host || !mesh_bufs.empty()) return;
    int64_t dims[4] = {m.nx, m.ny, m.NZ, m.k0};
    void* dd = dev_alloc(sizeof(dims), m.device, s);
    mesh_bufs.push_back(dd);
    DFG_CUDA(cudaMemcpyAsync(dd, dims, sizeof(dims), cudaMemcpyHostToDevice, s));
    st.h2d_count += 1;
    st.h2d_bytes += sizeof(dims);
    for (int a = 0; a < 3; ++a) {
      void* d = dev_alloc(m.host_tab[a].size(), m.device, s);
      mesh_bufs.push_back(d);
      DFG_CUDA(cudaMemcpyAsync(d, m.host_tab[a].data(), m.host_tab[a].size(), cudaMemcpyHostToDevice, s));
      st.h2d_count += 1;
      st.h2d_bytes += int64_t(m.host_tab[a].size());
      tab[a] = d;
    }
  };
  // buffer of a value (inputs: from local plane 0, ghost planes included)
  auto base_of = [&](const Ref& r) -> void* {
    if (!host && r.kind == Ref::Input) return m.fields[dag.inputs[r.id]].ptr;
    auto it = dev.find(key(r));
    if (it == dev.end()) fail(DFG_E_CUDA, "hybrid schedule: operand not resident");
    return it->second;
  };
  const int64_t goff = int64_t(m.ghost) * m.plane() * int64_t(ts);
  auto val = [&](const Ref& r) -> void* {
    return static_cast<char*>(base_of(r)) + (r.kind == Ref::Input ? goff : 0);
  };
  auto drop_dev = [&](const Key& k, size_t b) {
    cudaFreeAsync(dev[k], s);
    dev.erase(k);
    led.sub(b);
  };
  const Ref res = dag.result;
  const size_t nf = order.size();
  size_t pos = 0;
  for (const HybridEvent& e : hyb.ev) {
    const Key k = key(e.ref);
    const size_t b = e.ref.kind == Ref::Input ? m.field_bytes() : bytes_of(e.ref);
    switch (e.kind) {
      case HybridEvent::Upload: {
        led.add(b);
        void* d = dev_alloc(b, m.device, s);
        dev[k] = d;
        DFG_CUDA(cudaMemcpyAsync(d, m.fields[dag.inputs[e.ref.id]].ptr, b, cudaMemcpyHostToDevice, s));
        st.h2d_count += 1;
        st.h2d_bytes += int64_t(b);
        break;
      }
      case HybridEvent::Reload: {
        led.add(b);
        void* d = dev_alloc(b, m.device, s);
        dev[k] = d;
        DFG_CUDA(cudaMemcpyAsync(d, hcopy.at(k), b, cudaMemcpyHostToDevice, s));
        st.h2d_count += 1;
        st.h2d_bytes += int64_t(b);
        break;
      }
      case HybridEvent::Spill: {
        void* h = hp.get(b);
        host_bufs.push_back(h);
        hcopy[k] = h;
        DFG_CUDA(cudaMemcpyAsync(h, dev.at(k), b, cudaMemcpyDeviceToHost, s));
        st.d2h_count += 1;
        st.d2h_bytes += int64_t(b);
        drop_dev(k, b);
        break;
      }
      case HybridEvent::Discard: case HybridEvent::Drop: drop_dev(k, b); break;
      case HybridEvent::Run: {
        const Filter& f = dag.filters[size_t(e.ref.id)];
        std::vector<const void*> args;
        for (auto& r : f.in) {
          if (r.kind == Ref::Mesh) ensure_mesh();
          else args.push_back(val(r));
        }
        const bool writes_out = !host && res == e.ref && pos + 1 == nf;
        void* o = out;
        if (!writes_out) {
          led.add(b);
          o = dev_alloc(b, m.device, s);
          dev[k] = o;
        }
        const void* gsrc = nullptr;
        int64_t gghost = 0;
        if (f.op == Op::Grad3d) {
          gsrc = base_of(f.in[0]);
          gghost = f.in[0].kind == Ref::Input ? m.ghost : 0;
        }
        launch_primitive(m, f, o, args, gsrc, gghost, tab, s);
        DFG_CUDA(cudaGetLastError());
        st.kernel_count += 1;
        ++pos;
        for (auto& r : f.in) {
          if (r.kind == Ref::Mesh || --rc[key(r)] > 0) continue;
          if (dev.count(key(r))) drop_dev(key(r), r.kind == Ref::Input ? m.field_bytes() : bytes_of(r));
          hcopy.erase(key(r));
        }
        break;
      }
      case HybridEvent::SinkD2H:
        DFG_CUDA(cudaMemcpyAsync(out, val(res), bytes_of(res), cudaMemcpyDeviceToHost, s));
        st.d2h_count += 1;
        st.d2h_bytes += int64_t(bytes_of(res));
        break;
      case HybridEvent::SinkHost:
        DFG_CUDA(cudaMemcpyAsync(out, hcopy.at(k), bytes_of(res), cudaMemcpyHostToHost, s));
        break;
      case HybridEvent::SinkH2D:
        DFG_CUDA(cudaMemcpyAsync(out, hcopy.at(k), bytes_of(res), cudaMemcpyHostToDevice, s));
        st.h2d_count += 1;
        st.h2d_bytes += int64_t(bytes_of(res));
        break;
    }
  }
  // device mode: a result still resident (not computed into the output) or a bare input
  if (!host) {
    auto it = dev.find(key(res));
    const void* rp = it != dev.end() ? it->second : nullptr;
    if (res.kind == Ref::Input) rp = val(res);
    if (rp && rp != out) DFG_CUDA(cudaMemcpyAsync(out, rp, bytes_of(res), cudaMemcpyDeviceToDevice, s));
  }
  for (void* p : mesh_bufs) cudaFreeAsync(p, s);
  if (!host_bufs.empty() || host) DFG_CUDA(cudaStreamSynchronize(s));  // host copies / output complete
  for (void* h : host_bufs) hp.put(h);
  st.dev_highwater_bytes = std::max<int64_t>(st.dev_highwater_bytes, int64_t(led.high));
}

void PlanImpl::exec_staged(void* out, bool out_dev, cudaStream_t s) {
  MeshImpl& m = *mesh;
  const size_t ts = dsize(m.dt);
  const int64_t N = m.cells();
  const size_t sb = size_t(N) * ts;  // one scalar problem array
  const int64_t goff = int64_t(m.ghost) * m.plane();
  Ledger led(cap);
  std::vector<void*> to_free;
  struct Free {
    std::vector<void*>& v;
    cudaStream_t s;
    ~Free() {
      for (void* p : v) cudaFreeAsync(p, s);
    }
  } guard{to_free, s};

  Sources src = sources(dag);
  bool host = !out_dev;
  for (int i : src.inputs) host |= !m.fields[dag.inputs[i]].on_device;

  // reference counts (L85): uses as an input, plus the sink
  std::map<std::pair<int, int>, int64_t> rc;
  auto key = [](const Ref& r) { return std::make_pair(int(r.kind), r.id); };
  for (auto& f : dag.filters)
    for (auto& r : f.in)
      if (r.kind != Ref::Mesh) rc[key(r)] += 1;
  rc[key(dag.result)] += 1;

  std::map<int, void*> in_dev;   // input index -> device base (incl. ghost planes)
  std::map<int, bool> in_owned;  // uploaded by us (freed at refcount 0)
  std::vector<void*> fval(dag.filters.size(), nullptr);
  if (!host) {
    for (int i : src.inputs) {
      in_dev[i] = m.fields[dag.inputs[i]].ptr;
      in_owned[i] = false;
      led.add(m.field_bytes());
    }
    led.add(sb * size_t(dag.width(dag.result) == 1 ? 1 : 4));  // the caller's output buffer
  }
  auto ensure_input = [&](int i) {
    if (in_dev.count(i)) return;
    Binding& b = m.fields[dag.inputs[i]];
    if (b.on_device) {
      in_dev[i] = b.ptr;
      in_owned[i] = false;
      led.add(m.field_bytes());
      return;
    }
    size_t bytes = m.field_bytes();
    led.add(bytes);
    void* d = dev_alloc(bytes, m.device, s);
    DFG_CUDA(cudaMemcpyAsync(d, b.ptr, bytes, cudaMemcpyHostToDevice, s));
    st.h2d_count += 1;
    st.h2d_bytes += int64_t(bytes);
    in_dev[i] = d;
    in_owned[i] = true;
  };
  const void* tab[3] = {m.dev_tab[0], m.dev_tab[1], m.dev_tab[2]};
  bool mesh_up = false;
  auto ensure_mesh = [&]() {
    if (mesh_up || !host) return;
    mesh_up = true;
    int64_t dims[4] = {m.nx, m.ny, m.NZ, m.k0};
    void* dd = dev_alloc(sizeof(dims), m.device, s);
    to_free.push_back(dd);
    DFG_CUDA(cudaMemcpyAsync(dd, dims, sizeof(dims), cudaMemcpyHostToDevice, s));
    st.h2d_count += 1;
    st.h2d_bytes += sizeof(dims);
    for (int a = 0; a < 3; ++a) {
      void* d = dev_alloc(m.host_tab[a].size(), m.device, s);
      to_free.push_back(d);
      DFG_CUDA(cudaMemcpyAsync(d, m.host_tab[a].data(), m.host_tab[a].size(), cudaMemcpyHostToDevice, s));
      st.h2d_count += 1;
      st.h2d_bytes += int64_t(m.host_tab[a].size());
      tab[a] = d;
    }
  };
  // value pointer of a ref over the owned cells (inputs skip the ghost plane)
  auto val = [&](const Ref& r) -> const void* {
    if (r.kind == Ref::Filter) return fval[r.id];
    return static_cast<const char*>(in_dev[r.id]) + goff * int64_t(ts);
  };
  auto release = [&](const Ref& r) {
    if (r.kind == Ref::Mesh) return;
    if (--rc[key(r)] > 0) return;
    if (r.kind == Ref::Filter) {
      if (fval[r.id] && fval[r.id] != out) {
        cudaFreeAsync(fval[r.id], s);
        led.sub(sb * size_t(dag.filters[r.id].width == 1 ? 1 : 4));
      }
      fval[r.id] = nullptr;
    } else if (in_owned[r.id]) {
      cudaFreeAsync(in_dev[r.id], s);
      led.sub(m.field_bytes());
      in_dev.erase(r.id);
    }
  };

  const size_t nf = dag.filters.size();
  for (size_t pos = 0; pos < nf; ++pos) {
    const size_t k = size_t(order[pos]);  // list order, or the memory-aware order
    const Filter& f = dag.filters[k];
    for (auto& r : f.in) {
      if (r.kind == Ref::Input) ensure_input(r.id);
      if (r.kind == Ref::Mesh) ensure_mesh();
    }
    const size_t ob = sb * size_t(f.width == 1 ? 1 : 4);
    const bool into_out = out_dev && dag.result.kind == Ref::Filter && dag.result.id == int(k) && pos + 1 == nf;
    void* o;
    if (into_out) {
      o = out;
      if (host) led.add(ob);
    } else {
      led.add(ob);
      o = dev_alloc(ob, m.device, s);
    }
    fval[k] = o;
    std::vector<const void*> args;
    for (auto& r : f.in)
      if (r.kind != Ref::Mesh) args.push_back(val(r));
    const void* gsrc = nullptr;
    int64_t gghost = 0;
    if (f.op == Op::Grad3d) {
      const Ref& a0 = f.in[0];
      gsrc = a0.kind == Ref::Input ? in_dev[a0.id] : fval[a0.id];
      gghost = a0.kind == Ref::Input ? m.ghost : 0;
    }
    launch_primitive(m, f, o, args, gsrc, gghost, tab, s);
    DFG_CUDA(cudaGetLastError());
    st.kernel_count += 1;
    for (auto& r : f.in) release(r);
  }
  // the sink (L80): result -> caller's buffer
  const Ref& res = dag.result;
  const size_t rb = sb * size_t(dag.width(res) == 1 ? 1 : 4);
  const void* rp;
  if (res.kind == Ref::Input) {
    ensure_input(res.id);
    rp = val(res);
  } else {
    rp = fval[res.id];
  }
  if (rp != out) {
    if (out_dev) {
      DFG_CUDA(cudaMemcpyAsync(out, rp, rb, cudaMemcpyDeviceToDevice, s));
    } else {
      DFG_CUDA(cudaMemcpyAsync(out, rp, rb, cudaMemcpyDeviceToHost, s));
      st.d2h_count += 1;
      st.d2h_bytes += int64_t(rb);
    }
  }
  release(res);
  for (auto& kv : in_dev)
    if (in_owned[kv.first]) to_free.push_back(kv.second);
  if (!out_dev) DFG_CUDA(cudaStreamSynchronize(s));
  st.dev_highwater_bytes = std::max<int64_t>(st.dev_highwater_bytes, int64_t(led.high));
}

// ---------------------------------------------------------- roundtrip
void PlanImpl::exec_roundtrip(void* out, bool out_dev, cudaStream_t s) {
  MeshImpl& m = *mesh;
  const size_t ts = dsize(m.dt);
  const int64_t N = m.cells();
  const size_t sb = size_t(N) * ts;
  const int64_t goff = int64_t(m.ghost) * m.plane();
  Ledger led(cap);
  std::lock_guard<std::mutex> lk(g_host_mu);
  HostPool& hp = host_pool();

  Sources src = sources(dag);
  bool host = !out_dev;
  for (int i : src.inputs) host |= !m.fields[dag.inputs[i]].on_device;
  if (!host) {  // in situ: resident inputs and output are live throughout
    for (size_t q = 0; q < src.inputs.size(); ++q) led.add(m.field_bytes());
    led.add(sb * size_t(dag.width(dag.result) == 1 ? 1 : 4));
  }

  std::map<std::pair<int, int>, int64_t> rc;
  auto key = [](const Ref& r) { return std::make_pair(int(r.kind), r.id); };
  for (auto& f : dag.filters)
    for (auto& r : f.in)
      if (r.kind != Ref::Mesh) rc[key(r)] += 1;
  rc[key(dag.result)] += 1;
  std::vector<void*> hval(dag.filters.size(), nullptr);  // every result lives in host memory (L92)

  auto host_const = [&](const Filter& f) -> void* {
    void* h = hp.get(sb);
    if (m.dt == DType::F32) std::fill_n(static_cast<float*>(h), N, float(f.cval));
    else std::fill_n(static_cast<double*>(h), N, f.cval);
    return h;
  };
  auto release = [&](const Ref& r) {
    if (r.kind != Ref::Filter) return;
    if (--rc[key(r)] > 0) return;
    if (hval[r.id]) hp.put(hval[r.id]);
    hval[r.id] = nullptr;
  };

  for (size_t k = 0; k < dag.filters.size(); ++k) {
    const Filter& f = dag.filters[k];
    if (f.op == Op::Const) {  // a host buffer, uploaded by every consumer (L307)
      hval[k] = host_const(f);
      continue;
    }
    if (f.op == Op::Decompose) {  // on the host, no transfer (L289)
      const Ref& a = f.in[0];
      void* h = hp.get(sb);
      if (m.dt == DType::F32) {
        const float* v = static_cast<const float*>(hval[a.id]);
        float* o = static_cast<float*>(h);
        for (int64_t e = 0; e < N; ++e) o[e] = v[4 * e + f.k];
      } else {
        const double* v = static_cast<const double*>(hval[a.id]);
        double* o = static_cast<double*>(h);
        for (int64_t e = 0; e < N; ++e) o[e] = v[4 * e + f.k];
      }
      hval[k] = h;
      release(a);
      continue;
    }
    // one kernel: upload every argument, run, download the result (L92)
    std::vector<void*> dfree;
    std::vector<size_t> dsz;
    auto upload = [&](const void* h, size_t bytes) -> void* {
      led.add(bytes);
      void* d = dev_alloc(bytes, m.device, s);
      DFG_CUDA(cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice, s));
      st.h2d_count += 1;
      st.h2d_bytes += int64_t(bytes);
      dfree.push_back(d);
      dsz.push_back(bytes);
      return d;
    };
    auto upload_small = [&](const void* h, size_t bytes) -> void* {
      void* d = dev_alloc(bytes, m.device, s);
      DFG_CUDA(cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice, s));
      st.h2d_count += 1;
      st.h2d_bytes += int64_t(bytes);
      dfree.push_back(d);
      dsz.push_back(0);
      return d;
    };
    std::vector<const void*> args;   // owned-cell value pointers
    const void* grad_base = nullptr; // grad3d: base incl. ghost planes
    int64_t grad_ghost = 0;
    const void* tab[3] = {m.dev_tab[0], m.dev_tab[1], m.dev_tab[2]};
    int mesh_i = 0;
    for (auto& r : f.in) {
      if (r.kind == Ref::Mesh) {
        if (host) {
          if (r.id == 0) {
            int64_t dims[4] = {m.nx, m.ny, m.NZ, m.k0};
            upload_small(dims, sizeof(dims));
          } else {
            tab[r.id - 1] = upload_small(m.host_tab[r.id - 1].data(), m.host_tab[r.id - 1].size());
          }
        }
        ++mesh_i;
        continue;
      }
      if (r.kind == Ref::Input) {
        Binding& b = m.fields[dag.inputs[r.id]];
        const void* base = b.on_device ? b.ptr : upload(b.ptr, m.field_bytes());
        args.push_back(static_cast<const char*>(base) + goff * int64_t(ts));
        if (f.op == Op::Grad3d) {
          grad_base = base;
          grad_ghost = m.ghost;
        }
      } else {
        const Filter& g = dag.filters[r.id];
        size_t bytes = sb * size_t(g.width == 1 ? 1 : 4);
        const void* d = upload(hval[r.id], bytes);
        args.push_back(d);
        if (f.op == Op::Grad3d) {
          grad_base = d;
          grad_ghost = 0;
        }
      }
    }
    const size_t ob = sb * size_t(f.width == 1 ? 1 : 4);
    led.add(ob);
    void* o = dev_alloc(ob, m.device, s);
    dfree.push_back(o);
    dsz.push_back(ob);
    switch (f.op) {
      case Op::Add: case Op::Sub: case Op::Mult: case Op::Div:
      case Op::Gt: case Op::Lt: case Op::Ge: case Op::Le: case Op::Eq: case Op::Ne:
        kern::binary(f.op, m.dt, args[0], args[1], o, N, s);
        break;
      case Op::Neg: case Op::Sqrt: kern::unary(f.op, m.dt, args[0], o, N, s); break;
      case Op::Select: kern::select(m.dt, args[0], args[1], args[2], o, N, s); break;
      case Op::Compose: kern::compose(m.dt, args.data(), int(args.size()), o, N, s); break;
      case Op::Grad3d:
        kern::grad3d(m.dt, grad_base, o, tab[0], tab[1], tab[2], m.nx, m.ny, m.nzl, m.NZ, m.k0, grad_ghost, s);
        break;
      default: fail(DFG_E_INVALID, "internal: unexpected roundtrip op");
    }
    DFG_CUDA(cudaGetLastError());
    st.kernel_count += 1;
    void* h = hp.get(ob);
    DFG_CUDA(cudaMemcpyAsync(h, o, ob, cudaMemcpyDeviceToHost, s));
    st.d2h_count += 1;
    st.d2h_bytes += int64_t(ob);
    DFG_CUDA(cudaStreamSynchronize(s));
    hval[k] = h;
    for (size_t q = 0; q < dfree.size(); ++q) {
      cudaFreeAsync(dfree[q], s);
      led.sub(dsz[q]);
    }
    for (auto& r : f.in) release(r);
  }
  // the sink: host result -> caller's buffer
  const Ref& res = dag.result;
  const size_t rb = sb * size_t(dag.width(res) == 1 ? 1 : 4);
  if (res.kind == Ref::Input) {
    Binding& b = m.fields[dag.inputs[res.id]];
    const char* srcp = static_cast<const char*>(b.ptr) + goff * int64_t(ts);
    DFG_CUDA(cudaMemcpyAsync(out, srcp, rb, cudaMemcpyDefault, s));
  } else if (out_dev) {
    DFG_CUDA(cudaMemcpyAsync(out, hval[res.id], rb, cudaMemcpyHostToDevice, s));
    st.h2d_count += 1;
    st.h2d_bytes += int64_t(rb);
  } else {
    std::memcpy(out, hval[res.id], rb);
  }
  DFG_CUDA(cudaStreamSynchronize(s));
  release(res);
  for (auto& p : hval)
    if (p) hp.put(p);
  st.dev_highwater_bytes = std::max<int64_t>(st.dev_highwater_bytes, int64_t(led.high));
}

}  // namespace dfg
