// libdfg meshes: spacing tables (reading R1), the two-operation quotient check, device pools, NCCL setup.  See runtime.hpp; DESIGN.md sections 5 and 6.
#include "runtime.hpp"

#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <set>

#include "div2.hpp"
#include "driver.hpp"
#include "kernels.hpp"
#include "runtime_detail.hpp"

namespace dfg {
using namespace detail;

// ====================================================================== mesh
namespace detail {

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
  T* yl = nd + n; // low part of 1/d for the two-operation quotient
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
    // yl = RN(1/d - r) = RN(e / d) with the exact remainder e = 1 - r d (div2.hpp);
    // the kernels use it only on axes whose every divisor is certified below
    yl[i] = div2_low_part(d[i], r[i]);
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
    struct Free {
      float*& b;
      unsigned*& u;
      bool armed = true;
      ~Free() {
        if (armed && b) cudaFree(b);
        if (armed && u) cudaFree(u);
      }
    } guard{buf, bad};  // frees both if a CUDA call below throws
    DFG_CUDA(cudaMalloc(&buf, 3 * size_t(m) * sizeof(float)));
    DFG_CUDA(cudaMalloc(&bad, size_t(m) * sizeof(unsigned)));
    DFG_CUDA(cudaMemcpy(buf, qd.data(), m * sizeof(float), cudaMemcpyHostToDevice));
    DFG_CUDA(cudaMemcpy(buf + m, qr.data(), m * sizeof(float), cudaMemcpyHostToDevice));
    DFG_CUDA(cudaMemcpy(buf + 2 * m, ql.data(), m * sizeof(float), cudaMemcpyHostToDevice));
    DFG_CUDA(cudaMemset(bad, 0, size_t(m) * sizeof(unsigned)));
    kern::verify_div2(buf, buf + m, buf + 2 * m, m, bad, nullptr);
    std::vector<unsigned> hb(m);
    cudaError_t e = cudaMemcpy(hb.data(), bad, m * sizeof(unsigned), cudaMemcpyDeviceToHost);
    guard.armed = false;
    cudaFree(buf);
    cudaFree(bad);
    DFG_CUDA(e);
    for (int k = 0; k < m; ++k) g_div2_ok[div2_key(qd[k], ql[k])] = hb[k] == 0;
  }
  for (int64_t i = 0; i < n; ++i)
    if (!g_div2_ok[div2_key(d[i], yl[i])]) return false;
  return true;
}

// fp64 axes: certification by candidates on the host (div2.hpp); 2^52
// significands cannot be enumerated.  Cached per divisor like the fp32 check.
std::map<uint64_t, bool> g_div2_ok64;  // key: d bits (r and yl are functions of d)

bool axis_div2_f64(const std::vector<char>& tab, int64_t n) {
  const double* d = reinterpret_cast<const double*>(tab.data());
  const double* r = d + n;
  const double* yl = d + 3 * n;
  if (n == 1) return true;
  std::lock_guard<std::mutex> lk(g_div2_mu);
  bool all = true;
  for (int64_t i = 0; i < n; ++i) {
    uint64_t b;
    std::memcpy(&b, &d[i], 8);
    auto it = g_div2_ok64.find(b);
    bool ok;
    if (it != g_div2_ok64.end() && yl[i] == div2_low_part(d[i], r[i])) {
      ok = it->second;
    } else {
      ok = certify_div2<double>(d[i], r[i], yl[i]);
      if (yl[i] == div2_low_part(d[i], r[i])) g_div2_ok64[b] = ok;
    }
    all = all && ok;
  }
  return all;
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

}  // namespace detail

MeshImpl::~MeshImpl() {
  int cur = -1;
  cudaGetDevice(&cur);
  cudaSetDevice(device);
  for (auto& p : dev_tab)
    if (p) cudaFree(p);
  for (void* p : ipc_opened) cudaIpcCloseMemHandle(p);
  if (flags) cudaFree(flags);
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
  if (d2 && !std::strcmp(d2, "test-1op"))
    for (int a = 0; a < 3; ++a) {
      if (dt == DType::F32) std::fill_n(reinterpret_cast<float*>(m->host_tab[a].data()) + 3 * N[a], N[a], 0.0f);
      else std::fill_n(reinterpret_cast<double*>(m->host_tab[a].data()) + 3 * N[a], N[a], 0.0);
    }
  for (int a = 0; a < 3; ++a) {
    DFG_CUDA(cudaMalloc(&m->dev_tab[a], m->host_tab[a].size()));
    DFG_CUDA(cudaMemcpy(m->dev_tab[a], m->host_tab[a].data(), m->host_tab[a].size(), cudaMemcpyHostToDevice));
  }
  if (m->markstein_safe && !div2_off)
    for (int a = 0; a < 3; ++a)
      if (dt == DType::F32 ? axis_div2(m->host_tab[a], N[a]) : axis_div2_f64(m->host_tab[a], N[a]))
        m->div2_mask |= 1 << a;
  return m;
}

// ===================================================================== NCCL
namespace detail {

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
}  // namespace detail

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

// ------------------------------------------------------- peer-memory halo
namespace {
struct PeerBlobField {
  char name[48];
  cudaIpcMemHandle_t h;
  int64_t off;
};
struct PeerBlob {
  char magic[8];
  int32_t dtype, nfields;
  int64_t nx, ny, nzl, NZ, k0, ghost;
  cudaIpcMemHandle_t flags_h;
  int64_t flags_off;
  PeerBlobField f[24];
};
static_assert(sizeof(PeerBlob) <= kPeerBlobBytes, "peer blob too large");
const char kMagic[8] = {'d', 'f', 'g', 'p', 'e', 'e', 'r', '1'};

// IPC handle of the cudaMalloc allocation holding p, and p's offset in it
void ipc_export(const void* p, cudaIpcMemHandle_t* h, int64_t* off) {
  CUdeviceptr base = 0;
  size_t size = 0;
  DFG_CU(drv().MemGetAddressRange(&base, &size, reinterpret_cast<CUdeviceptr>(p)));
  cudaError_t e = cudaIpcGetMemHandle(h, reinterpret_cast<void*>(base));
  if (e != cudaSuccess) {
    cudaGetLastError();
    fail(DFG_E_UNSUPPORTED, std::string("cudaIpcGetMemHandle: ") + cudaGetErrorString(e) +
                                " (peer halo needs cudaMalloc-backed device fields)");
  }
  *off = int64_t(reinterpret_cast<CUdeviceptr>(p) - base);
}

// flag words (256 bytes) followed by the probe block dfg_peer_probe reads
void ensure_flags(MeshImpl& m) {
  if (m.flags) return;
  DFG_CUDA(cudaSetDevice(m.device));
  const size_t words = size_t(kern::kProbeRows) * kern::kProbeCols;
  DFG_CUDA(cudaMalloc(&m.flags, kern::kProbeOffset + words * 4));
  DFG_CUDA(cudaMemset(m.flags, 0, kern::kProbeOffset));
  std::vector<uint32_t> pat(words);
  for (size_t i = 0; i < words; ++i) pat[i] = kern::probe_word(uint32_t(i));
  DFG_CUDA(cudaMemcpy(reinterpret_cast<char*>(m.flags) + kern::kProbeOffset, pat.data(), words * 4,
                      cudaMemcpyHostToDevice));
  DFG_CUDA(cudaDeviceSynchronize());
}
}  // namespace

void mesh_peer_export(MeshImpl& m, void* out) {
  if (m.ghost != 1 || m.gxy != 0 || m.ghosts_supplied)
    fail(DFG_E_INVALID, "peer halo: the mesh must be a z-slab with one ghost plane per side (dfg_create_mesh ghost=1)");
  DFG_CUDA(cudaSetDevice(m.device));
  ensure_flags(m);
  PeerBlob b;
  std::memset(&b, 0, sizeof(b));
  std::memcpy(b.magic, kMagic, 8);
  b.dtype = m.dt == DType::F32 ? 0 : 1;
  b.nx = m.nx, b.ny = m.ny, b.nzl = m.nzl, b.NZ = m.NZ, b.k0 = m.k0, b.ghost = m.ghost;
  ipc_export(m.flags, &b.flags_h, &b.flags_off);
  m.exported.clear();
  for (auto& kv : m.fields) {
    if (!kv.second.on_device || !kv.second.ptr) continue;
    if (b.nfields == int32_t(sizeof(b.f) / sizeof(b.f[0]))) fail(DFG_E_UNSUPPORTED, "peer halo: too many bound fields");
    if (kv.first.size() >= sizeof(b.f[0].name)) fail(DFG_E_UNSUPPORTED, "peer halo: field name too long");
    PeerBlobField& f = b.f[b.nfields++];
    std::memcpy(f.name, kv.first.c_str(), kv.first.size());
    ipc_export(kv.second.ptr, &f.h, &f.off);
    m.exported[kv.first] = kv.second.ptr;
  }
  std::memset(out, 0, kPeerBlobBytes);
  std::memcpy(out, &b, sizeof(b));
}

void mesh_link_peers(MeshImpl& m, const void* lo_blob, const void* hi_blob) {
  const bool has_lo = m.k0 > 0, has_hi = m.k0 + m.nzl < m.NZ;
  if (!lo_blob && !hi_blob) {  // unlink: back to the other halo transports
    m.peer_lo.on = m.peer_hi.on = false;
    return;
  }
  if (has_lo != (lo_blob != nullptr) || has_hi != (hi_blob != nullptr))
    fail(DFG_E_INVALID, "peer halo: give the blob of every z neighbour and no other");
  if (m.ghost != 1) fail(DFG_E_INVALID, "peer halo: the mesh needs one ghost plane per side");
  DFG_CUDA(cudaSetDevice(m.device));
  ensure_flags(m);
  std::map<std::string, void*> opened;  // handle bytes -> mapped allocation base
  auto open = [&](const cudaIpcMemHandle_t& h) -> char* {
    std::string key(reinterpret_cast<const char*>(&h), sizeof(h));
    auto it = opened.find(key);
    if (it != opened.end()) return static_cast<char*>(it->second);
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      cudaGetLastError();
      fail(DFG_E_UNSUPPORTED, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
    }
    m.ipc_opened.push_back(p);
    opened[key] = p;
    return static_cast<char*>(p);
  };
  auto link = [&](const void* blob, MeshImpl::Peer& peer, bool below) {
    PeerBlob b;
    std::memcpy(&b, blob, sizeof(b));
    if (std::memcmp(b.magic, kMagic, 8) != 0) fail(DFG_E_INVALID, "peer halo: not a dfg_mesh_peer_export blob");
    if (b.dtype != (m.dt == DType::F32 ? 0 : 1) || b.nx != m.nx || b.ny != m.ny || b.NZ != m.NZ || b.ghost != 1)
      fail(DFG_E_INVALID, "peer halo: neighbour slab has another type, plane size, global depth or ghost width");
    if (below ? b.k0 + b.nzl != m.k0 : m.k0 + m.nzl != b.k0)
      fail(DFG_E_INVALID, "peer halo: blob is not the adjacent z slab");
    peer = MeshImpl::Peer{};
    peer.k0 = b.k0, peer.nzl = b.nzl, peer.ghost = b.ghost;
    peer.flags = reinterpret_cast<uint32_t*>(open(b.flags_h) + b.flags_off);
    for (int i = 0; i < b.nfields && i < int(sizeof(b.f) / sizeof(b.f[0])); ++i) {
      std::string name(b.f[i].name, strnlen(b.f[i].name, sizeof(b.f[i].name)));
      peer.fields[name] = open(b.f[i].h) + b.f[i].off;
    }
    peer.on = true;
  };
  // both sides or neither: a half-linked slab would wait on flags nobody writes
  MeshImpl::Peer lo, hi;
  if (lo_blob) link(lo_blob, lo, true);
  if (hi_blob) link(hi_blob, hi, false);
  m.peer_lo = lo;
  m.peer_hi = hi;
}

// Open the flag allocation of an exported slab on the current device, read
// its probe block with one TMA load (the access the in-place halo makes) and
// compare it with the pattern.  Meant to run in a short-lived process: a
// transport that faults takes down that process, not the caller's.
bool peer_probe(const void* blob) {
  PeerBlob b;
  std::memcpy(&b, blob, sizeof(b));
  if (std::memcmp(b.magic, kMagic, 8) != 0) fail(DFG_E_INVALID, "peer probe: not a dfg_mesh_peer_export blob");
  DFG_CUDA(cudaFree(0));
  void* base = nullptr;
  cudaError_t e = cudaIpcOpenMemHandle(&base, b.flags_h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    cudaGetLastError();
    fail(DFG_E_UNSUPPORTED, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
  }
  struct Close {
    void* p;
    ~Close() { cudaIpcCloseMemHandle(p); }
  } close{base};
  char* probe = static_cast<char*>(base) + b.flags_off + kern::kProbeOffset;
  CUtensorMap map;
  cuuint64_t gdim[2] = {cuuint64_t(kern::kProbeCols), cuuint64_t(kern::kProbeRows)};
  cuuint64_t gstride[1] = {cuuint64_t(kern::kProbeCols) * 4};
  cuuint32_t box[2] = {cuuint32_t(kern::kProbeCols), cuuint32_t(kern::kProbeRows)};
  cuuint32_t estr[2] = {1, 1};
  DFG_CU(drv().TensorMapEncodeTiled(&map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, probe, gdim, gstride, box, estr,
                                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                    CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE));
  const size_t words = size_t(kern::kProbeRows) * kern::kProbeCols;
  uint32_t* out = nullptr;
  DFG_CUDA(cudaMalloc(&out, words * 4));
  struct Free {
    void* p;
    ~Free() { cudaFree(p); }
  } fr{out};
  DFG_CUDA(cudaMemset(out, 0, words * 4));
  kern::tma_probe(&map, out, nullptr);
  DFG_CUDA(cudaGetLastError());
  DFG_CUDA(cudaDeviceSynchronize());
  std::vector<uint32_t> got(words);
  DFG_CUDA(cudaMemcpy(got.data(), out, words * 4, cudaMemcpyDeviceToHost));
  for (size_t i = 0; i < words; ++i)
    if (got[i] != kern::probe_word(uint32_t(i))) return false;
  return true;
}

}  // namespace dfg
