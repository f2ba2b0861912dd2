// libdfg plans: compile, execute, the fused strategy (TMA / general / point-wise launches, multi-block), the halo exchange and the streamed strategy.  See runtime.hpp; DESIGN.md sections 2, 5 and 6.
#include "runtime.hpp"

#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <set>

#include "driver.hpp"
#include "kernels.hpp"
#include "runtime_detail.hpp"

namespace dfg {
using namespace detail;

// ==================================================================== plans
namespace detail {


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


// one pool per plan would pin memory per plan; share per process instead
HostPool& host_pool() {
  static HostPool* pool = new HostPool();  // leaked on purpose: outlives plans at exit
  return *pool;
}
std::mutex g_host_mu;  // guards host_pool()

}  // namespace detail

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
  if (gexec) cudaGraphExecDestroy(gexec);
  if (sCap) cudaStreamDestroy(sCap);
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
    if (!prog || ref == 0) fail(DFG_E_INVALID, "reference kernels exist for \"velmag\", \"vortmag\" and \"qcrit\"");
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
    if (cfg.div_mode == 1 && !markstein_only) cfg.div2 = mesh->div2_mask;
    // scale folding is exact in the normal range only; "ieee" keeps every op
    const char* fold = std::getenv("DFG_SCALE_FOLD");
    cfg.fold = cfg.div_mode != 0 && !(fold && !std::strcmp(fold, "0"));
    const char* ncw = std::getenv("DFG_NCW");
    if (ncw) cfg.ncw = std::max(1, std::min(30, std::atoi(ncw)));
    const char* ctas = std::getenv("DFG_CTAS");
    if (ctas) cfg.ctas = std::max(1, std::min(4, std::atoi(ctas)));
    const char* st = std::getenv("DFG_STAGES");
    // >= 3: the cp.async tile ring waits on stage n+1 before it fills stage n+2
    if (st) cfg.stages = std::max(3, std::min(16, std::atoi(st)));
    // tile shape for this mesh (narrow meshes: several rows per warp)
    const char* rpw = std::getenv("DFG_RPW");
    const int64_t slots = int64_t(sm_count(mesh->device)) * cfg.ctas;
    if (rpw) {
      const int r = std::atoi(rpw);
      cfg.rpw = (r == 2 || r == 4) ? r : 1;
    } else if (ncw) {
      cfg.rpw = choose_rpw(mesh->dt, mesh->nx, mesh->ny, mesh->nzl, cfg.ncw, slots);
    } else {
      // layouts a tensor map cannot take run the row-class kernel (fused_tma.cuh
      // "rows"; DFG_FUSED_KERNEL=rows forces it where the maps could run)
      const int64_t vec = int64_t(16 / dsize(mesh->dt));
      const char* fk = std::getenv("DFG_FUSED_KERNEL");
      const bool force_rows = fk && !std::strcmp(fk, "rows");
      if (mesh->nx % vec == 0 && mesh->px() % vec == 0 && mesh->gx() % vec == 0 && !force_rows)
        choose_tile(mesh->dt, mesh->nx, mesh->ny, mesh->nzl, slots, &cfg.ncw, &cfg.rpw);
      else
        choose_rows_tile(mesh->dt, mesh->nx, mesh->ny, mesh->nzl, slots, &cfg.ncw, &cfg.rpw);
    }
    // axis degeneracy (n == 1) is a property of the GLOBAL mesh
    plan->fsrc = generate_fused(dag, mesh->NX, mesh->NY, mesh->NZ, cfg, ref);
    static const std::string kUnit = "dfg_fused.cu";
    const Cubin& cb = nvrtc_compile(plan->fsrc.source, kUnit);  // cached for the process lifetime
    plan->regs = cb.regs;
    plan->spill = cb.spill;
    // the runtime API owns the primary context; make it current for the driver API
    DFG_CUDA(cudaFree(0));
    plan->mod = load_module(cb, !plan->fsrc.layout.stencil_inputs.empty(), plan->fsrc.cfg.has_tma,
                            plan->fsrc.cfg.rstages >= 2);
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
                                         plan->fsrc.cfg.stages, plan->fsrc.cfg.rpw);
      DFG_CU(drv().FuncSetAttribute(plan->mod.tma, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(smem)));
      DFG_CU(drv().FuncSetAttribute(plan->mod.tma_multi, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(smem)));
      DFG_CU(drv().FuncSetAttribute(plan->mod.tile, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(smem)));
      DFG_CU(drv().FuncSetAttribute(plan->mod.tile_multi, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(smem)));
      const FusedConfig& c = plan->fsrc.cfg;
      const size_t rsmem = fused_rows_smem_bytes(mesh->dt, int(plan->fsrc.layout.stencil_inputs.size() +
                                                               plan->fsrc.layout.point_inputs.size()),
                                                 c.ncw, c.rpw, c.rstages);
      if (plan->mod.rows && rsmem <= 227 * 1024) {
        DFG_CU(drv().FuncSetAttribute(plan->mod.rows, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(rsmem)));
        DFG_CU(drv().FuncSetAttribute(plan->mod.rows_multi, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, int(rsmem)));
        plan->rows_smem = rsmem;
      }
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

std::pair<cudaEvent_t, cudaEvent_t> PlanImpl::kernel_begin(cudaStream_t s) {
  if (timing < 2) return {nullptr, nullptr};
  auto e = kernel_events();
  DFG_CUDA(cudaEventRecord(e.first, s));
  return e;
}

void PlanImpl::kernel_end(const std::pair<cudaEvent_t, cudaEvent_t>& e, cudaStream_t s) {
  if (e.second) DFG_CUDA(cudaEventRecord(e.second, s));
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
  NvtxRange nv(m.nccl ? "dfg halo nccl" : "dfg halo copies");
  const size_t ts = dsize(m.dt);
  const size_t pb = size_t(m.plane()) * ts;
  auto lo = m.link_lo.lock(), hi = m.link_hi.lock();
  if (m.nccl) {
    last_halo = 1;
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
    last_halo = 2;
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
  static const char* const kStrat[] = {"dfg_execute roundtrip", "dfg_execute staged", "dfg_execute fused",
                                      "dfg_execute streamed", "dfg_execute reference", "dfg_execute hybrid"};
  NvtxRange nv(kStrat[strategy]);
  if (timing >= 1) DFG_CUDA(cudaEventRecord(ev0, s));
  switch (strategy) {
    case DFG_FUSED: exec_fused(out, out_dev, s); break;
    case DFG_STREAMED: exec_streamed(out, out_dev, s); break;
    case DFG_REFERENCE: exec_fused(out, out_dev, s); break;
    case DFG_STAGED: {
      const char* g = std::getenv("DFG_GRAPH");
      bool device = out_dev;
      for (int i : sources(dag).inputs) device = device && m.fields[dag.inputs[i]].on_device;
      if (device && !(g && !std::strcmp(g, "0"))) exec_staged_graph(out, s);
      else exec_staged(out, out_dev, s);
      break;
    }
    case DFG_HYBRID: exec_hybrid(out, out_dev, s); break;
    case DFG_ROUNDTRIP: exec_roundtrip(out, out_dev, s); break;
  }
  if (timing >= 1) DFG_CUDA(cudaEventRecord(ev1, s));
  DFG_CUDA(cudaGetLastError());
  timed = timing >= 1;
  st.executes += 1;
  bool any_host = !out_dev;
  for (int i : sources(dag).inputs)
    if (!m.fields[dag.inputs[i]].on_device) any_host = true;
  // any host buffer makes the call synchronous (dfg.h): the uploads have read
  // the caller's inputs and the result is in place when dfg_execute returns
  if (any_host) DFG_CUDA(cudaStreamSynchronize(s));
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
void encode_map(CUtensorMap* map, const SlabView& m, void* base, int ncw, int rpw) {
  const size_t ts = dsize(m.dt);
  const int vec = int(16 / ts);
  cuuint64_t gdim[3] = {cuuint64_t(m.px()), cuuint64_t(m.py()), cuuint64_t(m.nzl + 2 * m.ghost)};
  cuuint64_t gstride[2] = {cuuint64_t(m.px()) * ts, cuuint64_t(m.px() * m.py()) * ts};
  cuuint32_t box[3] = {cuuint32_t(tma_tile_w(m.dt, rpw) + 2 * vec), cuuint32_t(tma_tile_h(ncw, rpw) + 2), 1};
  cuuint32_t estr[3] = {1, 1, 1};
  DFG_CU(drv().TensorMapEncodeTiled(map, m.dt == DType::F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64,
                                3, base, gdim, gstride, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE));
}

// Host image of DfgTmaParams (fused_tma.cuh): map[NF_] | map_lo[NSF_] |
// map_hi[NSF_] | DfgPeerInfo (64 B) | DfgParams, each map 128 B (64-aligned),
// total padded to 64 bytes.
struct TmaBlobLayout {
  size_t lo, hi, peer, params, size;
};
TmaBlobLayout tma_blob_layout(int nf, int nsf, size_t param_words) {
  const size_t NF = size_t(std::max(nf, 1)), NSF = size_t(std::max(nsf, 1));
  TmaBlobLayout b;
  b.lo = 128 * NF;
  b.hi = b.lo + 128 * NSF;
  b.peer = b.hi + 128 * NSF;
  b.params = b.peer + 64;
  b.size = (b.params + param_words * 8 + 63) / 64 * 64;
  return b;
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
// Row period P of the 16-byte residues of the row offsets y * px * sizeof(T)
// (fused_tma.cuh "rows"): 1, 2 or 4.
int row_period(const SlabView& m) {
  const int64_t rb = m.px() * int64_t(dsize(m.dt));
  int P = 1;
  while ((rb * P) % 16 != 0) P *= 2;
  return P;
}

// Host image of DfgRowsParams (fused_tma.cuh): map[NF_ * 4] (128 B each; map
// f * 4 + c = row class c of field f) | DfgRowsInfo {P, BR, o[4]} + pad to
// 64 B | DfgParams.  Class c of a field: the rows y = c (mod P) as a 3-D
// tensor from base + (c px T) rounded down to 16 bytes (o_c elements before
// the row's first element), dims {px + o_c, rows of the class, planes},
// strides {P px T, px py T} (both multiples of 16), box {TX + 2 VEC, BR, 2} (two planes).
std::vector<unsigned char> rows_blob(const std::vector<const void*>& fptr, int nf_, const SlabView& m, int ncw,
                                     int rpw, const std::vector<uint64_t>& words, PlanImpl::MapCache* cache) {
  const size_t ts = dsize(m.dt);
  const int vec = int(16 / ts);
  const int P = row_period(m);
  const int rows = tma_tile_h(ncw, rpw) + 2, BR = (rows + P - 1) / P;
  const size_t maps = size_t(128) * size_t(std::max(nf_, 1)) * 4;
  std::vector<unsigned char> blob((maps + 64 + words.size() * 8 + 63) / 64 * 64, 0);
  int32_t info[7] = {P, BR, 0, 0, 0, 0, P == 1 ? 0 : P == 2 ? 1 : 2};
  for (int c = 0; c < P; ++c) info[2 + c] = int32_t((int64_t(c) * m.px() * int64_t(ts)) % 16 / int64_t(ts));
  const int64_t mk[4] = {m.px(), m.py(), m.nzl, int64_t(m.ghost)};
  const bool cached = cache && cache->hit(fptr, mk) && cache->maps.size() == maps;
  for (size_t f = 0; f < fptr.size() && !cached; ++f) {
    for (int c = 0; c < P; ++c) {
      const int64_t off = int64_t(c) * m.px() * int64_t(ts);
      const int o = info[2 + c];
      char* base = static_cast<char*>(const_cast<void*>(fptr[f])) + (off - o * int64_t(ts));
      cuuint64_t gdim[3] = {cuuint64_t(m.px() + o), cuuint64_t((m.py() - c + P - 1) / P),
                            cuuint64_t(m.nzl + 2 * m.ghost)};
      cuuint64_t gstride[2] = {cuuint64_t(P) * cuuint64_t(m.px()) * ts, cuuint64_t(m.px() * m.py()) * ts};
      cuuint32_t box[3] = {cuuint32_t(tma_tile_w(m.dt, rpw) + 2 * vec), cuuint32_t(BR), 2};  // two planes
      cuuint32_t estr[3] = {1, 1, 1};
      DFG_CU(drv().TensorMapEncodeTiled(reinterpret_cast<CUtensorMap*>(blob.data() + 128 * (f * 4 + size_t(c))),
                                        m.dt == DType::F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                                           : CU_TENSOR_MAP_DATA_TYPE_FLOAT64,
                                        3, base, gdim, gstride, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE));
    }
  }
  if (cached) {
    std::memcpy(blob.data(), cache->maps.data(), maps);
  } else if (cache) {
    cache->maps.assign(blob.begin(), blob.begin() + std::ptrdiff_t(maps));
    cache->ptrs = fptr;
    std::copy(mk, mk + 4, cache->key);
  }
  std::memcpy(blob.data() + maps, info, sizeof(info));
  std::memcpy(blob.data() + maps + 64, words.data(), words.size() * 8);
  return blob;
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
  // peer-memory halo (dfg_mesh_link_peers): no exchange, the kernel reads the
  // neighbours' planes in place once their "ready" flag shows this step
  const bool peer = halo && (need_lo ? m.peer_lo.on : true) && (need_hi ? m.peer_hi.on : true);
  const bool overlap = halo && !peer && m.nzl >= 3 && !(ov && !std::strcmp(ov, "0"));
  if (peer) {
    led.add(size_t(N) * size_t(L.outw) * ts);
    exec_fused_peer(fptr, out, out_dev, s);
    st.dev_highwater_bytes = std::max<int64_t>(st.dev_highwater_bytes, int64_t(led.high));
    return;
  }
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
bool PlanImpl::tma_ok(const std::vector<const void*>& fptr, const void* dout, const SlabView& m) const {
  const int vec = int(16 / dsize(m.dt));
  const char* force = std::getenv("DFG_FUSED_KERNEL");
  if (force && (!std::strcmp(force, "general") || !std::strcmp(force, "tile") || !std::strcmp(force, "rows")))
    return false;
  return mod.tma && !fsrc.layout.stencil_inputs.empty() && m.nx % vec == 0 && m.px() % vec == 0 &&
         m.gx() % vec == 0 && aligned16(dout) &&
         std::all_of(fptr.begin(), fptr.end(), [](const void* p) { return aligned16(p); });
}

bool PlanImpl::rows_ok(const std::vector<const void*>& fptr, const SlabView& m) {
  const char* force = std::getenv("DFG_FUSED_KERNEL");
  if (force && (!std::strcmp(force, "general") || !std::strcmp(force, "tile"))) return false;
  // a class of rows needs at least one row per plane (py >= P)
  const bool layout = !fsrc.layout.stencil_inputs.empty() && fsrc.cfg.has_tma &&
                      (m.px() * m.py() * int64_t(dsize(m.dt))) % 16 == 0 && m.px() * m.py() < (int64_t(1) << 32) &&
                      m.px() < (int64_t(1) << 30) && m.py() >= row_period(m) &&
                      std::all_of(fptr.begin(), fptr.end(), [](const void* p) { return aligned16(p); });
  return layout && mod.rows && rows_smem != 0;
}

// Fused execute of a z-slab linked to its neighbours through peer memory.
// Per step e (the mesh's execute count, equal on every rank):
//   write own ready = e           (release: this rank's fields are final)
//   interior planes               (own planes only)
//   wait ready(lo), ready(hi) >= e
//   boundary planes               (TMA reads the neighbours' planes in place)
//   write lo.hi_done = e, hi.lo_done = e   (done reading their planes)
//   wait own lo_done, hi_done >= e (the caller may overwrite its fields after)
// The waits are stream memory operations (no SM spins).  Layouts the TMA
// kernel cannot take copy the neighbours' planes into the ghost planes
// (device-to-device through the mappings) and run one launch.
void PlanImpl::exec_fused_peer(const std::vector<const void*>& fptr, void* out, bool out_dev, cudaStream_t s) {
  MeshImpl& m = *mesh;
  if (!out_dev) fail(DFG_E_UNSUPPORTED, "peer halo: the output must be a device buffer");
  for (auto& kv : m.exported) {
    auto it = m.fields.find(kv.first);
    if (it == m.fields.end() || it->second.ptr != kv.second)
      fail(DFG_E_INVALID, "peer halo: field '" + kv.first + "' was rebound after dfg_mesh_peer_export");
  }
  const FusedLayout& L = fsrc.layout;
  for (int in : L.stencil_inputs)
    if (!m.exported.count(dag.inputs[size_t(in)]))
      fail(DFG_E_INVALID, "peer halo: field '" + dag.inputs[size_t(in)] + "' was bound after dfg_mesh_peer_export");
  const bool lo = m.k0 > 0, hi = m.k0 + m.nzl < m.NZ;
  const SlabView v = SlabView::of(m);
  // every check that can fail runs before this rank publishes "ready": a
  // throw after it would leave the neighbours waiting for the done flags.
  // In-place TMA reads need the neighbours' mapped fields 16-byte aligned too
  // (their tensor maps), else the planes are copied into the ghost planes.
  bool use_tma = tma_ok(fptr, out, v);
  for (const MeshImpl::Peer* pr : {lo ? &m.peer_lo : nullptr, hi ? &m.peer_hi : nullptr}) {
    if (!pr) continue;
    for (int in : L.stencil_inputs) {
      auto it = pr->fields.find(dag.inputs[size_t(in)]);
      if (it == pr->fields.end() || !it->second)
        fail(DFG_E_UNBOUND, "peer slab exported no field '" + dag.inputs[size_t(in)] + "'");
      use_tma = use_tma && aligned16(it->second);
    }
  }
  NvtxRange nv("dfg halo peer (in-place reads)");
  const uint32_t e = ++m.epoch;
  auto dptr = [](const uint32_t* p, int w) { return reinterpret_cast<CUdeviceptr>(p + w); };
  const CUstream cs = reinterpret_cast<CUstream>(s);
  DFG_CU(drv().StreamWriteValue32(cs, dptr(m.flags, kFlagReady), e, CU_STREAM_WRITE_VALUE_DEFAULT));
  const void* tab[3] = {m.dev_tab[0], m.dev_tab[1], m.dev_tab[2]};
  auto wait_ready = [&] {
    if (lo) DFG_CU(drv().StreamWaitValue32(cs, dptr(m.peer_lo.flags, kFlagReady), e, CU_STREAM_WAIT_VALUE_GEQ));
    if (hi) DFG_CU(drv().StreamWaitValue32(cs, dptr(m.peer_hi.flags, kFlagReady), e, CU_STREAM_WAIT_VALUE_GEQ));
  };
  const char* ik = std::getenv("DFG_PEER_INKERNEL");
  if (use_tma && !(ik && !std::strcmp(ik, "0"))) {
    // ONE launch: the producers wait in the kernel for the neighbours'
    // "ready" flags before loading their planes, and the z-chunks at the slab
    // ends run last, so the interior overlaps the wait (no stream waits, no
    // extra launches)
    peer_wait_epoch = e;
    try {
      launch_fused(fptr, out, tab, v, s, m.k0, m.k0 + m.nzl, true);
    } catch (...) {
      peer_wait_epoch = 0;
      throw;
    }
    peer_wait_epoch = 0;
  } else if (use_tma) {
    const int64_t a = m.k0 + (lo ? 1 : 0), b = m.k0 + m.nzl - (hi ? 1 : 0);
    if (a < b) launch_fused(fptr, out, tab, v, s, a, b);
    wait_ready();
    if (a >= b) {
      launch_fused(fptr, out, tab, v, s, m.k0, m.k0 + m.nzl, true);
    } else {
      if (lo) launch_fused(fptr, out, tab, v, s, m.k0, m.k0 + 1, true);
      if (hi) launch_fused(fptr, out, tab, v, s, b, b + 1, true);
    }
  } else {
    wait_ready();
    const size_t pb = size_t(m.plane()) * dsize(m.dt);
    for (int in : L.stencil_inputs) {
      const std::string& name = dag.inputs[size_t(in)];
      char* base = static_cast<char*>(m.fields[name].ptr);
      if (lo) {
        const char* src = static_cast<const char*>(m.peer_lo.fields.at(name)) + size_t(m.peer_lo.nzl) * pb;
        DFG_CUDA(cudaMemcpyAsync(base, src, pb, cudaMemcpyDeviceToDevice, s));
      }
      if (hi) {
        const char* src = static_cast<const char*>(m.peer_hi.fields.at(name)) + size_t(m.peer_hi.ghost) * pb;
        DFG_CUDA(cudaMemcpyAsync(base + size_t(m.nzl + 1) * pb, src, pb, cudaMemcpyDeviceToDevice, s));
      }
    }
    launch_fused(fptr, out, tab, v, s);
  }
  if (lo) DFG_CU(drv().StreamWriteValue32(cs, dptr(m.peer_lo.flags, kFlagHiDone), e, CU_STREAM_WRITE_VALUE_DEFAULT));
  if (hi) DFG_CU(drv().StreamWriteValue32(cs, dptr(m.peer_hi.flags, kFlagLoDone), e, CU_STREAM_WRITE_VALUE_DEFAULT));
  if (lo) DFG_CU(drv().StreamWaitValue32(cs, dptr(m.flags, kFlagLoDone), e, CU_STREAM_WAIT_VALUE_GEQ));
  if (hi) DFG_CU(drv().StreamWaitValue32(cs, dptr(m.flags, kFlagHiDone), e, CU_STREAM_WAIT_VALUE_GEQ));
  last_halo = use_tma ? 3 : 4;
  st.halo_bytes += int64_t(L.stencil_inputs.size()) * ((lo ? 1 : 0) + (hi ? 1 : 0)) * int64_t(m.plane()) *
                        int64_t(dsize(m.dt));
}

void PlanImpl::launch_fused(const std::vector<const void*>& fptr, void* dout, const void* const tab[3],
                            const SlabView& m, cudaStream_t s, int64_t kb, int64_t ke, bool peer) {
  const size_t ts = dsize(m.dt);
  const FusedLayout& L = fsrc.layout;
  const int64_t kbeg = kb < 0 ? m.k0 : kb, kend = ke < 0 ? m.k0 + m.nzl : ke;
  NvtxRange nv(kb < 0 && ke < 0 ? "dfg fused launch" : peer ? "dfg fused boundary planes (peer)" : "dfg fused planes");
  const int64_t N = m.nx * m.ny * (kend - kbeg);
  const int vec = int(16 / ts);
  // 16-byte point-wise loads / stores: aligned bases, whole vectors, and the
  // input / output offsets of plane kbeg (ghost planes shift the input) on
  // vector boundaries
  const int64_t in_off = (kbeg - m.k0 + m.ghost) * m.nx * m.ny, out_off = (kbeg - m.k0) * m.nx * m.ny;
  bool vec_ok = aligned16(dout) && (N % vec == 0) && m.gxy == 0 && m.px() == m.nx && m.gx() == 0 &&
                in_off % vec == 0 && out_off % vec == 0;
  for (auto p : fptr) vec_ok = vec_ok && aligned16(p);
  const char* force = std::getenv("DFG_FUSED_KERNEL");
  const bool want_general = force && !std::strcmp(force, "general");
  const int sms = sm_count(mesh->device);

  if (L.stencil_inputs.empty()) {
    auto w = pack_params(fptr, dout, tab[0], tab[1], tab[2], m, kbeg, kend, 0, 0, 0, 0, vec_ok ? 1 : 0);
    void* args[] = {w.data()};
    long long work = vec_ok ? N / vec : N;
    unsigned grid = unsigned(std::max<long long>(1, std::min<long long>((work + 255) / 256, sms * 8LL)));
    auto ke = kernel_begin(s);
    DFG_CU(drv().LaunchKernel(mod.pointwise, grid, 1, 1, 256, 1, 1, 0, s, args, nullptr));
    kernel_end(ke, s);
    last_variant = 3;
  } else if (tma_ok(fptr, dout, m)) {
    const int ncw = fsrc.cfg.ncw, rpw = fsrc.cfg.rpw;
    const int nsf = int(L.stencil_inputs.size() + L.point_inputs.size());  // TMA tiles per stage
    const int tw = tma_tile_w(m.dt, rpw), th = tma_tile_h(ncw, rpw);
    const int tiles_x = int((m.nx + tw - 1) / tw);
    const int tiles_y = int((m.ny + th - 1) / th);
    const int64_t range = kend - kbeg;
    size_t smem = fused_tma_smem_bytes(m.dt, nsf, ncw, fsrc.cfg.stages, rpw);
    int occ = 1;
    DFG_CU(drv().OccupancyMaxActiveBlocksPerMultiprocessor(&occ, mod.tma, (ncw + 1) * 32, smem));
    occ = std::max(occ, 1);
    const int64_t slots = int64_t(sms) * occ;
    // z-chunk length: balance whole rounds of items over the persistent CTAs
    // against the two extra (z-halo) planes each chunk loads.
    int64_t best_kz = range;
    const char* kzenv = std::getenv("DFG_KZ");
    if (kzenv) {
      best_kz = std::max<int64_t>(1, std::min<int64_t>(range, std::atoll(kzenv)));
    } else {
      best_kz = choose_kz(int64_t(tiles_x) * tiles_y, range, slots);
    }
    const int64_t items = int64_t(tiles_x) * tiles_y * ((range + best_kz - 1) / best_kz);
    const unsigned grid = unsigned(std::min<int64_t>(items, slots));
    // parameter blob: DfgTmap map[NSF_] (128 B each, 64-aligned) then DfgParams
    auto w = pack_params(fptr, dout, tab[0], tab[1], tab[2], m, kbeg, kend, items, tiles_x, tiles_y, int(best_kz),
                         vec_ok ? 1 : 0);
    const int nst = int(L.stencil_inputs.size());
    const TmaBlobLayout bl = tma_blob_layout(nsf, nst, w.size());
    alignas(64) unsigned char blob[4096];
    if (bl.size > sizeof(blob)) fail(DFG_E_UNSUPPORTED, "too many fields for the TMA kernel's parameters");
    std::memset(blob, 0, sizeof(blob));
    const int64_t mk[4] = {m.px(), m.py(), m.nzl, int64_t(m.ghost)};
    if (!tma_maps.hit(fptr, mk)) {
      tma_maps.maps.assign(size_t(128) * size_t(nsf), 0);
      for (int f = 0; f < nsf; ++f)
        encode_map(reinterpret_cast<CUtensorMap*>(tma_maps.maps.data() + 128 * f), m, const_cast<void*>(fptr[f]), ncw,
                   rpw);
      tma_maps.ptrs = fptr;
      std::copy(mk, mk + 4, tma_maps.key);
    }
    std::memcpy(blob, tma_maps.maps.data(), tma_maps.maps.size());
    if (peer) {
      // DfgPeerInfo: lo_k0, lo_ghost, hi_k0, hi_ghost | lo_on, hi_on, wait,
      // epoch | lo_ready, hi_ready
      int64_t info[4] = {0, 0, 0, 0};
      int32_t on[4] = {0, 0, peer_wait_epoch ? 1 : 0, int32_t(peer_wait_epoch)};
      const uint32_t* ready[2] = {nullptr, nullptr};
      const MeshImpl::Peer* sides[2] = {&mesh->peer_lo, &mesh->peer_hi};
      for (int sd = 0; sd < 2; ++sd) {
        const MeshImpl::Peer& pr = *sides[sd];
        if (!pr.on) continue;
        SlabView pv = m;
        pv.nzl = pr.nzl;
        pv.k0 = pr.k0;
        pv.ghost = int(pr.ghost);
        for (int f = 0; f < nst; ++f) {
          const std::string& name = dag.inputs[size_t(L.stencil_inputs[size_t(f)])];
          auto it = pr.fields.find(name);
          if (it == pr.fields.end()) fail(DFG_E_UNBOUND, "peer slab exported no field '" + name + "'");
          encode_map(reinterpret_cast<CUtensorMap*>(blob + (sd == 0 ? bl.lo : bl.hi) + 128 * f), pv, it->second, ncw,
                     rpw);
        }
        info[2 * sd] = pr.k0;
        info[2 * sd + 1] = pr.ghost;
        on[sd] = 1;
        ready[sd] = pr.flags + kFlagReady;
      }
      std::memcpy(blob + bl.peer, info, sizeof(info));
      std::memcpy(blob + bl.peer + sizeof(info), on, sizeof(on));
      std::memcpy(blob + bl.peer + sizeof(info) + sizeof(on), ready, sizeof(ready));
    }
    std::memcpy(blob + bl.params, w.data(), w.size() * 8);
    void* args[] = {blob};
    auto ke = kernel_begin(s);
    DFG_CU(drv().LaunchKernel(mod.tma, grid, 1, 1, (ncw + 1) * 32, 1, 1, unsigned(smem), s, args, nullptr));
    kernel_end(ke, s);
    last_variant = 1;
    last_kz = best_kz;
  } else if (rows_ok(fptr, m)) {
    // TMA row-class boxes, read in place by strided-cell consumers (+ the
    // producer and the x-end fixup warp)
    const int ncw = fsrc.cfg.ncw, rpw = fsrc.cfg.rpw, threads = (ncw + 2) * 32;
    const int tw = tma_tile_w(m.dt, rpw), th = tma_tile_h(ncw, rpw);
    const int tiles_x = int((m.nx + tw - 1) / tw);
    const int tiles_y = int((m.ny + th - 1) / th);
    const int64_t range = kend - kbeg;
    int occ = 1;
    DFG_CU(drv().OccupancyMaxActiveBlocksPerMultiprocessor(&occ, mod.rows, threads, rows_smem));
    const int64_t slots = int64_t(sms) * std::max(occ, 1);
    const char* kzenv = std::getenv("DFG_KZ");
    const int64_t kz = kzenv ? std::max<int64_t>(1, std::min<int64_t>(range, std::atoll(kzenv)))
                             : choose_kz(int64_t(tiles_x) * tiles_y, range, slots);
    const int64_t items = int64_t(tiles_x) * tiles_y * ((range + kz - 1) / kz);
    const unsigned grid = unsigned(std::min<int64_t>(items, slots));
    const bool out16 = aligned16(dout) && m.nx % vec == 0;
    auto w = pack_params(fptr, dout, tab[0], tab[1], tab[2], m, kbeg, kend, items, tiles_x, tiles_y, int(kz),
                         out16 ? 1 : 0);
    auto blob = rows_blob(fptr, int(L.stencil_inputs.size() + L.point_inputs.size()), m, ncw, rpw, w, &rows_maps);
    if (blob.size() > 32000) fail(DFG_E_UNSUPPORTED, "too many fields for the row-class kernel's parameters");
    void* args[] = {blob.data()};
    auto ke = kernel_begin(s);
    DFG_CU(drv().LaunchKernel(mod.rows, grid, 1, 1, threads, 1, 1, unsigned(rows_smem), s, args, nullptr));
    kernel_end(ke, s);
    last_variant = 7;
    last_kz = kz;
  } else if (mod.tile && !want_general && m.px() * m.py() < (int64_t(1) << 32)) {
    // same ring and consumers, filled by the consumer threads with cp.async
    const int ncw = fsrc.cfg.ncw, rpw = fsrc.cfg.rpw;
    const int nsf = int(L.stencil_inputs.size() + L.point_inputs.size());
    const int tw = tma_tile_w(m.dt, rpw), th = tma_tile_h(ncw, rpw);
    const int tiles_x = int((m.nx + tw - 1) / tw);
    const int tiles_y = int((m.ny + th - 1) / th);
    const int64_t range = kend - kbeg;
    size_t smem = fused_tma_smem_bytes(m.dt, nsf, ncw, fsrc.cfg.stages, rpw);
    int occ = 1;
    DFG_CU(drv().OccupancyMaxActiveBlocksPerMultiprocessor(&occ, mod.tile, ncw * 32, smem));
    const int64_t slots = int64_t(sms) * std::max(occ, 1);
    const char* kzenv = std::getenv("DFG_KZ");
    const int64_t kz = kzenv ? std::max<int64_t>(1, std::min<int64_t>(range, std::atoll(kzenv)))
                             : choose_kz(int64_t(tiles_x) * tiles_y, range, slots);
    const int64_t items = int64_t(tiles_x) * tiles_y * ((range + kz - 1) / kz);
    const unsigned grid = unsigned(std::min<int64_t>(items, slots));
    // 16-byte output stores need aligned rows (the inputs may be anything)
    const bool out16 = aligned16(dout) && m.nx % vec == 0;
    auto w = pack_params(fptr, dout, tab[0], tab[1], tab[2], m, kbeg, kend, items, tiles_x, tiles_y, int(kz),
                         out16 ? 1 : 0);
    void* args[] = {w.data()};
    auto ke = kernel_begin(s);
    DFG_CU(drv().LaunchKernel(mod.tile, grid, 1, 1, ncw * 32, 1, 1, unsigned(smem), s, args, nullptr));
    kernel_end(ke, s);
    last_variant = 5;
    last_kz = kz;
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
    auto ke = kernel_begin(s);
    DFG_CU(drv().LaunchKernel(mod.general, grid, 1, 1, 256, 1, 1, 0, s, args, nullptr));
    kernel_end(ke, s);
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
  // one launch when every block runs the same module on this device: the TMA
  // kernel if every block's layout suits tensor maps, else the cp.async ring
  bool batch = plans.size() > 1 && p0.strategy == DFG_FUSED && p0.mod.tma_multi && p0.mod.tile_multi &&
               p0.fsrc.cfg.has_tma && !(force && !std::strcmp(force, "general"));
  bool tma = !(force && (!std::strcmp(force, "tile") || !std::strcmp(force, "rows")));
  std::vector<std::vector<const void*>> fptrs(plans.size());
  for (size_t b = 0; b < plans.size() && batch; ++b) {
    PlanImpl& p = *plans[b];
    const MeshImpl& m = *p.mesh;
    const bool halo = (m.k0 > 0 || m.k0 + m.nzl < m.NZ) && !m.ghosts_supplied;
    batch = p.strategy == DFG_FUSED && p.fsrc.source == p0.fsrc.source && m.device == m0.device && !halo &&
            m.px() * m.py() < (int64_t(1) << 32);
    tma = tma && m.nx % vec == 0 && m.px() % vec == 0 && m.gx() % vec == 0 && aligned16(outs[b]);
    std::vector<int> ins = L.stencil_inputs;
    ins.insert(ins.end(), L.point_inputs.begin(), L.point_inputs.end());
    for (int i : ins) {
      auto it = m.fields.find(p.dag.inputs[size_t(i)]);
      if (it == m.fields.end() || !it->second.ptr) fail(DFG_E_UNBOUND, "input '" + p.dag.inputs[size_t(i)] + "' is not bound");
      batch = batch && it->second.on_device;
      tma = tma && aligned16(it->second.ptr);
      fptrs[b].push_back(it->second.ptr);
    }
  }
  if (!batch) {
    for (size_t b = 0; b < plans.size(); ++b) plans[b]->execute(outs[b], true, s);
    return;
  }
  // layouts a tensor map cannot describe: the row-copy ring when every block
  // meets its alignment preconditions, else the cp.async ring
  DFG_CUDA(cudaSetDevice(m0.device));
  bool rows = !tma;
  for (size_t b = 0; b < plans.size() && rows; ++b) rows = plans[b]->rows_ok(fptrs[b], SlabView::of(*plans[b]->mesh));
  rows = rows && p0.rows_smem;
  const FusedConfig& kc = p0.fsrc.cfg;
  const int ncw = kc.ncw, rpw = kc.rpw;
  const int tw = tma_tile_w(m0.dt, rpw), th = tma_tile_h(ncw, rpw);
  const int nsf = int(L.stencil_inputs.size() + L.point_inputs.size());
  const size_t smem = rows ? p0.rows_smem : fused_tma_smem_bytes(m0.dt, nsf, ncw, kc.stages, rpw);
  CUfunction fn = tma ? p0.mod.tma_multi : rows ? p0.mod.rows_multi : p0.mod.tile_multi;
  const int threads = rows ? (ncw + 2) * 32 : tma ? (ncw + 1) * 32 : ncw * 32;
  int occ = 1;
  DFG_CU(drv().OccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem));
  const int64_t slots = int64_t(sm_count(m0.device)) * std::max(occ, 1);
  // one z-chunk length for the batch: whole rounds of the concatenated items
  // against the two halo planes per chunk (as launch_fused)
  int64_t max_range = 1;
  for (auto* p : plans) max_range = std::max(max_range, p->mesh->nzl);
  auto items_for = [&](int64_t kz) {
    int64_t t = 0;
    for (auto* p : plans) {
      const MeshImpl& m = *p->mesh;
      t += int64_t((m.nx + tw - 1) / tw) * ((m.ny + th - 1) / th) * ((m.nzl + kz - 1) / kz);
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
    const int tx = int((m.nx + tw - 1) / tw), ty = int((m.ny + th - 1) / th);
    const int64_t items = int64_t(tx) * ty * ((m.nzl + best_kz - 1) / best_kz);
    const bool out16 = aligned16(outs[b]) && m.nx % vec == 0;  // tile kernel: 16-byte output stores
    words.push_back(pack_params(fptrs[b], outs[b], m.dev_tab[0], m.dev_tab[1], m.dev_tab[2], v, m.k0, m.k0 + m.nzl,
                                items, tx, ty, int(best_kz), tma ? 0 : (out16 ? 1 : 0)));
    wmax = std::max(wmax, words.back().size());
    first.push_back(first.back() + items);
  }
  // TMA: DfgTmaParams images (no peer halo: blocks carry their ghost
  // shells); rows: DfgRowsParams images; tile: plain DfgParams images
  const TmaBlobLayout bl = tma_blob_layout(nsf, int(L.stencil_inputs.size()), wmax);
  std::vector<std::vector<unsigned char>> rblobs;
  size_t rstride = 0;
  if (rows) {
    for (size_t b = 0; b < plans.size(); ++b) {
      std::vector<uint64_t> w = words[b];
      w.resize(wmax, 0);
      rblobs.push_back(rows_blob(fptrs[b], nsf, SlabView::of(*plans[b]->mesh), ncw, rpw, w, &plans[b]->rows_maps));
      rstride = std::max(rstride, rblobs.back().size());
    }
  }
  const size_t stride = tma ? bl.size : rows ? rstride : wmax * 8;
  std::vector<unsigned char> host(stride * plans.size() + sizeof(int64_t) * first.size(), 0);
  for (size_t b = 0; b < plans.size(); ++b) {
    unsigned char* blob = host.data() + stride * b;
    if (rows) {
      std::memcpy(blob, rblobs[b].data(), rblobs[b].size());
      continue;
    }
    if (!tma) {
      std::memcpy(blob, words[b].data(), words[b].size() * 8);
      continue;
    }
    const SlabView v = SlabView::of(*plans[b]->mesh);
    PlanImpl::MapCache& mc = plans[b]->tma_maps;
    const int64_t mk[4] = {v.px(), v.py(), v.nzl, int64_t(v.ghost)};
    if (!mc.hit(fptrs[b], mk)) {
      mc.maps.assign(size_t(128) * size_t(nsf), 0);
      for (int f = 0; f < nsf; ++f)
        encode_map(reinterpret_cast<CUtensorMap*>(mc.maps.data() + 128 * f), v, const_cast<void*>(fptrs[b][size_t(f)]),
                   ncw, rpw);
      mc.ptrs = fptrs[b];
      std::copy(mk, mk + 4, mc.key);
    }
    std::memcpy(blob, mc.maps.data(), mc.maps.size());
    std::memcpy(blob + bl.params, words[b].data(), words[b].size() * 8);
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
  if (p0.timing >= 1) DFG_CUDA(cudaEventRecord(p0.ev0, s));
  auto ke = p0.kernel_begin(s);
  const unsigned grid = unsigned(std::max<int64_t>(1, std::min(first.back(), slots)));
  DFG_CU(drv().LaunchKernel(fn, grid, 1, 1, threads, 1, 1, unsigned(smem), s, args, nullptr));
  p0.kernel_end(ke, s);
  if (p0.timing >= 1) DFG_CUDA(cudaEventRecord(p0.ev1, s));
  DFG_CUDA(cudaFreeAsync(dev, s));
  DFG_CUDA(cudaGetLastError());
  p0.timed = p0.timing >= 1;
  p0.st.kernel_count += 1;
  for (auto* p : plans) {
    p->st.executes += 1;
    p->last_variant = tma ? 4 : rows ? 8 : 6;
    p->last_kz = best_kz;
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

}  // namespace dfg
