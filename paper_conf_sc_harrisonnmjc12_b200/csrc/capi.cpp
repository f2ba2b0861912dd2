// extern "C" entry points of libdfg.so (include/dfg.h).  Each one catches
// every internal DfgError, records the message for dfg_last_error() and
// returns the status; nothing throws across the ABI.
#include <cuda_runtime.h>

#include <cmath>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <string>
#include <vector>

#include "dfg.h"
#include "div2.hpp"
#include "runtime.hpp"

struct dfg_mesh_s {
  std::shared_ptr<dfg::MeshImpl> m;
};
struct dfg_plan_s {
  std::unique_ptr<dfg::PlanImpl> p;
};

namespace dfg {
namespace {
thread_local std::string t_err;
}
void set_last_error(const std::string& m) { t_err = m; }
void clear_last_error() { t_err.clear(); }
}  // namespace dfg

namespace {

template <typename F>
int guard(F&& f) {
  try {
    dfg::clear_last_error();
    f();
    return DFG_OK;
  } catch (const dfg::DfgError& e) {
    dfg::set_last_error(e.what());
    return e.status;
  } catch (const std::bad_alloc&) {
    dfg::set_last_error("host out of memory");
    return DFG_E_NOMEM;
  } catch (const std::exception& e) {
    dfg::set_last_error(std::string("internal error: ") + e.what());
    return DFG_E_INVALID;
  }
}

int copy_out(const std::string& s, char* buf, size_t cap, size_t* needed) {
  if (needed) *needed = s.size() + 1;
  if (!buf || cap < s.size() + 1) {
    if (buf && cap) {
      std::memcpy(buf, s.data(), cap - 1);
      buf[cap - 1] = '\0';
    }
    dfg::fail(DFG_E_RANGE, "buffer too small: need " + std::to_string(s.size() + 1) + " bytes");
  }
  std::memcpy(buf, s.c_str(), s.size() + 1);
  return 0;
}

std::vector<std::string> names_of(const char* const* inputs, int n) {
  if (n < 0 || (n > 0 && !inputs)) dfg::fail(DFG_E_INVALID, "bad input name list");
  std::vector<std::string> v;
  for (int i = 0; i < n; ++i) {
    if (!inputs[i]) dfg::fail(DFG_E_INVALID, "null input name");
    v.emplace_back(inputs[i]);
  }
  return v;
}

dfg::DType to_dtype(int d) {
  if (d != DFG_F32 && d != DFG_F64) dfg::fail(DFG_E_INVALID, "bad dtype");
  return d == DFG_F32 ? dfg::DType::F32 : dfg::DType::F64;
}

}  // namespace

extern "C" {

int dfg_version(void) { return 100; }

const char* dfg_last_error(void) { return dfg::t_err.c_str(); }

int dfg_create_mesh(dfg_dtype dtype, int64_t nx, int64_t ny, int64_t nz_local, const void* x, const void* y,
                    const void* z, int64_t nz_global, int64_t z_offset, int ghost, dfg_mesh* out) {
  return guard([&] {
    if (!out) dfg::fail(DFG_E_INVALID, "null output handle");
    *out = nullptr;
    auto m = dfg::create_mesh(to_dtype(dtype), nx, ny, nz_local, x, y, z, nz_global, z_offset, ghost);
    *out = new dfg_mesh_s{std::move(m)};
  });
}

int dfg_create_block(dfg_dtype dtype, int64_t nx, int64_t ny, int64_t nz, const void* x, const void* y,
                     const void* z, int64_t NX, int64_t NY, int64_t NZ, int64_t i0, int64_t j0, int64_t k0, int ghost,
                     int64_t row_pitch, int64_t x_offset, dfg_mesh* out) {
  return guard([&] {
    if (!out) dfg::fail(DFG_E_INVALID, "null output handle");
    *out = nullptr;
    auto m = dfg::create_block(to_dtype(dtype), nx, ny, nz, x, y, z, NX, NY, NZ, i0, j0, k0, ghost, row_pitch,
                               x_offset);
    *out = new dfg_mesh_s{std::move(m)};
  });
}

void dfg_destroy_mesh(dfg_mesh mesh) { delete mesh; }

int dfg_partition(int64_t nz_global, int nranks, int rank, int64_t* z_offset, int64_t* nz_local) {
  return guard([&] {
    if (nranks < 1 || nz_global < nranks || rank < 0 || rank >= nranks || !z_offset || !nz_local)
      dfg::fail(DFG_E_INVALID, "need 1 <= nranks <= nz_global and 0 <= rank < nranks");
    int64_t q = nz_global / nranks, r = nz_global % nranks;
    *nz_local = q + (rank < r ? 1 : 0);
    *z_offset = int64_t(rank) * q + (rank < r ? rank : r);
  });
}

int dfg_halo_map(dfg_mesh mesh, int64_t out[16]) {
  return guard([&] {
    if (!mesh || !out) dfg::fail(DFG_E_INVALID, "null argument");
    const dfg::MeshImpl& m = *mesh->m;
    const int64_t k1 = m.k0 + m.nzl;
    const int64_t lo = m.k0 > 0, hi = k1 < m.NZ;
    int64_t v[16] = {m.rank,          m.nranks,         m.NZ,          m.k0,
                     k1,              m.nzl,            lo,            hi,
                     lo ? m.rank - 1 : -1, hi ? m.rank + 1 : -1, lo ? 1 : -1, hi ? m.nzl : -1,
                     lo ? 0 : -1,     hi ? m.nzl + 1 : -1, m.nx * m.ny * int64_t(dfg::dsize(m.dt)), m.ghost};
    std::memcpy(out, v, sizeof(v));
  });
}

int dfg_nccl_unique_id(void* out128) {
  return guard([&] {
    if (!out128) dfg::fail(DFG_E_INVALID, "null buffer");
    dfg::nccl_unique_id(out128);
  });
}

int dfg_mesh_init_comm(dfg_mesh mesh, const void* id128, int rank, int nranks) {
  return guard([&] {
    if (!mesh || (!id128 && nranks > 1)) dfg::fail(DFG_E_INVALID, "null argument");
    dfg::mesh_init_comm(*mesh->m, id128, rank, nranks);
  });
}

int dfg_mesh_peer_export(dfg_mesh mesh, void* blob, size_t cap) {
  return guard([&] {
    if (!mesh || !blob) dfg::fail(DFG_E_INVALID, "null argument");
    if (cap < dfg::kPeerBlobBytes) dfg::fail(DFG_E_RANGE, "peer blob needs DFG_PEER_BLOB_BYTES bytes");
    dfg::mesh_peer_export(*mesh->m, blob);
  });
}

int dfg_mesh_link_peers(dfg_mesh mesh, const void* lo_blob, const void* hi_blob) {
  return guard([&] {
    if (!mesh) dfg::fail(DFG_E_INVALID, "null mesh");
    dfg::mesh_link_peers(*mesh->m, lo_blob, hi_blob);
  });
}

int dfg_peer_probe(const void* blob, int* ok) {
  return guard([&] {
    if (!blob || !ok) dfg::fail(DFG_E_INVALID, "null argument");
    *ok = 0;
    *ok = dfg::peer_probe(blob) ? 1 : 0;
  });
}

int dfg_mesh_link_local(dfg_mesh lo, dfg_mesh hi) {
  return guard([&] {
    if (!lo || !hi) dfg::fail(DFG_E_INVALID, "null mesh");
    auto& a = *lo->m;
    auto& b = *hi->m;
    if (a.k0 + a.nzl != b.k0 || a.NZ != b.NZ || a.nx != b.nx || a.ny != b.ny || a.dt != b.dt)
      dfg::fail(DFG_E_INVALID, "meshes are not adjacent z slabs of one mesh");
    a.link_hi = hi->m;
    b.link_lo = lo->m;
  });
}

int dfg_bind_field(dfg_mesh mesh, const char* name, void* ptr, int on_device) {
  return guard([&] {
    if (!mesh || !name) dfg::fail(DFG_E_INVALID, "null argument");
    std::string n(name);
    if (!dfg::valid_input_name(n)) dfg::fail(DFG_E_INVALID, "invalid field name '" + n + "'");
    if (!ptr) {
      mesh->m->fields.erase(n);
      return;
    }
    if (on_device) {
      cudaPointerAttributes a{};
      if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess || a.type != cudaMemoryTypeDevice) {
        cudaGetLastError();
        if (a.type != cudaMemoryTypeManaged)
          dfg::fail(DFG_E_INVALID, "field '" + n + "' is not a device pointer");
      }
    }
    mesh->m->fields[n] = dfg::Binding{ptr, on_device != 0};
  });
}

int dfg_compile(dfg_mesh mesh, const char* expr, dfg_strategy strategy, size_t cap, dfg_plan* out) {
  return guard([&] {
    if (!mesh || !expr || !out) dfg::fail(DFG_E_INVALID, "null argument");
    *out = nullptr;
    auto p = dfg::compile_plan(mesh->m, expr, strategy, cap);
    *out = new dfg_plan_s{std::move(p)};
  });
}

void dfg_destroy_plan(dfg_plan plan) { delete plan; }

int dfg_execute(dfg_plan plan, void* out, int out_on_device, void* stream) {
  return guard([&] {
    if (!plan) dfg::fail(DFG_E_INVALID, "null plan");
    plan->p->execute(out, out_on_device != 0, static_cast<cudaStream_t>(stream));
  });
}

int dfg_execute_blocks(dfg_plan const* plans, int n, void* const* outs, void* stream) {
  return guard([&] {
    if (!plans || !outs || n < 1) dfg::fail(DFG_E_INVALID, "need n >= 1 plans and outputs");
    std::vector<dfg::PlanImpl*> ps;
    std::vector<void*> os;
    for (int b = 0; b < n; ++b) {
      if (!plans[b] || !outs[b]) dfg::fail(DFG_E_INVALID, "null plan or output");
      ps.push_back(plans[b]->p.get());
      os.push_back(outs[b]);
    }
    dfg::execute_blocks(ps, os, static_cast<cudaStream_t>(stream));
  });
}

int dfg_plan_stats(dfg_plan plan, dfg_stats* out) {
  return guard([&] {
    if (!plan || !out) dfg::fail(DFG_E_INVALID, "null argument");
    auto& p = *plan->p;
    if (p.timed) {
      DFG_CUDA(cudaEventSynchronize(p.ev1));
      float ms = 0;
      DFG_CUDA(cudaEventElapsedTime(&ms, p.ev0, p.ev1));
      p.st.last_ms = ms;
    }
    p.resolve_kernel_times();
    *out = p.st;
  });
}

int dfg_plan_set_timing(dfg_plan plan, int level) {
  return guard([&] {
    if (!plan) dfg::fail(DFG_E_INVALID, "null plan");
    if (level < 0 || level > 2) dfg::fail(DFG_E_INVALID, "timing level must be 0, 1 or 2");
    plan->p->resolve_kernel_times();
    plan->p->timing = level;
    if (level == 0) plan->p->timed = false;
  });
}

int dfg_reset_stats(dfg_plan plan) {
  return guard([&] {
    if (!plan) dfg::fail(DFG_E_INVALID, "null plan");
    plan->p->resolve_kernel_times();
    plan->p->st = dfg_stats{};
    plan->p->st.last_ms = -1;
    plan->p->timed = false;
  });
}

int dfg_plan_info(dfg_plan plan, int64_t out[14]) {
  return guard([&] {
    if (!plan || !out) dfg::fail(DFG_E_INVALID, "null argument");
    auto& p = *plan->p;
    const auto& m = *p.mesh;
    out[0] = p.strategy;
    out[1] = p.dag.width(p.dag.result) == 1 ? 1 : 4;
    out[2] = int64_t(p.dag.filters.size());
    out[3] = p.last_variant;
    out[4] = p.regs > 0 ? p.regs : 0;
    out[5] = p.spill > 0 ? p.spill : 0;
    const int64_t unit = m.cells() * int64_t(dfg::dsize(m.dt));
    out[6] = dfg::model(p.dag, p.strategy, false).units * unit;
    out[7] = dfg::model(p.dag, p.strategy, true).units * unit;
    out[8] = p.fsrc.cfg.div2;
    const bool tma = p.fsrc.cfg.has_tma;
    out[9] = tma ? p.fsrc.cfg.rpw : 0;
    out[10] = tma ? dfg::tma_tile_w(m.dt, p.fsrc.cfg.rpw) : 0;
    out[11] = tma ? dfg::tma_tile_h(p.fsrc.cfg.ncw, p.fsrc.cfg.rpw) : 0;
    out[12] = p.last_kz;
    out[13] = p.last_halo;
  });
}

int dfg_plan_arith(dfg_plan plan, int64_t out[4]) {
  return guard([&] {
    if (!plan || !out) dfg::fail(DFG_E_INVALID, "null argument");
    const auto& p = *plan->p;
    const bool fused = p.strategy == DFG_FUSED || p.strategy == DFG_STREAMED || p.strategy == DFG_REFERENCE;
    const int div = fused ? p.fsrc.cfg.div_mode : 0;  // per-primitive kernels: IEEE div.rn
    const bool fold = fused && p.fsrc.cfg.fold;
    out[0] = div;
    out[1] = fold ? 1 : 0;
    out[2] = fused ? p.fsrc.cfg.div2 : 0;
    // 2: equal to the oracle for every input; 1: for every input whose
    // literal-network intermediates are all zero or normal and finite;
    // 0: within tolerance (fast quotient, hand-written reference body)
    out[3] = p.strategy == DFG_REFERENCE || div == 2 ? 0 : (div == 0 && !fold) ? 2 : 1;
  });
}

int dfg_plan_schedule(dfg_plan plan, int32_t* order, size_t cap, size_t* n) {
  return guard([&] {
    if (!plan || !n) dfg::fail(DFG_E_INVALID, "null argument");
    const auto& o = plan->p->order;
    *n = o.size();
    for (size_t i = 0; i < o.size() && i < cap && order; ++i) order[i] = o[i];
  });
}

int dfg_plan_transfers(dfg_plan plan, int32_t* events, size_t cap, size_t* n) {
  return guard([&] {
    if (!plan || !n) dfg::fail(DFG_E_INVALID, "null argument");
    const auto& p = *plan->p;
    if (p.strategy != DFG_HYBRID) dfg::fail(DFG_E_INVALID, "not a hybrid plan");
    const auto& ev = p.hyb.ev;
    *n = ev.size();
    for (size_t i = 0; i < ev.size() && i < cap && events; ++i) {
      events[2 * i] = int32_t(ev[i].kind);
      events[2 * i + 1] = ev[i].ref.kind == dfg::Ref::Input ? -1 - ev[i].ref.id : ev[i].ref.id;
    }
  });
}

int dfg_dump_dag(dfg_plan plan, char* buf, size_t cap, size_t* needed) {
  return guard([&] {
    if (!plan) dfg::fail(DFG_E_INVALID, "null plan");
    copy_out(plan->p->dag.dump(), buf, cap, needed);
  });
}

int dfg_dump_kernel(dfg_plan plan, char* buf, size_t cap, size_t* needed) {
  return guard([&] {
    if (!plan) dfg::fail(DFG_E_INVALID, "null plan");
    copy_out(plan->p->fsrc.source, buf, cap, needed);
  });
}

}  // extern "C"

namespace {
template <typename T>
void axes_from_points3d(int64_t nx, int64_t ny, int64_t nz, const T* x3, const T* y3, const T* z3, T* x, T* y, T* z) {
  const int64_t px = nx + 1, py = ny + 1, pz = nz + 1;
  for (int64_t i = 0; i < px; ++i) x[i] = x3[i];
  for (int64_t j = 0; j < py; ++j) y[j] = y3[j * px];
  for (int64_t k = 0; k < pz; ++k) z[k] = z3[k * px * py];
  for (int64_t k = 0; k < pz; ++k)
    for (int64_t j = 0; j < py; ++j)
      for (int64_t i = 0; i < px; ++i) {
        const int64_t e = (k * py + j) * px + i;
        if (!(x3[e] == x[i] && y3[e] == y[j] && z3[e] == z[k]))
          dfg::fail(DFG_E_INVALID, "point coordinates are not rectilinear at (" + std::to_string(i) + "," +
                                       std::to_string(j) + "," + std::to_string(k) + ")");
      }
}
}  // namespace

extern "C" {

int dfg_points3d_to_axes(dfg_dtype dtype, int64_t nx, int64_t ny, int64_t nz, const void* x3, const void* y3,
                         const void* z3, void* x, void* y, void* z) {
  return guard([&] {
    if (nx < 1 || ny < 1 || nz < 1) dfg::fail(DFG_E_INVALID, "mesh sizes must be >= 1");
    if (!x3 || !y3 || !z3 || !x || !y || !z) dfg::fail(DFG_E_INVALID, "null pointer");
    if (to_dtype(dtype) == dfg::DType::F32)
      axes_from_points3d(nx, ny, nz, static_cast<const float*>(x3), static_cast<const float*>(y3),
                         static_cast<const float*>(z3), static_cast<float*>(x), static_cast<float*>(y),
                         static_cast<float*>(z));
    else
      axes_from_points3d(nx, ny, nz, static_cast<const double*>(x3), static_cast<const double*>(y3),
                         static_cast<const double*>(z3), static_cast<double*>(x), static_cast<double*>(y),
                         static_cast<double*>(z));
  });
}

int dfg_paper_program(const char* which, char* buf, size_t cap, size_t* needed) {
  return guard([&] {
    if (!which) dfg::fail(DFG_E_INVALID, "null name");
    int id = 0;
    const char* prog = dfg::reference_program(which, &id);
    if (!prog) dfg::fail(DFG_E_INVALID, "paper programs: \"velmag\", \"vortmag\", \"qcrit\", \"intro\"");
    copy_out(prog, buf, cap, needed);
  });
}

int dfg_div2_check(dfg_dtype dtype, const void* d, int64_t n, int method, uint8_t* ok, int64_t* tested) {
  return guard([&] {
    if (!d || !ok || n < 0) dfg::fail(DFG_E_INVALID, "null pointer or negative count");
    if (method != 0 && method != 1) dfg::fail(DFG_E_INVALID, "method must be 0 (candidates) or 1 (exhaustive)");
    if (method == 1 && to_dtype(dtype) != dfg::DType::F32) dfg::fail(DFG_E_UNSUPPORTED, "exhaustive check is fp32 only");
    for (int64_t i = 0; i < n; ++i) {
      long c = 0;
      bool v;
      if (to_dtype(dtype) == dfg::DType::F32) {
        const float di = static_cast<const float*>(d)[i];
        if (!(di > 0.0f) || !std::isnormal(di)) dfg::fail(DFG_E_INVALID, "divisors must be positive normal numbers");
        const float r = 1.0f / di, yl = dfg::div2_low_part(di, r);
        v = method == 0 ? dfg::certify_div2<float>(di, r, yl, 16, &c) : dfg::exhaustive_div2_f32(di, r, yl);
      } else {
        const double di = static_cast<const double*>(d)[i];
        if (!(di > 0.0) || !std::isnormal(di)) dfg::fail(DFG_E_INVALID, "divisors must be positive normal numbers");
        const double r = 1.0 / di, yl = dfg::div2_low_part(di, r);
        v = dfg::certify_div2<double>(di, r, yl, 16, &c);
      }
      ok[i] = v ? 1 : 0;
      if (tested) tested[i] = c;
    }
  });
}

int dfg_dag_dump(const char* expr, const char* const* inputs, int n_inputs, dfg_dtype dtype, char* buf, size_t cap,
                 size_t* needed) {
  return guard([&] {
    if (!expr) dfg::fail(DFG_E_INVALID, "null expression");
    dfg::Dag d = dfg::build_dag(expr, names_of(inputs, n_inputs), to_dtype(dtype));
    copy_out(d.dump(), buf, cap, needed);
  });
}

int dfg_model(const char* expr, const char* const* inputs, int n_inputs, dfg_strategy strategy, int host_mode,
              int64_t out[4]) {
  return guard([&] {
    if (!expr || !out) dfg::fail(DFG_E_INVALID, "null argument");
    if (strategy < DFG_ROUNDTRIP || strategy > DFG_HYBRID) dfg::fail(DFG_E_INVALID, "bad strategy");
    int ref = 0;
    const char* prog = strategy == DFG_REFERENCE ? dfg::reference_program(expr, &ref) : expr;
    if (strategy == DFG_REFERENCE && ref == 0) dfg::fail(DFG_E_INVALID, "reference kernels exist for velmag, vortmag and qcrit");
    dfg::Dag d = dfg::build_dag(prog, names_of(inputs, n_inputs), dfg::DType::F32);
    dfg::Model m = dfg::model(d, strategy, host_mode != 0);
    out[0] = m.h2d;
    out[1] = m.d2h;
    out[2] = m.kernels;
    out[3] = m.units;
  });
}

int dfg_hybrid_model(const char* expr, const char* const* inputs, int n_inputs, int host_mode, int64_t cap_units,
                     const int32_t* order, size_t n_order, int32_t* events, size_t cap, size_t* n, int64_t out[5]) {
  return guard([&] {
    if (!expr || !n || !out) dfg::fail(DFG_E_INVALID, "null argument");
    dfg::Dag d = dfg::build_dag(expr, names_of(inputs, n_inputs), dfg::DType::F32);
    const size_t nf = d.filters.size();
    std::vector<int> o(nf);
    for (size_t k = 0; k < nf; ++k) o[k] = int(k);
    if (order) {
      if (n_order != nf) dfg::fail(DFG_E_INVALID, "order must list every filter once");
      std::vector<int> pos(nf, -1);
      for (size_t i = 0; i < nf; ++i) {
        const int k = order[i];
        if (k < 0 || size_t(k) >= nf || pos[size_t(k)] >= 0) dfg::fail(DFG_E_INVALID, "order must list every filter once");
        pos[size_t(k)] = int(i);
        o[i] = k;
      }
      for (size_t k = 0; k < nf; ++k)
        for (auto& r : d.filters[k].in)
          if (r.kind == dfg::Ref::Filter && pos[size_t(r.id)] > pos[k]) dfg::fail(DFG_E_INVALID, "order is not topological");
    }
    dfg::HybridPlan hp = dfg::plan_hybrid(d, o, cap_units, host_mode != 0);
    *n = hp.ev.size();
    for (size_t i = 0; i < hp.ev.size() && i < cap && events; ++i) {
      events[2 * i] = int32_t(hp.ev[i].kind);
      events[2 * i + 1] = hp.ev[i].ref.kind == dfg::Ref::Input ? -1 - hp.ev[i].ref.id : hp.ev[i].ref.id;
    }
    out[0] = hp.high;
    out[1] = hp.h2d;
    out[2] = hp.d2h;
    out[3] = hp.h2d_units;
    out[4] = hp.d2h_units;
  });
}

int dfg_fused_source(const char* expr, const char* const* inputs, int n_inputs, dfg_dtype dtype, int64_t nx,
                     int64_t ny, int64_t nz, int compile, char* buf, size_t cap, size_t* needed, int* regs,
                     int* spill) {
  return guard([&] {
    if (!expr) dfg::fail(DFG_E_INVALID, "null expression");
    if (nx < 1 || ny < 1 || nz < 1) dfg::fail(DFG_E_INVALID, "mesh sizes must be >= 1");
    dfg::Dag d = dfg::build_dag(expr, names_of(inputs, n_inputs), to_dtype(dtype));
    // no mesh here: describe the kernel of a mesh whose divisors all verified
    // (two-operation quotient on every axis), unless DFG_FUSED_VARIANT=markstein
    dfg::FusedConfig cfg;
    const char* var = std::getenv("DFG_FUSED_VARIANT");
    if (!(var && !std::strcmp(var, "markstein"))) cfg.div2 = 7;
    // tile shape: DFG_RPW (15 warps), else the planner's choice for a 148-SM B200
    // (rows of nx cells: the row-class kernel's when they are not 16-byte
    // multiples, or with DFG_FUSED_KERNEL=rows, as compile_plan)
    const char* rpw = std::getenv("DFG_RPW");
    const char* fk = std::getenv("DFG_FUSED_KERNEL");
    const int64_t vec = d.dtype == dfg::DType::F32 ? 4 : 2;
    if (rpw) cfg.rpw = std::atoi(rpw);
    else if (nx % vec != 0 || (fk && !std::strcmp(fk, "rows")))
      dfg::choose_rows_tile(d.dtype, nx, ny, nz, 148, &cfg.ncw, &cfg.rpw);
    else dfg::choose_tile(d.dtype, nx, ny, nz, 148, &cfg.ncw, &cfg.rpw);
    if (cfg.rpw != 2 && cfg.rpw != 4) cfg.rpw = 1;
    dfg::FusedSource fs = dfg::generate_fused(d, nx, ny, nz, cfg);
    if (compile) {
      static const std::string kUnit = "dfg_fused.cu";
      const dfg::Cubin& c = dfg::nvrtc_compile(fs.source, kUnit);
      if (regs) *regs = c.regs;
      if (spill) *spill = c.spill;
    }
    copy_out(fs.source, buf, cap, needed);
  });
}

}  // extern "C"
