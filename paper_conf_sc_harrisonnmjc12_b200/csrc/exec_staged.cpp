// libdfg staged, hybrid and roundtrip executors: one primitive kernel per filter.
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
#include "runtime_detail.hpp"

namespace dfg {
using namespace detail;

// ------------------------------------------------------------- staged
namespace {
// One primitive kernel over the owned cells of a whole mesh: o = f(args)
// (args: operand values, mesh references skipped); grad3d reads `gsrc`, its
// field's buffer from local plane 0, which has `gghost` ghost planes.
void launch_primitive(const MeshImpl& m, const Filter& f, void* o, const std::vector<const void*>& a,
                      const void* gsrc, int64_t gghost, const void* const tab[3], cudaStream_t s) {
  const int64_t N = m.cells();
  NvtxRange nv(op_name(f.op));
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

// Device-resident staged execute as a CUDA graph: the first execute for an
// (output, inputs) binding captures exec_staged on a private stream (the
// kernels, the stream-ordered allocations and frees of the intermediates)
// and every execute launches the instantiated graph on the caller's stream:
// one host call instead of one launch + allocation + free per filter.
void PlanImpl::exec_staged_graph(void* out, cudaStream_t s) {
  MeshImpl& m = *mesh;
  std::vector<const void*> key{out};
  for (int i : sources(dag).inputs) key.push_back(m.fields[dag.inputs[i]].ptr);
  if (!gexec || key != gkey) {
    if (gexec) {
      DFG_CUDA(cudaGraphExecDestroy(gexec));
      gexec = nullptr;
    }
    if (!sCap) DFG_CUDA(cudaStreamCreateWithFlags(&sCap, cudaStreamNonBlocking));
    pool_for(m.device);  // created outside the capture (pool creation is not capturable)
    const dfg_stats before = st;
    // the captured execute's own ledger high-water (replays repeat it)
    st.dev_highwater_bytes = 0;
    DFG_CUDA(cudaStreamBeginCapture(sCap, cudaStreamCaptureModeThreadLocal));
    cudaGraph_t g = nullptr;
    try {
      exec_staged(out, true, sCap);
    } catch (...) {
      cudaStreamEndCapture(sCap, &g);  // leave the stream usable
      if (g) cudaGraphDestroy(g);
      cudaGetLastError();
      st.dev_highwater_bytes = std::max(st.dev_highwater_bytes, before.dev_highwater_bytes);
      throw;
    }
    const int64_t captured_high = st.dev_highwater_bytes;
    st.dev_highwater_bytes = std::max(captured_high, before.dev_highwater_bytes);
    DFG_CUDA(cudaStreamEndCapture(sCap, &g));
    cudaError_t e = cudaGraphInstantiate(&gexec, g, 0);
    cudaGraphDestroy(g);
    DFG_CUDA(e);
    gdelta = dfg_stats{};
    gdelta.kernel_count = st.kernel_count - before.kernel_count;
    gdelta.h2d_count = st.h2d_count - before.h2d_count;
    gdelta.d2h_count = st.d2h_count - before.d2h_count;
    gdelta.h2d_bytes = st.h2d_bytes - before.h2d_bytes;
    gdelta.d2h_bytes = st.d2h_bytes - before.d2h_bytes;
    gdelta.dev_highwater_bytes = captured_high;
    gkey = key;
  } else {
    st.kernel_count += gdelta.kernel_count;
    st.h2d_count += gdelta.h2d_count;
    st.d2h_count += gdelta.d2h_count;
    st.h2d_bytes += gdelta.h2d_bytes;
    st.d2h_bytes += gdelta.d2h_bytes;
    st.dev_highwater_bytes = std::max(st.dev_highwater_bytes, gdelta.dev_highwater_bytes);
    graph_launches += 1;
  }
  DFG_CUDA(cudaGraphLaunch(gexec, s));
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
  // the decompose filters of each vector result: the first one to run
  // extracts every lane they need in one pass over the 4-wide host buffer
  // (same values, no transfers either way; one read of the vector instead of
  // one per lane -- the host pass is memory-bound)
  std::vector<std::vector<int>> dec_of(dag.filters.size());
  for (size_t k = 0; k < dag.filters.size(); ++k)
    if (dag.filters[k].op == Op::Decompose && dag.filters[k].in[0].kind == Ref::Filter)
      dec_of[size_t(dag.filters[k].in[0].id)].push_back(int(k));
  std::vector<char> extracted(dag.filters.size(), 0);

  auto host_const = [&](const Filter& f) -> void* {
    void* h = hp.get(sb);
    parallel_for(N, [&](int64_t a, int64_t b) {
      if (m.dt == DType::F32) std::fill(static_cast<float*>(h) + a, static_cast<float*>(h) + b, float(f.cval));
      else std::fill(static_cast<double*>(h) + a, static_cast<double*>(h) + b, f.cval);
    });
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
      if (extracted[k]) continue;  // taken with an earlier lane of the same vector
      const Ref& a = f.in[0];
      std::vector<int> ks = a.kind == Ref::Filter ? dec_of[size_t(a.id)] : std::vector<int>{int(k)};
      const int nk = int(ks.size());
      int lanes[4] = {0, 0, 0, 0};
      void* outs[4] = {nullptr, nullptr, nullptr, nullptr};
      for (int j = 0; j < nk; ++j) {
        lanes[j] = dag.filters[size_t(ks[size_t(j)])].k;
        outs[j] = hp.get(sb);
      }
      auto extract = [&](auto* v, auto** o) {
        parallel_for(N, [&](int64_t lo, int64_t hi) {
          for (int64_t e = lo; e < hi; ++e)
            for (int j = 0; j < nk; ++j) o[j][e] = v[4 * e + lanes[j]];
        });
      };
      if (m.dt == DType::F32) extract(static_cast<const float*>(hval[a.id]), reinterpret_cast<float**>(outs));
      else extract(static_cast<const double*>(hval[a.id]), reinterpret_cast<double**>(outs));
      for (int j = 0; j < nk; ++j) {
        hval[size_t(ks[size_t(j)])] = outs[j];
        extracted[size_t(ks[size_t(j)])] = 1;
        release(a);
      }
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
    const char* hsrc = static_cast<const char*>(hval[res.id]);
    parallel_for(int64_t(rb), [&](int64_t lo, int64_t hi) {
      std::memcpy(static_cast<char*>(out) + lo, hsrc + lo, size_t(hi - lo));
    });
  }
  DFG_CUDA(cudaStreamSynchronize(s));
  release(res);
  for (auto& p : hval)
    if (p) hp.put(p);
  st.dev_highwater_bytes = std::max<int64_t>(st.dev_highwater_bytes, int64_t(led.high));
}

}  // namespace dfg
