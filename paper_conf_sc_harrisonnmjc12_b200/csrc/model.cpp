// libdfg planner models: Table II counts, Fig. 2 footprints, the memory-aware staged order and the hybrid spill schedule.
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

// ==================================================================== model
namespace detail {
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
}  // namespace detail

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

}  // namespace dfg
