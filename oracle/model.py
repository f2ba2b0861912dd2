"""Oracle: device-event counts and device-memory footprint of the three
execution strategies.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Paper passages followed:

* roundtrip (L92-L94): one kernel per primitive, every result goes back to
  the host; arguments come from host memory, so every argument of every
  kernel is uploaded, duplicates included; decompose runs on the host
  (L289: only staged "implements the decomposition primitive using a kernel");
  constants are host buffers uploaded per use (L307).
* staged (L96): one kernel per primitive, intermediates stay in device
  memory; decompose is a kernel (L289); one fill kernel per distinct constant
  (reading R12, pinned by Table II: 67 = 57 + 9 decompose + 1 const).
* fusion (L97): one generated kernel, intermediates in registers.
* Table II (L271-L285): counts of host-to-device transfers (Dev-W),
  device-to-host transfers (Dev-R), kernel executions (K-Exe).
* Fig. 2 (L107-L114): device memory in problem-sized arrays: roundtrip holds
  one kernel's arguments and result; staged uploads inputs lazily and frees
  every array whose reference count reaches zero (L85 "reference counting");
  fusion holds all inputs and the output.

Modes (reading R13): ``host`` = the paper's host interface (L116-L118): the
bound fields live in host memory, the mesh arrays dims/x/y/z are uploaded
like the fields (Table II counts 7 = u,v,w,dims,x,y,z).  ``device`` = in situ
on the GPU: bound fields and mesh arrays are already resident, the output
buffer is on the device.

Footprint units: one scalar problem-sized array = 1; a vector array is
stored 4-wide (L104) = 4; the O(n) mesh arrays count 0.
"""

from __future__ import annotations

from dataclasses import dataclass

from .lang import Dag, MESH_NAMES


@dataclass(frozen=True)
class Counts:
    h2d: int
    d2h: int
    kernels: int


def _units(dag: Dag, ref: str) -> int:
    return 1 if dag.width_of(ref) == 1 else 4


def _is_filter(dag: Dag, ref: str) -> bool:
    return dag.ref_filter(ref) is not None


def _sources(dag: Dag):
    """Bound input fields the network reads, in first-use order, and whether
    it needs the mesh arrays (any grad3d)."""
    seen = []
    mesh = False
    for f in dag.filters:
        for r in f.inputs:
            if r in MESH_NAMES:
                mesh = True
            elif not _is_filter(dag, r) and r not in seen:
                seen.append(r)
    if not _is_filter(dag, dag.result) and dag.result not in seen:
        seen.append(dag.result)
    return seen, mesh


def counts(dag: Dag, strategy: str, mode: str = "host") -> Counts:
    """Device events of one execution (Table II in ``host`` mode)."""
    srcs, mesh = _sources(dag)
    F = len(dag.filters)
    bare = not _is_filter(dag, dag.result)
    if mode == "host":
        uploads = len(srcs) + (4 if mesh else 0)
        if strategy == "fused":
            return Counts(uploads, 1, 1)
        if strategy == "staged":
            return Counts(uploads, 1, F)
        if strategy == "roundtrip":
            h2d = k = 0
            for f in dag.filters:
                if f.op in ("decompose", "const"):
                    continue                      # host side, no transfer
                h2d += len(f.inputs)              # every argument, every use
                k += 1
            return Counts(h2d, k, k)
    elif mode == "device":
        if strategy == "fused":
            return Counts(0, 0, 1)
        if strategy == "staged":
            return Counts(0, 0, F)
        if strategy == "roundtrip":
            h2d = k = 0
            for f in dag.filters:
                if f.op in ("decompose", "const"):
                    continue
                # device-resident fields / mesh arrays are used in place;
                # intermediates and constants come from host memory
                h2d += sum(1 for r in f.inputs if _is_filter(dag, r))
                k += 1
            # a non-bare result travels host -> device output buffer
            return Counts(h2d + (0 if bare else 1), k, k)
    raise ValueError((strategy, mode))


def _refcounts(dag: Dag):
    rc: dict = {}
    for f in dag.filters:
        for r in f.inputs:
            if r not in MESH_NAMES:
                rc[r] = rc.get(r, 0) + 1
    rc[dag.result] = rc.get(dag.result, 0) + 1       # the sink holds the result
    return rc


def is_topological(dag: Dag, order) -> bool:
    """Every filter exactly once, each after all the filters it reads."""
    if sorted(order) != list(range(len(dag.filters))):
        return False
    pos = {k: i for i, k in enumerate(order)}
    for k, f in enumerate(dag.filters):
        for r in f.inputs:
            j = dag.ref_filter(r)
            if j is not None and pos[int(r[1:])] > pos[k]:
                return False
    return True


def footprint(dag: Dag, strategy: str, mode: str = "host", order=None) -> int:
    """Device high-water in problem-array units (Fig. 2).  ``order`` = the
    execution order of the staged strategy (default: list order, L72/L85)."""
    if order is not None and strategy == "staged":
        assert is_topological(dag, order)
        return _staged_footprint(dag, mode, order)
    srcs, _ = _sources(dag)
    out_units = _units(dag, dag.result)
    if strategy == "fused":
        return sum(_units(dag, s) for s in srcs) + out_units
    if strategy == "roundtrip":
        base = 0
        if mode == "device":
            base = sum(_units(dag, s) for s in srcs) + out_units
        high = base
        for k, f in enumerate(dag.filters):
            if f.op in ("decompose", "const"):
                continue
            args = 0
            for r in f.inputs:
                if r in MESH_NAMES:
                    continue
                if mode == "device" and not _is_filter(dag, r):
                    continue                      # resident, counted in base
                if _is_filter(dag, r) and dag.ref_filter(r).op == "decompose":
                    args += 1                     # host-decomposed scalar
                else:
                    args += _units(dag, r)
            high = max(high, base + args + _units(dag, f"f{k}"))
        return high
    if strategy == "staged":
        return _staged_footprint(dag, mode, range(len(dag.filters)))
    raise ValueError(strategy)


def _staged_footprint(dag: Dag, mode: str, order) -> int:
    """Lazy upload, free at reference count zero, filters run in ``order``."""
    srcs, _ = _sources(dag)
    out_units = _units(dag, dag.result)
    order = list(order)
    if True:
        rc = _refcounts(dag)
        live = 0
        high = 0
        resident: set = set()
        if mode == "device":
            live = sum(_units(dag, s) for s in srcs) + out_units
            resident = set(srcs)
            high = live
        last = order[-1] if order else -1
        for k in order:
            f = dag.filters[k]
            ref = f"f{k}"
            for r in f.inputs:
                if r in MESH_NAMES or _is_filter(dag, r) or r in resident:
                    continue
                resident.add(r)                   # lazy upload
                live += _units(dag, r)
            writes_out = mode == "device" and ref == dag.result and k == last
            if not writes_out:
                live += _units(dag, ref)
            high = max(high, live)
            for r in f.inputs:
                if r in MESH_NAMES:
                    continue
                rc[r] -= 1
                if rc[r] == 0 and not (mode == "device" and not _is_filter(dag, r)):
                    live -= _units(dag, r)        # free at refcount 0
        if not _is_filter(dag, dag.result) and dag.result not in resident:
            live += _units(dag, dag.result)       # bare input result: upload it
            high = max(high, live)
        return high


# ---------------------------------------------------------------- hybrid
# Staged execution under a device-memory cap with spill-to-host (SURVEY 8f
# NEXT #3, the Fig. 2 argument L107-L114 that staged execution can run where
# memory is short, carried one step further).  The policy is stated in
# DESIGN.md section 5b ("Hybrid"); this is a plain restatement of it, written
# independently of libdfg's C++ planner.

@dataclass
class Hybrid:
    events: list      # (kind, ref) in execution order
    counts: Counts    # h2d / d2h transfers and kernels of one execution
    high: int         # device high-water in units
    h2d_units: int    # problem-array units moved host -> device
    d2h_units: int    # problem-array units moved device -> host


class HybridInfeasible(Exception):
    """The cap is below the working set of some filter."""


def hybrid(dag: Dag, mode: str, cap: int, order=None) -> Hybrid:
    """Run the filters in ``order`` (default list order) holding at most
    ``cap`` units on the device.

    * device mode: the bound inputs and the output buffer stay resident and
      count against the cap throughout; host mode: inputs are uploaded when a
      filter needs them.
    * Before a filter runs, each operand that is not resident is brought in
      (an input: upload from the caller's host array; an intermediate: reload
      from its pinned host copy), then its result array is allocated (unless,
      in device mode, it is the result computed last, which goes straight into
      the output buffer).  Whenever the next array does not fit, the resident
      array with the furthest next use is evicted (ties: the larger, then
      filters before inputs, then the higher id), never an operand of the
      current filter: an intermediate without a host copy is spilled
      (device -> host, once: values never change; later evictions just discard
      the device copy), an input is dropped.
    * After the filter, every operand whose reference count reaches zero is
      freed (device and host copies).
    * The sink: the result goes to the caller (host mode: device -> host if it
      is resident, else from its host copy without a transfer; device mode:
      nothing if computed into the output buffer, a device copy if resident,
      else host -> device from its host copy).
    """
    if order is None:
        order = list(range(len(dag.filters)))
    order = list(order)
    assert is_topological(dag, order)
    srcs, mesh = _sources(dag)
    n = len(order)
    uses: dict = {}
    for p, k in enumerate(order):
        for r in dag.filters[k].inputs:
            if r not in MESH_NAMES:
                uses.setdefault(r, []).append(p)
    uses.setdefault(dag.result, []).append(n)          # the sink reads the result

    def next_use(ref, pos):
        later = [p for p in uses.get(ref, []) if p >= pos]
        return min(later) if later else n + 1

    def tie_key(ref):
        kind = 1 if _is_filter(dag, ref) else 0
        ident = int(ref[1:]) if kind else list(dag.inputs).index(ref)
        return (kind, ident)

    rc = _refcounts(dag)
    events: list = []
    resident: dict = {}                 # evictable device arrays -> units
    host_copy: set = set()
    base = 0
    if mode == "device":
        base = sum(_units(dag, s) for s in srcs) + _units(dag, dag.result)
    if base > cap:
        raise HybridInfeasible(f"cap {cap} below the resident inputs and output ({base})")
    high = base
    h2d = d2h = h2du = d2hu = 0
    mesh_up = False

    def live():
        return base + sum(resident.values())

    def make_room(units, protect, pos):
        nonlocal d2h, d2hu
        while live() + units > cap:
            cands = [r for r in resident if r not in protect]
            if not cands:
                raise HybridInfeasible(f"cap {cap} below the working set at position {pos}")
            victim = max(cands, key=lambda r: (next_use(r, pos), resident[r]) + tie_key(r))
            if _is_filter(dag, victim):
                if victim not in host_copy:
                    events.append(("spill", victim))
                    host_copy.add(victim)
                    d2h += 1
                    d2hu += resident[victim]
                else:
                    events.append(("discard", victim))      # host copy still valid
            else:
                events.append(("drop", victim))
            del resident[victim]

    def bring(ref, protect, pos):
        nonlocal h2d, h2du
        if ref in resident or (mode == "device" and not _is_filter(dag, ref)):
            return
        u = _units(dag, ref)
        make_room(u, protect, pos)
        if _is_filter(dag, ref):
            assert ref in host_copy
            events.append(("reload", ref))
        else:
            events.append(("upload", ref))
        h2d += 1
        h2du += u
        resident[ref] = u

    for pos, k in enumerate(order):
        f = dag.filters[k]
        ref = f"f{k}"
        need = [r for r in f.inputs if r not in MESH_NAMES]
        if mode == "host" and not mesh_up and any(r in MESH_NAMES for r in f.inputs):
            mesh_up = True
            h2d += 4                                        # dims, x, y, z (R13)
        for r in dict.fromkeys(need):
            bring(r, set(need), pos)
        writes_out = mode == "device" and ref == dag.result and pos == n - 1
        if not writes_out:
            make_room(_units(dag, ref), set(need), pos)
            resident[ref] = _units(dag, ref)
        high = max(high, live())
        events.append(("run", ref))
        for r in need:
            rc[r] -= 1
            if rc[r] == 0:
                resident.pop(r, None)
                host_copy.discard(r)

    res = dag.result
    if mode == "host":
        if res in resident:
            events.append(("sink_d2h", res))
            d2h += 1
            d2hu += _units(dag, res)
        elif res in host_copy:
            events.append(("sink_host", res))
        else:                                               # bare input result
            bring(res, {res}, n)
            high = max(high, live())
            events.append(("sink_d2h", res))
            d2h += 1
            d2hu += _units(dag, res)
    else:
        if _is_filter(dag, res) and res not in resident and not (order and f"f{order[-1]}" == res):
            events.append(("sink_h2d", res))
            h2d += 1
            h2du += _units(dag, res)
    return Hybrid(events, Counts(h2d, d2h, len(order)), high, h2du, d2hu)
