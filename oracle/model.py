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
