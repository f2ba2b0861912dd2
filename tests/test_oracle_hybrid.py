"""Pins of the oracle's hybrid (staged + spill-to-host) schedule
(oracle/model.py ``hybrid``).

* a worked example on the Fig. 2 network (L107-L114), derived by hand;
* reduction: when the cap holds the staged footprint nothing moves that the
  staged model (Table II / Fig. 2, pinned in test_oracle_lang.py) does not move;
* optimality: with every array one unit wide, evicting the furthest next use
  re-transfers as few arrays as any eviction choice (Belady), checked against
  an exhaustive search written here, on random networks;
* the schedule is valid: replayed by an independent checker, every operand
  is on the device when its filter runs and the cap is never exceeded.
"""

import random
from functools import lru_cache

import pytest

from oracle import model as M
from oracle.lang import MESH_NAMES, PAPER_PROGRAMS, build_dag

FIG2 = "r = (a + b) * (c + d)\n"


def test_fig2_worked_example():
    """cap 3, host mode, list order (derived by hand):
    f0 = a+b needs a, b, f0 = 3 units; a, b freed.  f1 = c+d: c, d uploaded
    (f0 + c + d = 3), f1 does not fit -> f0 (next use: f2) is spilled.  f2:
    f0 reloaded (f1 + f0 = 2), f2 allocated (3).  Sink: f2 device -> host."""
    dag = build_dag(FIG2, ("a", "b", "c", "d"))
    h = M.hybrid(dag, "host", 3)
    assert h.events == [("upload", "a"), ("upload", "b"), ("run", "f0"), ("upload", "c"), ("upload", "d"),
                        ("spill", "f0"), ("run", "f1"), ("reload", "f0"), ("run", "f2"), ("sink_d2h", "f2")]
    assert h.counts == M.Counts(5, 2, 3) and h.high == 3
    assert (h.h2d_units, h.d2h_units) == (5, 2)
    # cap 4 = the staged footprint of Fig. 2: no spill
    h4 = M.hybrid(dag, "host", 4)
    assert h4.counts == M.counts(dag, "staged", "host") and h4.high == 4
    with pytest.raises(M.HybridInfeasible):
        M.hybrid(dag, "host", 2)          # f0 alone needs a, b and its result


def test_device_mode_needs_room_for_resident_arrays():
    """Device mode keeps the bound inputs and the output on the device: a
    cap below them is infeasible even for a network with no filter."""
    dag = build_dag("a = u\n", ("u",))
    with pytest.raises(M.HybridInfeasible):
        M.hybrid(dag, "device", 1)
    assert M.hybrid(dag, "device", 2).high == 2
    h = M.hybrid(dag, "host", 1)                # host mode: upload u, copy it back
    assert h.events == [("upload", "u"), ("sink_d2h", "u")] and h.counts == M.Counts(1, 1, 0)


@pytest.mark.parametrize("prog", ["velmag", "vortmag", "qcrit", "intro"])
@pytest.mark.parametrize("mode", ["host", "device"])
def test_reduces_to_staged_when_the_cap_suffices(prog, mode):
    src, names = PAPER_PROGRAMS[prog]
    dag = build_dag(src, names)
    fp = M.footprint(dag, "staged", mode)
    for cap in (fp, fp + 3):
        h = M.hybrid(dag, mode, cap)
        assert h.high == fp
        assert h.counts == M.counts(dag, "staged", mode)
        assert not any(k in ("spill", "reload", "discard", "drop", "sink_h2d", "sink_host") for k, _ in h.events)


def replay(dag, mode, cap, order, events):
    """Independent validity check of an event list; returns re-transfers."""
    units = lambda r: 1 if dag.width_of(r) == 1 else 4  # noqa: E731
    is_f = lambda r: dag.ref_filter(r) is not None      # noqa: E731
    srcs = []
    for f in dag.filters:
        for r in f.inputs:
            if r not in MESH_NAMES and not is_f(r) and r not in srcs:
                srcs.append(r)
    dev = {}
    fixed = sum(units(s) for s in srcs) + units(dag.result) if mode == "device" else 0
    on_host = set()
    loaded_once, again = set(), 0
    runs = [k for k, _ in events if k == "run"]
    assert len(runs) == len(order)
    step = 0
    remaining = {}
    for k in order:
        for r in dag.filters[k].inputs:
            if r not in MESH_NAMES:
                remaining[r] = remaining.get(r, 0) + 1
    for kind, r in events:
        if kind in ("upload", "reload"):
            assert r not in dev
            if kind == "reload":
                assert r in on_host
            else:
                assert not is_f(r) and mode == "host"
            if r in loaded_once:
                again += 1
            loaded_once.add(r)
            dev[r] = units(r)
        elif kind == "spill":
            assert r in dev and is_f(r)
            on_host.add(r)
            del dev[r]
        elif kind == "discard":
            assert r in dev and r in on_host
            del dev[r]
        elif kind == "drop":
            assert r in dev and not is_f(r)
            del dev[r]
        elif kind == "run":
            k = order[step]
            assert r == f"f{k}"
            for a in dag.filters[k].inputs:
                if a in MESH_NAMES or (mode == "device" and not is_f(a)):
                    continue
                assert a in dev, (a, "not resident at", r)
            last = step == len(order) - 1
            if not (mode == "device" and r == dag.result and last):
                dev[r] = units(r)
            assert fixed + sum(dev.values()) <= cap
            loaded_once.add(r)
            for a in dag.filters[k].inputs:
                if a in MESH_NAMES:
                    continue
                remaining[a] -= 1
                if remaining[a] == 0 and a != dag.result:
                    dev.pop(a, None)
                    on_host.discard(a)
            step += 1
    assert step == len(order)
    return again


def min_retransfers(dag, cap, order):
    """Exhaustive search, host mode, every array one unit: the fewest arrays
    brought to the device a second time over all eviction choices."""
    is_f = lambda r: dag.ref_filter(r) is not None  # noqa: E731
    steps = []
    rc = {}
    for k in order:
        for r in dag.filters[k].inputs:
            rc[r] = rc.get(r, 0) + 1
    rc[dag.result] = rc.get(dag.result, 0) + 1
    left = dict(rc)
    for k in order:
        need = tuple(dict.fromkeys(dag.filters[k].inputs))
        dead = []
        for r in dag.filters[k].inputs:
            left[r] -= 1
            if left[r] == 0:
                dead.append(r)
        steps.append((need, f"f{k}", tuple(dead)))

    @lru_cache(maxsize=None)
    def go(i, j, dev, seen):
        # i: step; j: operand index (len(need) = the output); dev: resident set
        if i == len(steps):
            return 0
        need, out, dead = steps[i]
        if j <= len(need):
            want = need[j] if j < len(need) else out
            if j < len(need) and want in dev:
                return go(i, j + 1, dev, seen)
            cost = 1 if (j < len(need) and want in seen) else 0
            if len(dev) + 1 <= cap:
                return cost + go(i, j + 1, dev | {want}, seen | {want})
            best = None
            for v in dev:
                if v in need:
                    continue
                r = go(i, j, dev - {v}, seen)
                best = r if best is None else min(best, r)
            return float("inf") if best is None else best
        return go(i + 1, 0, frozenset(d for d in dev if d not in dead), seen)

    return go(0, 0, frozenset(), frozenset())


def random_program(rng, n_inputs=4, n_stmts=7):
    names = ["a", "b", "c", "d", "e"][:n_inputs]
    pool = list(names)
    lines = []
    for s in range(n_stmts):
        x, y = rng.choice(pool), rng.choice(pool)
        op = rng.choice(["+", "-", "*"])
        t = f"t{s}"
        lines.append(f"{t} = {x} {op} {y}")
        pool.append(t)
    # the result combines the last few temporaries so most values stay live
    lines.append("r = " + " + ".join(pool[-3:]))
    return "\n".join(lines) + "\n", tuple(names)


@pytest.mark.parametrize("seed", range(12))
def test_furthest_next_use_is_optimal_on_unit_arrays(seed):
    rng = random.Random(seed)
    src, names = random_program(rng)
    dag = build_dag(src, names)
    order = list(range(len(dag.filters)))
    fp = M.footprint(dag, "staged", "host")
    checked = 0
    for cap in range(2, fp + 1):
        try:
            h = M.hybrid(dag, "host", cap, order)
        except M.HybridInfeasible:
            assert min_retransfers(dag, cap, order) == float("inf")
            continue
        again = replay(dag, "host", cap, order, h.events)
        assert again == min_retransfers(dag, cap, order), (src, cap)
        checked += 1
    assert checked >= 1


@pytest.mark.parametrize("prog", ["vortmag", "qcrit", "intro"])
@pytest.mark.parametrize("mode", ["host", "device"])
def test_paper_programs_schedules_are_valid(prog, mode):
    src, names = PAPER_PROGRAMS[prog]
    dag = build_dag(src, names)
    fp = M.footprint(dag, "staged", mode)
    feasible = 0
    for cap in range(1, fp + 1):
        try:
            h = M.hybrid(dag, mode, cap)
        except M.HybridInfeasible:
            continue
        feasible += 1
        replay(dag, mode, cap, list(range(len(dag.filters))), h.events)
        assert h.high <= cap
        assert h.counts.kernels == len(dag.filters)
    assert feasible >= 2
