"""GPU parity: libdfg (all strategies, both kernels) against the oracle,
element by element on the same seeded inputs.  Exact-division mode (the
default) must be bit-identical to the oracle."""

import os

import numpy as np
import pytest
import torch

import synth
from oracle import evaluate as oev
from oracle import model as omodel
from oracle.lang import PAPER_PROGRAMS, build_dag
from dfg_testutil import assert_parity, run_lib, run_oracle, tdtype

pytestmark = pytest.mark.gpu

PROGS = ["velmag", "vortmag", "qcrit", "intro"]
NAMES = {"velmag": ("u", "v", "w"), "vortmag": ("u", "v", "w"), "qcrit": ("u", "v", "w"), "intro": ("b", "c")}


def _rows_layout(px, py, itemsize, plan=None):
    """The row-class kernel's preconditions (16-byte aligned bases, as torch
    allocations are, 16-byte plane strides, a row of every class per plane,
    -- its lanes own whole cells of RPW rows -- RPW <= VEC / 2, and at most
    14 consumer warps (with its producer and fixup warps, 16 warps keep 128
    registers)): layouts the tensor maps cannot take run on it (variant 7),
    the rest on the cp.async ring (5)."""
    period = next(p for p in (1, 2, 4) if (px * itemsize * p) % 16 == 0)
    ok = (px * py * itemsize) % 16 == 0 and py >= period
    if plan is not None:
        info = plan.info()
        ok = ok and info["rows_per_warp"] <= 8 // itemsize and info["tile_h"] // info["rows_per_warp"] <= 14
    return ok


def _inputs(shape, T, names=("u", "v", "w")):
    x, y, z, f = synth.rt_inputs(*shape, dtype=T, names=names)
    return x, y, z, {k: v.numpy() for k, v in f.items()}


@pytest.fixture(autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_harrisonnmjc12_b200  # noqa: F401  (fails loudly if the .so is missing)


@pytest.mark.parametrize("prog", PROGS)
@pytest.mark.parametrize("strategy", ["fused", "staged", "roundtrip"])
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(32, 32, 32), (132, 40, 33), (67, 45, 37)])
def test_parity_paper_programs(prog, strategy, T, shape):
    """32^3 is config 1; 132 x 40 x 33 spans two x tiles, a ragged y tile and
    odd z (TMA path); nx = 67 is not a multiple of 4 (general kernel)."""
    x, y, z, f = _inputs(shape, T, NAMES[prog])
    src = PAPER_PROGRAMS[prog][0]
    want = run_oracle(src, f, x, y, z)
    got = run_lib(src, f, x, y, z, strategy)
    assert_parity(got, want)


@pytest.mark.parametrize("T", [np.float32, np.float64])
def test_tma_and_general_kernels_identical(T, monkeypatch):
    x, y, z, f = _inputs((128, 48, 40), T)
    src = PAPER_PROGRAMS["qcrit"][0]
    a, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["variant"] == 1           # TMA pipeline ran
    monkeypatch.setenv("DFG_FUSED_KERNEL", "general")
    b, plan2, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan2.info()["variant"] == 2
    assert np.array_equal(a, b)
    monkeypatch.setenv("DFG_FUSED_KERNEL", "tile")
    c, plan3, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan3.info()["variant"] == 5
    assert np.array_equal(a, c)


@pytest.mark.parametrize("prog", PROGS)
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(67, 45, 37), (130, 17, 5), (5, 70, 9), (1, 33, 6), (129, 1, 4), (3, 2, 1)])
@pytest.mark.parametrize("rpw", ["1", "2", "4"])
def test_tile_kernel(prog, T, shape, rpw, monkeypatch):
    """The cp.async-filled ring (layouts a tensor map cannot describe): rows
    that are not a multiple of 16 bytes, ragged last vectors, degenerate
    axes, every tile shape -- the oracle's bits."""
    x, y, z, f = _inputs(shape, T, NAMES[prog])
    src = PAPER_PROGRAMS[prog][0]
    want = run_oracle(src, f, x, y, z)
    monkeypatch.setenv("DFG_RPW", rpw)
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    if prog != "velmag":
        vec = 4 if T == np.float32 else 2
        ragged = 7 if _rows_layout(shape[0], shape[1], np.dtype(T).itemsize, plan) else 5
        assert plan.info()["variant"] == (ragged if shape[0] % vec else 1)
    assert_parity(got, want)


@pytest.mark.parametrize("prog", PROGS)
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(66, 8, 9), (67, 16, 7), (65, 32, 6), (130, 12, 10), (6, 2, 3), (1, 4, 5),
                                   (131, 4, 3), (258, 2, 4), (33, 4, 2), (2, 8, 1), (197, 36, 12)])
def test_rows_kernel(prog, T, shape, monkeypatch):
    """The row-copy ring (one bulk copy per halo'd tile row, rows shifted by
    their global misalignment, warp-uniform realignment in the consumers):
    rows of 2 mod 4, odd and 1 cells (every shift 0..3 recurs), ragged last
    vectors, one-cell axes, several x tiles -- the oracle's bits, and the
    cp.async ring's."""
    isz = np.dtype(T).itemsize
    if not _rows_layout(shape[0], shape[1], isz):
        pytest.skip("plane stride not a multiple of 16 bytes for this type")
    x, y, z, f = _inputs(shape, T, NAMES[prog])
    src = PAPER_PROGRAMS[prog][0]
    want = run_oracle(src, f, x, y, z)
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    vec = 16 // isz
    if prog != "velmag":
        assert plan.info()["variant"] == ((7 if _rows_layout(shape[0], shape[1], isz, plan) else 5)
                                          if shape[0] % vec else 1)
    assert_parity(got, want)
    if prog != "velmag":
        monkeypatch.setenv("DFG_FUSED_KERNEL", "rows")     # also where the tensor maps could run
        got2, plan2, *_ = run_lib(src, f, x, y, z, return_plan=True)
        assert plan2.info()["variant"] == (7 if _rows_layout(shape[0], shape[1], isz, plan2) else 5)
        assert_parity(got2, want)
        monkeypatch.setenv("DFG_FUSED_KERNEL", "tile")
        got3, plan3, *_ = run_lib(src, f, x, y, z, return_plan=True)
        assert plan3.info()["variant"] == 5
        assert np.array_equal(got.view(np.uint8), got3.view(np.uint8))


@pytest.mark.parametrize("kz", ["1", "2", "5", "1000"])
def test_rows_kernel_z_chunks(kz, monkeypatch):
    """Every z-chunk length on the row-copy ring (producer and consumers
    cross item boundaries)."""
    x, y, z, f = _inputs((66, 32, 29), np.float32)
    src = PAPER_PROGRAMS["qcrit"][0]
    monkeypatch.setenv("DFG_KZ", kz)
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["variant"] == 7 and plan.info()["kz"] == min(int(kz), 29)
    assert_parity(got, run_oracle(src, f, x, y, z))


@pytest.mark.parametrize("kz", ["1", "2", "5", "1000"])
def test_tile_kernel_z_chunks(kz, monkeypatch):
    """Every z-chunk length: the fill cursor crosses item boundaries."""
    x, y, z, f = _inputs((67, 31, 29), np.float32)
    src = PAPER_PROGRAMS["qcrit"][0]
    want = run_oracle(src, f, x, y, z)
    monkeypatch.setenv("DFG_KZ", kz)
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["variant"] == 5 and plan.info()["kz"] == min(int(kz), 29)
    assert_parity(got, want)


@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(132, 40, 33), (67, 45, 37)])
def test_two_operation_quotient(shape, T, monkeypatch):
    """on axes whose every divisor passed the check
    (fp32: exhaustive enumeration on the device; fp64: certification by
    candidate numerators) the fused kernels form d f/d axis as
    RN(num*r + RN(num*yl)); the bits equal the oracle's IEEE division and the
    three-operation correction's (TMA and general kernels)."""
    x, y, z, f = _inputs(shape, T)
    src = PAPER_PROGRAMS["qcrit"][0]
    want = run_oracle(src, f, x, y, z)
    a, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["div2_axes"] == 7
    assert_parity(a, want)
    u = np.uint32 if T == np.float32 else np.uint64
    monkeypatch.setenv("DFG_FUSED_VARIANT", "markstein")
    b, plan2, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan2.info()["div2_axes"] == 0
    assert np.array_equal(a.view(u), b.view(u))
    monkeypatch.delenv("DFG_FUSED_VARIANT")
    monkeypatch.setenv("DFG_DIV2", "0")
    c, plan3, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan3.info()["div2_axes"] == 0
    assert np.array_equal(a.view(u), c.view(u))


@pytest.mark.parametrize("T", [np.float32, np.float64])
def test_two_operation_check_rejects_one_operation(T, monkeypatch):
    """The checks are not vacuous: with yl = 0 (the one-operation RN(num*r),
    not correctly rounded for most divisors) every axis of the RT mesh is
    rejected, while on a uniform mesh with power-of-two spacing, where
    r = 1/d exactly and RN(num*r) = RN(num/d), all three are accepted."""
    monkeypatch.setenv("DFG_DIV2", "test-1op")
    src = PAPER_PROGRAMS["vortmag"][0]
    x, y, z, f = _inputs((64, 24, 20), T)
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["div2_axes"] == 0
    assert_parity(got, run_oracle(src, f, x, y, z))
    x, y, z = (synth.uniform_coords(n, dtype=T) for n in (64, 24, 20))
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["div2_axes"] == 7
    assert_parity(got, run_oracle(src, f, x, y, z))


def test_two_operation_quotient_fp64_mixed_axes():
    """fp64 x axis with jittered geometric spacing (ratio ~1.35: divisors with
    full-precision significands; with seed 1 the certificate rejects one of
    them): that axis keeps the three-operation correction, the others use two
    operations, and the mesh's choice equals the host checker's verdict on
    the same spacing table; bit-exact parity."""
    from paper_conf_sc_harrisonnmjc12_b200._dfg import dfg_div2_check
    nx, ny, nz = 120, 24, 20
    _, y, z, f = _inputs((nx, ny, nz), np.float64)
    x = np.exp(0.3 * np.arange(nx + 1) + 0.1 * np.random.default_rng(1).uniform(size=nx + 1))
    want_mask = 0
    for a, p in enumerate((x, y, z)):
        c = (p[:-1] + p[1:]) * 0.5
        i = np.arange(c.size)
        d = c[np.minimum(i + 1, c.size - 1)] - c[np.maximum(i - 1, 0)]
        want_mask |= int(dfg_div2_check(d, 0)[0].all()) << a
    assert want_mask == 6, "the geometric x axis should contain a rejected divisor"
    src = PAPER_PROGRAMS["qcrit"][0]
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["div2_axes"] == want_mask
    assert_parity(got, run_oracle(src, f, x, y, z))


@pytest.mark.parametrize("kz", ["1", "3", "7", "1000"])
def test_tma_z_chunking(kz, monkeypatch):
    """Every z-chunk length gives the same bits (halo planes at chunk ends)."""
    x, y, z, f = _inputs((64, 31, 29), np.float32)
    src = PAPER_PROGRAMS["qcrit"][0]
    want = run_oracle(src, f, x, y, z)
    monkeypatch.setenv("DFG_KZ", kz)
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.info()["variant"] == 1
    assert_parity(got, want)


@pytest.mark.parametrize("shape", [(1, 5, 6), (4, 1, 3), (8, 6, 1), (2, 2, 2), (3, 3, 3), (4, 4, 2), (1, 1, 1)])
@pytest.mark.parametrize("strategy", ["fused", "staged", "roundtrip"])
def test_degenerate_shapes(shape, strategy):
    x, y, z, f = _inputs(shape, np.float32)
    for prog in ("qcrit", "vortmag"):
        src = PAPER_PROGRAMS[prog][0]
        assert_parity(run_lib(src, f, x, y, z, strategy), run_oracle(src, f, x, y, z))


EDGE = [
    ("g = grad(u)", ("u",)),
    ("g = grad(u * u + 1)", ("u",)),
    ("c = {u, v * 2, u - v}", ("u", "v")),
    ("c = {u, v}", ("u", "v")),
    ("a = u", ("u",)),
    ("a = 2.5", ("u",)),
    ("a = u / v\nb = -a * (a >= 0.5) + (v != u)", ("u", "v")),
    ("a = if (grad(u)[0] > grad(v)[1]) then (sqrt(u * u)) else (v / u)", ("u", "v")),
    ("d = grad({u, v}[1] - u)\ne = norm(d) + d[2]", ("u", "v")),
    # power-of-two scale folding: free scalings, FMA adds
    # of unequal scales, sqrt of even / odd scales, compare / select / vector /
    # result materialisation, the exponent cap, constant x constant
    ("a = 0.5 * (u - v)\nb = a * a + 0.25 * u * (2 * v) - 4 * a / (0.125 * v)\nc = sqrt(0.25 * u * u) + b * 0.5",
     ("u", "v")),
    ("a = (u * 0.5) * (v * 0.25)\nb = if (a > 0.0625 * u) then (a / 2) else (-a * 8)\nc = {a * 2, b, sqrt(a * 4)}",
     ("u", "v")),
    ("a = u * 256 * 256 * 256 * 256 * 0.5 + v * (0.5 * 0.5)\nb = a / 256 / 256 / 256 - grad(u * 0.5)[0] * 0.25",
     ("u", "v")),
]


@pytest.mark.parametrize("src,names", EDGE)
@pytest.mark.parametrize("strategy", ["fused", "staged", "roundtrip"])
@pytest.mark.parametrize("T", [np.float32, np.float64])
def test_edge_programs(src, names, strategy, T):
    x, y, z, f = _inputs((20, 9, 7), T, names)
    assert_parity(run_lib(src, f, x, y, z, strategy), run_oracle(src, f, x, y, z))


@pytest.mark.parametrize("kind", ["rotation", "strain", "shear", "linear"])
def test_closed_forms_on_gpu(kind):
    T = np.float32
    x, y, z = (synth.dyadic_coords(12, s, T, o) for s, o in ((5, 0.5), (6, -0.25), (7, 1.0)))
    f = {k: v.astype(T) for k, v in synth.closed_form(kind, x, y, z).items()}
    progs = ["g = grad(f)"] if kind == "linear" else [PAPER_PROGRAMS["vortmag"][0], PAPER_PROGRAMS["qcrit"][0]]
    for src in progs:
        for s in ("fused", "staged"):
            assert_parity(run_lib(src, f, x, y, z, s), run_oracle(src, f, x, y, z))


@pytest.mark.parametrize("prog", ["velmag", "vortmag", "qcrit"])
@pytest.mark.parametrize("strategy", ["roundtrip", "staged", "fused"])
def test_table2_counts_measured(prog, strategy):
    """Host-interface mode reproduces Table II (L271-L285) physically."""
    import json
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table2.json")))
    x, y, z, f = _inputs((16, 12, 8), np.float32)
    src = PAPER_PROGRAMS[prog][0]
    got, plan, *_ = run_lib(src, f, x, y, z, strategy, host=True, return_plan=True)
    st = plan.stats()
    assert [st["h2d_count"], st["d2h_count"], st["kernel_count"]] == gold[prog][strategy]
    assert_parity(got, run_oracle(src, f, x, y, z))
    # device-resident (in situ) counts follow the same model
    got, plan, *_ = run_lib(src, f, x, y, z, strategy, host=False, return_plan=True)
    st = plan.stats()
    c = omodel.counts(build_dag(src, ("u", "v", "w")), strategy, "device")
    assert [st["h2d_count"], st["d2h_count"], st["kernel_count"]] == [c.h2d, c.d2h, c.kernels]


@pytest.mark.parametrize("strategy", ["roundtrip", "staged", "fused"])
@pytest.mark.parametrize("host", [True, False])
def test_memory_highwater_measured(strategy, host):
    """Fig. 2 (L112) in host mode; the ledger's high-water equals the model."""
    g = {"roundtrip": 3, "staged": 4, "fused": 5}
    x, y, z, f = _inputs((16, 8, 8), np.float32, ("a", "b", "c", "d"))
    f["d"] = f["a"] * 2
    src = "r = (a + b) * (c + d)\n"
    got, plan, *_ = run_lib(src, f, x, y, z, strategy, host=host, return_plan=True)
    N = 16 * 8 * 8 * 4
    units = omodel.footprint(build_dag(src, tuple(f)), strategy, "host" if host else "device")
    if host:
        assert units == g[strategy]
    assert plan.stats()["dev_highwater_bytes"] == units * N
    assert_parity(got, run_oracle(src, f, x, y, z))
    for prog in ("vortmag", "qcrit"):
        src = PAPER_PROGRAMS[prog][0]
        x, y, z, f = _inputs((16, 8, 8), np.float32)
        _, plan, *_ = run_lib(src, f, x, y, z, strategy, host=host, return_plan=True)
        units = omodel.footprint(build_dag(src, tuple(f)), strategy, "host" if host else "device")
        assert plan.stats()["dev_highwater_bytes"] == units * N


@pytest.mark.parametrize("host", [True, False])
@pytest.mark.parametrize("prog", ["qcrit", "vortmag"])
def test_memory_aware_staged_order(host, prog):
    """A cap below the list-order footprint but above the memory-aware one:
    the planner reorders (a valid topological order), the ledger's
    high-water equals the oracle's simulation of that order, results stay
    bit-identical."""
    src, names = PAPER_PROGRAMS[prog]
    x, y, z, f = _inputs((24, 16, 12), np.float32, names)
    dag = build_dag(src, names)
    mode = "host" if host else "device"
    N = 24 * 16 * 12 * 4
    list_units = omodel.footprint(dag, "staged", mode)
    got, plan, *_ = run_lib(src, f, x, y, z, "staged", host=host, cap=(list_units - 1) * N, return_plan=True)
    order = plan.schedule()
    assert omodel.is_topological(dag, order) and order != list(range(len(dag.filters)))
    units = omodel.footprint(dag, "staged", mode, order=order)
    assert units < list_units
    assert plan.stats()["dev_highwater_bytes"] == units * N
    assert_parity(got, run_oracle(src, f, x, y, z))
    # without a cap the paper's list order runs
    _, plan2, *_ = run_lib(src, f, x, y, z, "staged", host=host, return_plan=True)
    assert plan2.schedule() == list(range(len(dag.filters)))


@pytest.mark.parametrize("prog", ["qcrit", "intro", "vortmag"])
@pytest.mark.parametrize("host", [True, False])
@pytest.mark.parametrize("where", ["min", "mid", "below_greedy"])
def test_hybrid_spill_to_host(prog, host, where, monkeypatch):
    """DFG_HYBRID: under a cap below even the
    memory-aware staged footprint, intermediates spill to pinned host memory
    and come back when needed.  Results bit-identical to the oracle; the
    transfer events, counts, bytes and device high-water equal the oracle's
    schedule (oracle/model.py hybrid) for the memory-aware order."""
    src, names = PAPER_PROGRAMS[prog]
    shape = (40, 12, 10)
    x, y, z, f = _inputs(shape, np.float32, names)
    dag = build_dag(src, names)
    mode = "host" if host else "device"
    N = shape[0] * shape[1] * shape[2] * 4
    monkeypatch.setenv("DFG_STAGED_ORDER", "greedy")
    _, sp, *_ = run_lib(src, f, x, y, z, "staged", host=host, return_plan=True)
    greedy = sp.schedule()
    monkeypatch.delenv("DFG_STAGED_ORDER")
    fpg = omodel.footprint(dag, "staged", mode, order=greedy)
    lo = None
    for c in range(1, fpg + 1):
        try:
            omodel.hybrid(dag, mode, c, greedy)
            lo = c
            break
        except omodel.HybridInfeasible:
            pass
    hi = min(fpg, omodel.footprint(dag, "staged", mode)) - 1   # below both orders' footprints
    cap = {"min": lo, "mid": (lo + hi) // 2, "below_greedy": hi}[where]
    got, plan, *_ = run_lib(src, f, x, y, z, "hybrid", host=host, cap=cap * N, return_plan=True)
    assert_parity(got, run_oracle(src, f, x, y, z))
    assert plan.schedule() == greedy
    want = omodel.hybrid(dag, mode, cap, greedy)
    assert any(k in ("spill", "drop") for k, _ in want.events)   # the cap forces evictions
    code = lambda r: int(r[1:]) if dag.ref_filter(r) is not None else -1 - list(names).index(r)  # noqa: E731
    assert plan.transfers() == [(k, code(r)) for k, r in want.events]
    st = plan.stats()
    assert (st["h2d_count"], st["d2h_count"], st["kernel_count"]) == (want.counts.h2d, want.counts.d2h,
                                                                      want.counts.kernels)
    assert st["d2h_bytes"] == want.d2h_units * N
    assert st["dev_highwater_bytes"] == want.high * N <= cap * N
    assert st["predicted_highwater_bytes"] == want.high * N


@pytest.mark.parametrize("src,names", EDGE)
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("host", [True, False])
def test_hybrid_edge_programs(src, names, T, host):
    """Every EDGE program (vector results, bare-input and constant results,
    select, compose) under the tightest feasible cap: bit-identical results
    and the oracle's transfer events."""
    x, y, z, f = _inputs((20, 9, 7), T, names)
    dag = build_dag(src, names)
    mode = "host" if host else "device"
    N = 20 * 9 * 7 * np.dtype(T).itemsize
    fp = omodel.footprint(dag, "staged", mode)
    cap = next(c for c in range(1, fp + 2) if _feasible(dag, mode, c))
    got, plan, *_ = run_lib(src, f, x, y, z, "hybrid", host=host, cap=cap * N, return_plan=True)
    assert_parity(got, run_oracle(src, f, x, y, z))
    want = omodel.hybrid(dag, mode, cap, plan.schedule())
    code = lambda r: int(r[1:]) if dag.ref_filter(r) is not None else -1 - list(names).index(r)  # noqa: E731
    assert plan.transfers() == [(k, code(r)) for k, r in want.events]
    assert plan.stats()["dev_highwater_bytes"] == want.high * N


def _feasible(dag, mode, cap):
    try:
        omodel.hybrid(dag, mode, cap)
        return True
    except omodel.HybridInfeasible:
        return False


def test_hybrid_edges():
    """No cap: hybrid is staged (same counts, same bits).  A cap below a
    filter's working set is DFG_E_NOMEM at compile; mixed host / device
    bindings are DFG_E_UNSUPPORTED."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    src, names = PAPER_PROGRAMS["qcrit"]
    x, y, z, f = _inputs((24, 10, 8), np.float32)
    a, p1, *_ = run_lib(src, f, x, y, z, "hybrid", host=True, return_plan=True)
    b, p2, *_ = run_lib(src, f, x, y, z, "staged", host=True, return_plan=True)
    assert np.array_equal(a, b)
    for k in ("h2d_count", "d2h_count", "kernel_count", "h2d_bytes", "d2h_bytes", "dev_highwater_bytes"):
        assert p1.stats()[k] == p2.stats()[k], k
    with pytest.raises(dfg.DfgError) as e:
        run_lib(src, f, x, y, z, "hybrid", host=True, cap=4 * 24 * 10 * 8 * 4)
    assert e.value.name == "DFG_E_NOMEM"
    mesh = dfg.Mesh(x, y, z)
    keep = [torch.from_numpy(f["u"]).cuda(), f["v"], f["w"]]
    mesh.bind("u", keep[0])
    mesh.bind("v", keep[1], on_device=False)
    mesh.bind("w", keep[2], on_device=False)
    plan = dfg.Plan(mesh, src, "hybrid", 12 * 24 * 10 * 8 * 4)
    with pytest.raises(dfg.DfgError) as e:
        plan.execute(np.empty((8, 10, 24), np.float32), out_on_device=False)
    assert e.value.name == "DFG_E_UNSUPPORTED"


@pytest.mark.parametrize("shape,split", [((62, 30, 20), (2, 2, 2)), ((61, 23, 17), (2, 3, 2)),
                                         ((128, 30, 20), (2, 2, 2)), ((192, 20, 12), (1, 2, 2)),
                                         ((126, 14, 9), (1, 2, 3))])
@pytest.mark.parametrize("prog", ["qcrit", "intro", "velmag"])
@pytest.mark.parametrize("strategy", ["fused", "reference"])
@pytest.mark.parametrize("pitch", ["natural", "padded"])
def test_visit_blocks_with_ghost_shells(shape, split, prog, strategy, pitch):
    """VisIt-style multi-block (L253-L255, L315; NEXT #4): every block gets a
    one-cell ghost shell on all six faces filled from the global field (what
    VisIt's ghost exchange does); the stitched block interiors equal the
    whole-mesh result bit for bit (and the oracle).  "padded": owned cells
    from column 4 (16 bytes), rows padded past a multiple of 16 bytes
    (padding = NaN, never read), which puts blocks whose width is a multiple
    of 4 on the TMA kernel."""
    _visit_blocks(shape, split, prog, strategy, pitch)


@pytest.mark.parametrize("pitch", ["natural", "padded"])
def test_visit_blocks_several_items_per_cta(pitch):
    """27 blocks of 128 x 128 x 16 (243 tile columns for 148 persistent CTAs):
    in the one-launch multi-block kernels a CTA's items, and the ring fill
    running ahead of its consumers, cross from one block into the next."""
    _visit_blocks((384, 384, 48), (3, 3, 3), "qcrit", "fused", pitch)


def _visit_blocks(shape, split, prog, strategy, pitch):
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    if strategy == "reference" and prog == "intro":
        pytest.skip("no reference kernel for the intro expression")
    names = NAMES[prog]
    x, y, z, f = _inputs(shape, np.float32, names)
    src = PAPER_PROGRAMS[prog][0] if strategy == "fused" else prog
    whole = run_lib(src, f, x, y, z, strategy)
    if strategy == "fused":
        assert_parity(whole, run_oracle(src, f, x, y, z))
    nx, ny, nz = shape
    cuts = [np.linspace(0, n, s + 1).astype(int) for n, s in zip(shape, split)]
    got = np.empty_like(whole)
    blocks = []
    pad = {n: np.pad(a, 1, mode="edge") for n, a in f.items()}   # ghosts at the global ends are ignored
    for a in range(split[0]):
        for b in range(split[1]):
            for c in range(split[2]):
                i0, i1 = cuts[0][a], cuts[0][a + 1]
                j0, j1 = cuts[1][b], cuts[1][b + 1]
                k0, k1 = cuts[2][c], cuts[2][c + 1]
                bx = i1 - i0
                xo = 1 if pitch == "natural" else 4
                rp = bx + 2 if pitch == "natural" else (xo + bx + 1 + 3) // 4 * 4 + 4
                m = dfg.Mesh.block(x, y, z, bx, j1 - j0, k1 - k0, i0, j0, k0, ghost=1, row_pitch=rp, x_offset=xo)
                keep = []
                for n in names:
                    buf = np.full((k1 - k0 + 2, j1 - j0 + 2, rp), np.nan, np.float32)
                    buf[:, :, xo - 1:xo + bx + 1] = pad[n][k0:k1 + 2, j0:j1 + 2, i0:i1 + 2]
                    t = torch.from_numpy(buf).cuda()
                    keep.append(t)
                    m.bind(n, t)
                p = dfg.Plan(m, src, strategy)
                o = torch.empty((k1 - k0, j1 - j0, bx), device="cuda")
                p.execute(o)
                torch.cuda.synchronize()
                if pitch == "padded" and bx % 4 == 0 and prog != "velmag":
                    assert p.info()["variant"] == 1          # TMA kernel on the padded shell
                elif prog != "velmag":                       # packed shell: row copies or the cp.async ring
                    assert p.info()["variant"] == (7 if _rows_layout(rp, j1 - j0 + 2, 4, p) else 5)
                got[k0:k1, j0:j1, i0:i1] = o.cpu().numpy()
                blocks.append((p, torch.full_like(o, float("nan")), (k0, k1, j0, j1, i0, i1), m, keep,
                               p.info()["variant"]))
    assert np.array_equal(got, whole)
    # all blocks in one launch (dfg_execute_blocks): the same bits
    dfg.execute_blocks([b[0] for b in blocks], [b[1] for b in blocks])
    torch.cuda.synchronize()
    got2 = np.full_like(whole, np.nan)
    for p, o, (k0, k1, j0, j1, i0, i1), _, _, _ in blocks:
        got2[k0:k1, j0:j1, i0:i1] = o.cpu().numpy()
    assert np.array_equal(got2, whole)
    if strategy == "fused" and prog != "velmag" and len(blocks) > 1:
        tma = pitch == "padded" and all((b[2][5] - b[2][4]) % 4 == 0 for b in blocks)
        rows = all(b[5] == 7 for b in blocks)
        # one launch: TMA, row copies or the cp.async ring
        assert blocks[0][0].info()["variant"] == (4 if tma else 8 if rows else 6)


def test_memory_cap():
    """A cap below the predicted footprint fails at compile with
    DFG_E_NOMEM (the paper's failed GPU cases, L309); fused fits."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    x, y, z, f = _inputs((32, 32, 32), np.float32)
    src = PAPER_PROGRAMS["qcrit"][0]
    N = 32 ** 3 * 4
    staged_units = omodel.footprint(build_dag(src, ("u", "v", "w")), "staged", "device")
    with pytest.raises(dfg.DfgError) as e:          # below any schedule's footprint
        run_lib(src, f, x, y, z, "staged", cap=5 * N)
    assert e.value.name == "DFG_E_NOMEM"
    with pytest.raises(dfg.DfgError) as e:
        run_lib(src, f, x, y, z, "fused", cap=4 * N - 1)
    assert e.value.name == "DFG_E_NOMEM"
    got = run_lib(src, f, x, y, z, "staged", cap=staged_units * N)
    assert_parity(got, run_oracle(src, f, x, y, z))
    got = run_lib(src, f, x, y, z, "fused", cap=4 * N)
    assert_parity(got, run_oracle(src, f, x, y, z))


@pytest.mark.parametrize("G", [2, 3, 5, 12])
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("overlap", ["1", "0"])
def test_zslab_emulation_matches_single_gpu(G, T, overlap, monkeypatch):
    """G z-slabs with one ghost plane each, halo by device copies
    (dfg_mesh_link_local): the concatenated result equals the one-slab
    result bit for bit, and the halo maps equal the closed form.  With the
    overlap the exchange runs on a side stream during the
    interior planes and each slab launches 1 + (number of halo sides) kernels."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    from oracle import halo as ohalo
    monkeypatch.setenv("DFG_HALO_OVERLAP", overlap)
    shape = (64, 20, 23)
    x, y, z, f = _inputs(shape, T)
    src = PAPER_PROGRAMS["qcrit"][0]
    whole = run_lib(src, f, x, y, z)
    NZ = shape[2]
    meshes, plans, outs, keep = [], [], [], []
    for r in range(G):
        k0, nzr = dfg.dfg_partition(NZ, G, r)
        m = dfg.Mesh(x, y, z, nz_local=nzr, z_offset=k0, ghost=1)
        for n, a in f.items():
            buf = torch.zeros((nzr + 2,) + a.shape[1:], dtype=tdtype(T), device="cuda")
            buf[1:nzr + 1] = torch.from_numpy(a[k0:k0 + nzr])
            keep.append(buf)
            m.bind(n, buf)
        meshes.append(m)
        want = ohalo.halo_map(NZ, k0, nzr, r, G, shape[0], shape[1], np.dtype(T).itemsize)
        got = m.halo_map()
        assert got[2:8] == want[2:8] and got[10:] == want[10:]
    for r in range(G - 1):
        dfg.dfg_mesh_link_local(meshes[r].handle, meshes[r + 1].handle)
    for r, m in enumerate(meshes):
        p = dfg.Plan(m, src, "fused")
        o = torch.empty((m.nz, shape[1], shape[0]), dtype=tdtype(T), device="cuda")
        p.execute(o)
        plans.append(p)
        outs.append(o)
    torch.cuda.synchronize()
    got = torch.cat(outs).cpu().numpy()
    assert np.array_equal(got, whole)
    assert_parity(got, run_oracle(src, f, x, y, z))       # the stitched slabs against the oracle itself
    for r, p in enumerate(plans):
        sides = (r > 0) + (r < G - 1)
        st = p.stats()
        assert st["halo_bytes"] == 3 * sides * shape[0] * shape[1] * np.dtype(T).itemsize
        assert st["kernel_count"] == (1 + sides if overlap == "1" and meshes[r].nz >= 3 else 1)


def test_config2_192_all_strategies():
    """Config 2: 192^3, VelMag + VortMag + Q, all three strategies."""
    x, y, z, f = _inputs((192, 192, 192), np.float32)
    for prog in ("velmag", "vortmag", "qcrit"):
        src = PAPER_PROGRAMS[prog][0]
        want = run_oracle(src, f, x, y, z)
        for s in ("fused", "staged", "roundtrip"):
            assert_parity(run_lib(src, f, x, y, z, s), want)


def _windows(shape, rng, n_random=6, w=10):
    nx, ny, nz = shape
    wins = []
    for cz in (0, nz - w):
        for cy in (0, ny - w):
            for cx in (0, nx - w):
                wins.append((cz, cy, cx))
    for _ in range(n_random):
        wins.append((int(rng.integers(0, nz - w)), int(rng.integers(0, ny - w)), int(rng.integers(0, nx - w))))
    return [(k, k + w, j, j + w, i, i + w) for k, j, i in wins]


def _sampled_parity(src, names, shape, T, strategy="fused", seed=0):
    """Full-size run on the GPU; oracle on sampled windows (8 corners + random
    interior), each evaluated with global indices and global coordinates."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    nx, ny, nz = shape
    x, y, z = synth.rt_coords(nx, ny, nz, T)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    bufs = {}
    for n, comp in zip(names, "uvw"):
        bufs[n] = synth.rt_velocity(comp, x64, y64, z64, dtype=tdtype(T), device="cuda")
        mesh.bind(n, bufs[n])
    plan = dfg.Plan(mesh, src, strategy)
    out = torch.empty((nz, ny, nx), dtype=tdtype(T), device="cuda")
    plan.execute(out)
    torch.cuda.synchronize()
    dag = build_dag(src, names, "f32" if T == np.float32 else "f64")
    rng = np.random.default_rng(seed)
    for (k0, k1, j0, j1, i0, i1) in _windows(shape, rng):
        e = lambda a, b, n: (max(a - 1, 0), min(b + 1, n))
        K0, K1 = e(k0, k1, nz)
        J0, J1 = e(j0, j1, ny)
        I0, I1 = e(i0, i1, nx)
        win = {n: bufs[n][K0:K1, J0:J1, I0:I1].cpu().numpy() for n in names}
        res, valid = oev.evaluate(dag, win, oev.MeshWindow(x, y, z, i0=I0, j0=J0, k0=K0))
        sl = (slice(k0 - K0, k1 - K0), slice(j0 - J0, j1 - J0), slice(i0 - I0, i1 - I0))
        assert valid[sl].all()
        got = out[k0:k1, j0:j1, i0:i1].cpu().numpy()
        assert_parity(got, res[sl])
    return plan


def test_config4_1024_fused_q_sampled():
    """Config 4 at 1 GPU (the bench workload): 1024^3 fused Q, fp32."""
    plan = _sampled_parity(PAPER_PROGRAMS["qcrit"][0], ("u", "v", "w"), (1024, 1024, 1024), np.float32)
    assert plan.info()["variant"] == 1


@pytest.mark.parametrize("prog", PROGS)
@pytest.mark.parametrize("T", [np.float32, np.float64])
def test_config5_768_sweep_sampled(prog, T):
    """Config 5: 768^3 complexity sweep, fp32 and fp64, fused."""
    _sampled_parity(PAPER_PROGRAMS[prog][0], NAMES[prog], (768, 768, 768), T)


def test_config3_512_staged_caps():
    """Config 3: 512^3 Q, staged under device-memory caps vs fused."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    GiB = 1 << 30
    n = 512
    x, y, z = synth.rt_coords(n, n, n, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    bufs = {c: synth.rt_velocity(c, x64, y64, z64, dtype=torch.float32, device="cuda") for c in "uvw"}
    for c, b in bufs.items():
        mesh.bind(c, b)
    src = PAPER_PROGRAMS["qcrit"][0]
    fused = dfg.Plan(mesh, src, "fused", 4 * GiB)
    o1 = torch.empty((n, n, n), device="cuda")
    fused.execute(o1)
    units = omodel.footprint(build_dag(src, ("u", "v", "w")), "staged", "device")
    need = units * n ** 3 * 4
    for cap in (8 * GiB, 4 * GiB):
        assert need > cap
        with pytest.raises(dfg.DfgError) as e:
            dfg.Plan(mesh, src, "staged", cap)
        assert e.value.name == "DFG_E_NOMEM"
    staged = dfg.Plan(mesh, src, "staged", 16 * GiB)
    o2 = torch.empty((n, n, n), device="cuda")
    staged.execute(o2)
    torch.cuda.synchronize()
    assert torch.equal(o1, o2)
    assert staged.stats()["dev_highwater_bytes"] == need


@pytest.mark.parametrize("planes", ["1", "3", "5", "64"])
@pytest.mark.parametrize("prog", ["qcrit", "intro", "velmag"])
@pytest.mark.parametrize("shape", [(68, 20, 23), (67, 9, 11), (66, 8, 13)])
def test_streamed_strategy(planes, prog, shape, monkeypatch):
    """Streamed fusion (z-chunks through a 3-slot ring, overlapped copies):
    any chunk height gives the oracle's bits, host or pinned buffers."""
    monkeypatch.setenv("DFG_STREAM_PLANES", planes)
    x, y, z, f = _inputs(shape, np.float32, NAMES[prog])
    src = PAPER_PROGRAMS[prog][0]
    want = run_oracle(src, f, x, y, z)
    got, plan, *_ = run_lib(src, f, x, y, z, "streamed", host=True, return_plan=True)
    assert_parity(got, want)
    st = plan.stats()
    nch = -(-shape[2] // min(int(planes), shape[2]))
    assert st["kernel_count"] == nch
    assert st["d2h_count"] == nch
    # device-resident everything: identical to fusion
    assert_parity(run_lib(src, f, x, y, z, "streamed", host=False), want)


@pytest.mark.parametrize("planes", ["4", "12"])
@pytest.mark.parametrize("prog", ["velmag", "qcrit"])
def test_streamed_odd_plane_vector_offsets(planes, prog, monkeypatch):
    """a chunk of 4 or 12 planes of a 67 x 9 plane holds a whole
    number of 16-byte vectors, but its first owned plane sits one odd plane
    (the ghost) into the slot: the point-wise kernel must not take its
    16-byte path there (it would load misaligned)."""
    monkeypatch.setenv("DFG_STREAM_PLANES", planes)
    shape = (67, 9, 12)
    x, y, z, f = _inputs(shape, np.float32, NAMES[prog])
    src = PAPER_PROGRAMS[prog][0]
    got = run_lib(src, f, x, y, z, "streamed", host=True)
    assert_parity(got, run_oracle(src, f, x, y, z))


def test_streamed_pinned_large(monkeypatch):
    """Streamed at 256^3 with pinned host buffers equals fused on the device."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    monkeypatch.setenv("DFG_STREAM_PLANES", "32")
    n = 256
    x, y, z = synth.rt_coords(n, n, n, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    dev = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    host = {c: t.cpu().pin_memory() for c, t in dev.items()}
    src = PAPER_PROGRAMS["qcrit"][0]
    m1 = dfg.Mesh(x, y, z)
    for c, t in dev.items():
        m1.bind(c, t)
    o1 = torch.empty((n, n, n), device="cuda")
    dfg.Plan(m1, src, "fused").execute(o1)
    m2 = dfg.Mesh(x, y, z)
    for c, t in host.items():
        m2.bind(c, t, on_device=False)
    p2 = dfg.Plan(m2, src, "streamed")
    o2 = torch.empty((n, n, n)).pin_memory()
    for _ in range(2):
        p2.execute(o2, out_on_device=False)
    assert torch.equal(o1.cpu(), o2)
    st = p2.stats()
    assert st["dev_highwater_bytes"] < 4 * n ** 3 * 4      # bounded ring, below fused's footprint


@pytest.mark.parametrize("prog", ["velmag", "vortmag", "qcrit"])
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(64, 40, 33), (67, 21, 9)])
def test_reference_kernels(prog, T, shape):
    """Hand-written reference kernels (L243): same I/O as fusion, fewer flops;
    they agree with the oracle within the floating-point tolerance (R15),
    not bit for bit (one rounding more per derivative, FMA, Q = -tr(J^2)/2)."""
    x, y, z, f = _inputs(shape, T)
    want = run_oracle(PAPER_PROGRAMS[prog][0], f, x, y, z)
    got, plan, *_ = run_lib(prog, f, x, y, z, "reference", return_plan=True)
    assert_parity(got, want, exact=False)
    assert plan.stats()["kernel_count"] == 1
    assert "dfg-dag v1" in plan.dag()
    # unknown quantities are rejected
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    with pytest.raises(dfg.DfgError):
        run_lib("intro", f, x, y, z, "reference")


@pytest.mark.parametrize("prog", PROGS)
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(132, 40, 33), (67, 45, 37)])
def test_fast_variant_within_tolerance(prog, T, shape, monkeypatch):
    """DFG_FUSED_VARIANT=fast (derivative = num * RN(1/d), FMA allowed in the
    quotient only) is not bit-identical to the literal network, but stays within
    the R15 bound (1e-5 / 1e-12 normwise) on both kernels (TMA and general)."""
    x, y, z, f = _inputs(shape, T, NAMES[prog])
    src = PAPER_PROGRAMS[prog][0]
    want = run_oracle(src, f, x, y, z)
    monkeypatch.setenv("DFG_FUSED_VARIANT", "fast")
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert_parity(got, want, exact=False)


@pytest.mark.parametrize("rpw", ["1", "2", "4"])
@pytest.mark.parametrize("T", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(200, 37, 21), (132, 40, 33), (8, 70, 9)])
def test_tma_rows_per_warp(rpw, T, shape, monkeypatch):
    """Every TMA tile shape (1, 2 or 4 rows per consumer warp: tiles of
    32*VEC/rpw x 15*rpw cells) gives the oracle's bits, ragged x and y tiles
    included."""
    x, y, z, f = _inputs(shape, T)
    src = PAPER_PROGRAMS["qcrit"][0]
    want = run_oracle(src, f, x, y, z)
    monkeypatch.setenv("DFG_RPW", rpw)
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    info = plan.info()
    assert info["variant"] == 1 and info["rows_per_warp"] == int(rpw)
    vec = 4 if T == np.float32 else 2
    assert info["tile_w"] == 32 * vec // int(rpw) and info["tile_h"] == info["rows_per_warp"] * 15
    assert_parity(got, want)


def test_tile_shape_choice():
    """Narrow meshes take several rows per warp (no idle lanes in a ragged x
    tile); the 1024-wide bench mesh keeps one row per warp; 192^3 (config 2)
    takes 12 warps x 2 rows (8 whole tiles of 24 rows), bit-exact."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    for n, nz, want in ((192, 192, 2), (1024, 64, 1)):
        x, y, z = synth.rt_coords(n, n, nz, np.float32)
        mesh = dfg.Mesh(x, y, z)
        fields = [torch.zeros((nz, n, n), device="cuda") for _ in range(3)]
        for c, t in zip("uvw", fields):
            mesh.bind(c, t)
        plan = dfg.Plan(mesh, PAPER_PROGRAMS["qcrit"][0], "fused")
        assert plan.info()["rows_per_warp"] == want, (n, plan.info())
        if n == 192:
            assert plan.info()["tile_h"] == 24, plan.info()
        plan.close()


@pytest.mark.parametrize("T", [np.float32, np.float64])
def test_staged_graph_replay(T, monkeypatch):
    """Device-resident staged executes run as a captured CUDA graph (every
    filter's kernel, allocation and free): replays give the oracle's bits,
    the Table II kernel count per execute, and a re-capture when a binding
    or the output changes; DFG_GRAPH=0 (plain stream launches) gives the
    same bits."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    shape = (48, 20, 17)
    x, y, z, f = _inputs(shape, T)
    src = PAPER_PROGRAMS["qcrit"][0]
    mesh = dfg.Mesh(x, y, z)
    dev = {k: torch.from_numpy(v).cuda() for k, v in f.items()}
    for k, v in dev.items():
        mesh.bind(k, v)
    plan = dfg.Plan(mesh, src, "staged")
    out = torch.empty(shape[::-1], dtype=tdtype(T), device="cuda")
    want = run_oracle(src, f, x, y, z)
    for _ in range(3):
        out.fill_(float("nan"))
        plan.execute(out)
        torch.cuda.synchronize()
        assert_parity(out.cpu().numpy(), want)
    st = plan.stats()
    assert st["executes"] == 3 and st["kernel_count"] == 3 * 67
    # the ledger high-water survives a stats reset on the replay path (row a10)
    units = omodel.footprint(build_dag(src, ("u", "v", "w")), "staged", "device")
    elem = int(np.prod(shape)) * np.dtype(T).itemsize
    assert st["dev_highwater_bytes"] == units * elem
    plan.reset_stats()
    assert plan.stats()["dev_highwater_bytes"] == 0
    plan.execute(out)
    torch.cuda.synchronize()
    st = plan.stats()
    assert st["executes"] == 1 and st["kernel_count"] == 67
    assert st["dev_highwater_bytes"] == units * elem
    # new data under the same pointer: the replay reads it
    f2 = {k: (v * 2).astype(T) for k, v in f.items()}
    for k in dev:
        dev[k].copy_(torch.from_numpy(f2[k]))
    plan.execute(out)
    torch.cuda.synchronize()
    want2 = run_oracle(src, f2, x, y, z)
    assert_parity(out.cpu().numpy(), want2)
    # a new binding and a new output: re-captured
    u2 = torch.from_numpy(f["u"]).cuda()
    mesh.bind("u", u2)
    out2 = torch.empty_like(out)
    plan.execute(out2)
    torch.cuda.synchronize()
    f3 = dict(f2, u=f["u"])
    assert_parity(out2.cpu().numpy(), run_oracle(src, f3, x, y, z))
    monkeypatch.setenv("DFG_GRAPH", "0")
    out3 = torch.empty_like(out)
    plan.execute(out3)
    torch.cuda.synchronize()
    assert torch.equal(out2, out3)


@pytest.mark.parametrize("seed", range(4))
def test_differential_fuzz_fused(seed, monkeypatch):
    """Random well-formed programs (the parser fuzz generator of
    test_lib_host: arithmetic, sqrt, unary minus, grad3d / decompose, norm,
    compose, if / comparisons, constants incl. 1e39 and 0) through the
    generated fused kernel -- value numbering, scale folding and the
    verified two-operation quotient included -- on TMA-aligned, row-class
    and ragged (cp.async ring) meshes in fp32 and fp64: the oracle's bits on
    every cell of the exactness domain (oracle.evaluate.in_range_mask), and
    on every cell with DFG_FUSED_VARIANT=ieee."""
    import random
    from test_lib_host import _rand_program
    from oracle.lang import DfgError as OracleError
    rng = random.Random(1000 + seed)
    n_run = 0
    for it in range(24):
        src = _rand_program(rng)
        T = np.float32 if it % 2 == 0 else np.float64
        shape = ((24, 13, 9), (23, 13, 9), (22, 8, 9))[it % 3]
        x, y, z, f = _inputs(shape, T)
        try:
            want = run_oracle(src, f, x, y, z)
        except OracleError:
            continue
        dag = build_dag(src, ("u", "v", "w"), "f32" if T == np.float32 else "f64")
        mask = oev.in_range_mask(dag, f, x, y, z)
        if want.ndim == 4:
            mask = np.broadcast_to(mask[..., None], want.shape)
        monkeypatch.setenv("DFG_FUSED_VARIANT", "ieee")
        got = run_lib(src, f, x, y, z, "fused")
        assert _same_bits(got, want), ("ieee", src)
        monkeypatch.delenv("DFG_FUSED_VARIANT")
        got = run_lib(src, f, x, y, z, "fused")
        assert _same_bits(got, want, mask), ("exact", src)
        n_run += 1
    assert n_run >= 12


def _same_bits(got, want, where=None):
    """Bit-for-bit equality except NaN payloads (x86 and the GPU produce
    different default NaNs): NaN positions equal, every other value -- signed
    zeros and infinities included -- equal as bits."""
    u = np.uint32 if got.dtype == np.float32 else np.uint64
    if where is None:
        where = np.ones(got.shape, dtype=bool)
    gn, wn = np.isnan(got) & where, np.isnan(want) & where
    if not np.array_equal(gn, wn):
        return False
    keep = where & ~wn
    return bool(np.array_equal(got.view(u)[keep], want.view(u)[keep]))


def _extreme_fields(T, shape):
    """RT-like velocity with three planted regions: u = 2^64 y (fp32; 2^600
    y in fp64) in the low z quarter -- the literal network stays finite but
    a power-of-two-folded square of (du[1] + dv[0]) would be 4x larger --
    w = 2^-70 x (2^-1000 x) in the high quarter, whose squares underflow to
    subnormals, and a few subnormal / infinite / NaN input cells."""
    x, y, z = (synth.dyadic_coords(n, s, T) for n, s in zip(shape, (5, 6, 7)))
    _, _, _, f = _inputs(shape, T)
    big, tiny = (2.0 ** 64, 2.0 ** -70) if T == np.float32 else (2.0 ** 600, 2.0 ** -1000)
    yc, xc = synth.centres64(y), synth.centres64(x)
    nz = shape[2]
    f["u"][: nz // 4] = (big * yc)[None, :, None].astype(T)
    f["w"][3 * nz // 4:] = (tiny * xc)[None, None, :].astype(T)
    f["v"][nz // 2, 3, 5] = np.finfo(T).tiny / 8          # subnormal input
    f["v"][nz // 2, 5, 9] = np.inf
    f["u"][nz // 2 + 1, 7, 2] = np.nan
    return x, y, z, f


@pytest.mark.parametrize("T", [np.float32, np.float64])
def test_exactness_domain_extreme_values(T, monkeypatch):
    """VERDICT r1 (parity scope): the contract of each arithmetic variant on
    inputs whose intermediates overflow or go subnormal.  dfg_plan_arith
    reports the domain; IEEE-only plans (the staged kernels, and the fused
    kernel with DFG_FUSED_VARIANT=ieee) equal the oracle bit for bit on
    EVERY cell, NaN / Inf positions and signed zeros included; the default
    fused kernel equals it on every cell of oracle.evaluate.in_range_mask
    (DESIGN.md section 5), and the planted regions do leave that domain."""
    shape = (40, 24, 20)
    x, y, z, f = _extreme_fields(T, shape)
    src = PAPER_PROGRAMS["qcrit"][0]
    want = run_oracle(src, f, x, y, z)
    dag = build_dag(src, ("u", "v", "w"), "f32" if T == np.float32 else "f64")
    mask = oev.in_range_mask(dag, f, x, y, z)
    assert 0.2 < mask.mean() < 0.9, mask.mean()
    assert not np.isfinite(want).all()
    for strategy in ("staged", "roundtrip"):
        got, plan, *_ = run_lib(src, f, x, y, z, strategy, return_plan=True)
        assert plan.arith()["exact_domain"] == "all_inputs"
        assert _same_bits(got, want), strategy
    monkeypatch.setenv("DFG_FUSED_VARIANT", "ieee")
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    assert plan.arith() == {"div_mode": "ieee", "fold": False, "div2_axes": 0, "exact_domain": "all_inputs"}
    assert _same_bits(got, want)
    monkeypatch.delenv("DFG_FUSED_VARIANT")
    got, plan, *_ = run_lib(src, f, x, y, z, return_plan=True)
    ar = plan.arith()
    assert ar["exact_domain"] == "normal_range" and ar["fold"] and ar["div_mode"] == "exact_normal"
    assert _same_bits(got, want, mask)


def test_visit_blocks_mixed_tile_shapes():
    """Blocks whose row counts make the planner pick different tiles (28 rows:
    14 warps; 24 rows: 12 x 2, DFG's choose_rows_tile) compile different
    kernels, so dfg_execute_blocks cannot batch them into one launch: it runs
    them one by one (row-class kernel each), with the same bits as the whole
    mesh and the oracle."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    shape = (67, 52, 10)
    x, y, z, f = _inputs(shape, np.float32)
    src = PAPER_PROGRAMS["qcrit"][0]
    whole = run_lib(src, f, x, y, z, "fused")
    assert_parity(whole, run_oracle(src, f, x, y, z))
    pad = {n: np.pad(a, 1, mode="edge") for n, a in f.items()}
    rp, xo, nx, nz = 70, 1, 67, 10
    plans, outs, keep, cuts = [], [], [], [(0, 28), (28, 52)]
    for j0, j1 in cuts:
        m = dfg.Mesh.block(x, y, z, nx, j1 - j0, nz, 0, j0, 0, ghost=1, row_pitch=rp, x_offset=xo)
        for n in "uvw":
            buf = np.full((nz + 2, j1 - j0 + 2, rp), np.nan, np.float32)
            buf[:, :, xo - 1:xo + nx + 1] = pad[n][0:nz + 2, j0:j1 + 2, 0:nx + 2]
            t = torch.from_numpy(buf).cuda()
            keep.append(t)
            m.bind(n, t)
        keep.append(m)
        plans.append(dfg.Plan(m, src, "fused"))
        outs.append(torch.full((nz, j1 - j0, nx), float("nan"), device="cuda"))
    assert plans[0].kernel_source() != plans[1].kernel_source()
    dfg.execute_blocks(plans, outs)
    torch.cuda.synchronize()
    got = np.empty_like(whole)
    for (j0, j1), p, o in zip(cuts, plans, outs):
        assert p.info()["variant"] == 7
        got[:, j0:j1, :] = o.cpu().numpy()
    assert np.array_equal(got, whole)
