"""Pins of the data-layout readings (R17 / SURVEY S3, S5) against
Table I (L206-L221), and the 3-D point-array converter of the C ABI."""

import json
import math
import os

import numpy as np
import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden", "table1.json")
LIB = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_sc_harrisonnmjc12_b200", "libdfg.so")


def _fmt(b):
    mib = b / 2 ** 20
    return f"{math.ceil(mib)} MB" if mib < 1000 else f"{math.ceil(b / 2 ** 30 * 10) / 10:.1f} GB"


def _size(nz, cells, field_bytes, point_bytes_per_point, coords3d=True):
    pts = 193 * 193 * (nz + 1) if coords3d else (193 + 193 + nz + 1)
    return 3 * field_bytes * cells + (3 * point_bytes_per_point if coords3d else point_bytes_per_point) * pts


def test_table1_cells_and_sizes():
    """u, v, w cell-centred fp32 (12 B/cell) + x, y, z as full 3-D fp32 point
    arrays (12 B/point) reproduce all 12 data sizes; fp64 fields or 1-D
    coordinate arrays do not."""
    rows = json.load(open(GOLD))["rows"]
    hit = {"fp32_3d": 0, "fp64_3d": 0, "fp32_1d": 0}
    for nz, cells, txt in rows:
        assert cells == 192 * 192 * nz
        hit["fp32_3d"] += _fmt(_size(nz, cells, 4, 4)) == txt
        hit["fp64_3d"] += _fmt(_size(nz, cells, 8, 4)) == txt
        hit["fp32_1d"] += _fmt(_size(nz, cells, 4, 4, coords3d=False)) == txt
    assert hit["fp32_3d"] == 12
    assert hit["fp64_3d"] < 12 and hit["fp32_1d"] < 12


@pytest.mark.skipif(not os.path.exists(LIB), reason="libdfg.so not built")
@pytest.mark.parametrize("T", [np.float32, np.float64])
def test_points3d_to_axes(T):
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    import synth
    x, y, z = synth.rt_coords(7, 5, 4, T)
    Z3, Y3, X3 = np.meshgrid(z, y, x, indexing="ij")
    ax = dfg.dfg_points3d_to_axes(X3, Y3, Z3)
    for a, b in zip(ax, (x, y, z)):
        assert a.dtype == T and np.array_equal(a, b)
    X3 = X3.copy()
    X3[2, 3, 1] = np.nextafter(X3[2, 3, 1], T(2))        # not rectilinear any more
    with pytest.raises(dfg.DfgError) as e:
        dfg.dfg_points3d_to_axes(X3, Y3, Z3)
    assert e.value.name == "DFG_E_INVALID"
