"""Helpers shared by the GPU parity tests: run a program through the C ABI
(device-resident or host-pointer mode) and compare with the oracle."""

from __future__ import annotations

import numpy as np
import torch

from oracle import evaluate as oev
from oracle.lang import build_dag


def tdtype(T):
    return torch.float32 if np.dtype(T) == np.float32 else torch.float64


def run_lib(expr, fields: dict, x, y, z, strategy="fused", host=False, cap=0, return_plan=False, mesh_kw=None):
    """fields: name -> numpy array [nz, ny, nx] (T).  Returns numpy result."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    T = x.dtype
    mesh = dfg.Mesh(x, y, z, **(mesh_kw or {}))
    keep = {}
    for n, a in fields.items():
        if host:
            buf = np.ascontiguousarray(a)
        else:
            buf = torch.from_numpy(np.ascontiguousarray(a)).cuda()
        keep[n] = buf
        mesh.bind(n, buf, on_device=not host)
    plan = dfg.Plan(mesh, expr, strategy, cap)
    width = plan.info()["width"]
    shape = (mesh.nz, mesh.ny, mesh.nx) + ((4,) if width == 4 else ())
    if host:
        out = np.empty(shape, dtype=T)
        plan.execute(out, out_on_device=False)
        res = out
    else:
        out = torch.empty(shape, dtype=tdtype(T), device="cuda")
        plan.execute(out)
        torch.cuda.synchronize()
        res = out.cpu().numpy()
    if return_plan:
        return res, plan, mesh, keep
    return res


def run_oracle(expr, fields, x, y, z):
    dt = "f32" if x.dtype == np.float32 else "f64"
    dag = build_dag(expr, tuple(fields), dt)
    return oev.evaluate_full(dag, {k: np.ascontiguousarray(v) for k, v in fields.items()}, x, y, z)


def normwise(got, want):
    fin = np.isfinite(want)
    scale = np.abs(want[fin]).max() if fin.any() else 0.0
    err = np.abs(got[fin].astype(np.float64) - want[fin].astype(np.float64)).max() if fin.any() else 0.0
    return err / scale if scale > 0 else err


def assert_parity(got, want, exact=True, tol=None):
    """NaN / Inf positions and signs must agree; finite values bit-equal
    (exact) or within the normwise tolerance (R15)."""
    assert got.shape == want.shape, (got.shape, want.shape)
    assert got.dtype == want.dtype
    assert np.array_equal(np.isnan(got), np.isnan(want)), "NaN positions differ"
    assert np.array_equal(np.isposinf(got), np.isposinf(want)), "+Inf positions differ"
    assert np.array_equal(np.isneginf(got), np.isneginf(want)), "-Inf positions differ"
    fin = np.isfinite(want)
    if exact:
        bad = np.count_nonzero(got[fin] != want[fin])
        assert bad == 0, f"{bad} of {fin.sum()} finite values differ; normwise {normwise(got, want):.3e}"
    else:
        if tol is None:
            tol = 1e-5 if got.dtype == np.float32 else 1e-12
        assert normwise(got, want) <= tol
