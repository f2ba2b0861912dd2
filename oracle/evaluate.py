"""Oracle: literal evaluation of a dataflow network over whole arrays.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Every primitive is applied to whole arrays, one filter at a time, in network
order -- exactly the "staged" picture of the paper (L96) with no fusion, no
blocking and no reordering.  Every operation is rounded to the field type T
(numpy float32 / float64 ufuncs: IEEE add, sub, mul, div and sqrt, correctly
rounded, no contraction).

Primitives (L86 lists add, sub, mult, sqrt, decompose and the 3-D rectilinear
gradient; div, neg, the comparisons, select and compose are the extensions
the intro expression L19 and north_star need -- DESIGN.md R3):

* add/sub/mult/div/neg/sqrt -- IEEE in T.
* const   -- broadcast of the literal parsed to T (L76, L103).
* gt/lt/ge/le/eq/ne -- T(1) or T(0); NaN compares false (R7).
* select(c, a, b) -- (c != 0) ? a : b; both branches evaluated (R7).
* decompose(v, k) -- lane k of a vector value (L74, L105).
* compose(a, b, ...) -- vector of the scalars (R3).
* grad3d(f, dims, x, y, z) -- reading R1: with cell-centred f
  (L154, L223) and point coordinates p[0..n] per axis (L165, L225), the
  centre of cell i is c_i = (p_i + p_{i+1}) * T(0.5); then with
  ip = min(i+1, n-1), im = max(i-1, 0):
      d f / d axis at i = (f[ip] - f[im]) / (c[ip] - c[im])      (in T)
  i.e. a central difference over the neighbour-centre distance inside the
  mesh and a one-sided difference at the two mesh ends; 0 when n == 1.
  Components: [0] = d/dx, [1] = d/dy, [2] = d/dz (pinned by Eq. 1 vs
  Fig. 3B: w_x = dw[1] - dv[2] = dw/dy - dv/dz, L136 / L168).

Windows.  ``evaluate`` works on a rectangular window of the global mesh
(origin (k0, j0, i0), the shape of the input arrays).  Gradients use global
indices for the clamping and global centre coordinates for the spacing, so a
window evaluated alone gives the same values as the whole mesh wherever the
stencil neighbours lie inside the window; ``valid`` marks those cells.  This
is what the sampled parity checks at full size and the z-slab checks use.
"""

from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .lang import Dag, MESH_NAMES


@dataclass
class MeshWindow:
    """Global point coordinates (T) and the window origin."""
    x: np.ndarray          # nx+1 point coordinates, dtype T
    y: np.ndarray          # ny+1
    z: np.ndarray          # NZ+1 (global)
    i0: int = 0
    j0: int = 0
    k0: int = 0


def centres(p: np.ndarray) -> np.ndarray:
    """c_i = (p_i + p_{i+1}) * 0.5 in T (reading R1; cell-centred data L154)."""
    T = p.dtype.type
    return (p[:-1] + p[1:]) * T(0.5)


def grad3d(f: np.ndarray, mw: MeshWindow):
    """Gradient of a cell-centred scalar window f[k, j, i]; returns
    (g[..., 3], valid) -- see module docstring (reading R1)."""
    T = f.dtype.type
    comps = []
    valid = np.ones(f.shape, dtype=bool)
    for axis, p, o in ((2, mw.x, mw.i0), (1, mw.y, mw.j0), (0, mw.z, mw.k0)):
        n = len(p) - 1
        w = f.shape[axis]
        if n == 1:
            comps.append(np.zeros(f.shape, dtype=f.dtype))
            continue
        c = centres(p)
        g = o + np.arange(w)                       # global indices in window
        ip = np.minimum(g + 1, n - 1)
        im = np.maximum(g - 1, 0)
        ok = (ip - o < w) & (im - o >= 0)
        f_ip = np.take(f, np.clip(ip - o, 0, w - 1), axis=axis)
        f_im = np.take(f, np.clip(im - o, 0, w - 1), axis=axis)
        num = f_ip - f_im                          # T
        den = c[ip] - c[im]                        # T
        shape = [1, 1, 1]
        shape[axis] = w
        with np.errstate(divide="ignore", invalid="ignore"):
            comps.append(num / den.reshape(shape))
        valid &= ok.reshape(shape)
    assert all(cp.dtype == f.dtype for cp in comps)
    out = np.stack(comps, axis=-1)
    assert out.dtype.type is T
    return out, valid


_BINARY = {
    "add": np.add, "sub": np.subtract, "mult": np.multiply, "div": np.divide,
}
_CMP = {
    "gt": np.greater, "lt": np.less, "ge": np.greater_equal,
    "le": np.less_equal, "eq": np.equal, "ne": np.not_equal,
}


def evaluate(dag: Dag, inputs: dict, mw: MeshWindow, on_value=None):
    """Evaluate every filter in list order over whole arrays.

    inputs: name -> array[k, j, i] of dtype T (all the same window shape).
    Returns (result, valid): result is [k, j, i] for a scalar program or
    [k, j, i, 4] (lanes beyond the used width are 0) for a vector program.
    on_value(k, filter, value, args), if given, sees every filter's value
    and its (non-mesh) argument values (an observer: it cannot change the
    evaluation).
    """
    T = np.float32 if dag.dtype == "f32" else np.float64
    shape = None
    for name, a in inputs.items():
        assert a.dtype == T, (name, a.dtype)
        shape = a.shape if shape is None else shape
        assert a.shape == shape, "all inputs must share the window shape"
    assert shape is not None, "at least one input field is required"
    vals: dict = {}
    valid = np.ones(shape, dtype=bool)

    def get(ref):
        if ref in vals:
            return vals[ref]
        return inputs[ref]

    with np.errstate(all="ignore"):
        for k, f in enumerate(dag.filters):
            ref = f"f{k}"
            a = [get(r) for r in f.inputs if r not in MESH_NAMES]
            if f.op == "const":
                v = np.full(shape, f.attr, dtype=T)
            elif f.op in _BINARY:
                v = _BINARY[f.op](a[0], a[1])
            elif f.op in _CMP:
                v = np.where(_CMP[f.op](a[0], a[1]), T(1), T(0)).astype(T)
            elif f.op == "neg":
                v = np.negative(a[0])
            elif f.op == "sqrt":
                v = np.sqrt(a[0])
            elif f.op == "select":
                v = np.where(a[0] != 0, a[1], a[2])
            elif f.op == "decompose":
                v = a[0][..., f.attr]
            elif f.op == "compose":
                v = np.stack(a, axis=-1)
            elif f.op == "grad3d":
                v, ok = grad3d(a[0], mw)
                valid &= ok
            else:
                raise AssertionError(f.op)
            assert v.dtype == T, (f.op, v.dtype)
            vals[ref] = v
            if on_value is not None:
                on_value(k, f, v, a)
    res = get(dag.result)
    if res.ndim == 4:
        pad = np.zeros(shape + (4,), dtype=T)
        pad[..., : res.shape[-1]] = res
        res = pad
    else:
        res = res.copy()
    return res, valid


def evaluate_full(dag: Dag, inputs: dict, x, y, z):
    """Whole-mesh evaluation (window = mesh); returns the result array."""
    res, valid = evaluate(dag, inputs, MeshWindow(x, y, z))
    assert valid.all()
    return res


def in_range_mask(dag: Dag, inputs: dict, x, y, z):
    """Whole mesh: True at the cells where every input value, every grad3d
    numerator f[ip] - f[im] (each axis; and none of these is -0) and every
    value of the literal network (each filter, each lane) is zero or has a
    magnitude in [2^(emin + 2p), 2^(emax - p)] of T (fp32: [2^-78, 2^104], fp64:
    [2^-916, 2^970]; p = significand bits) -- finite, normal, with 2^p of
    headroom above and 2^(2p) below.  This is the sufficient condition of
    DESIGN.md section 5 under which the default fused kernel's reciprocal
    quotients and power-of-two scale folding round exactly like the literal
    network; it is written as a plain definition over the oracle's values."""
    T = np.float32 if dag.dtype == "f32" else np.float64
    fi = np.finfo(T)
    p = fi.nmant + 1
    lo = np.ldexp(1.0, fi.minexp + 2 * p)
    hi = np.ldexp(1.0, fi.maxexp - 1 - p)

    def ok(a):
        a = np.abs(a.astype(np.float64))
        return (a == 0) | ((a >= lo) & (a <= hi))

    shape = next(iter(inputs.values())).shape
    mask = np.ones(shape, dtype=bool)
    for a in inputs.values():
        mask &= ok(a)

    def numerators(f):
        # and no numerator is -0: the two-operation quotient's low product
        # takes the sign of yl, so -0 / d may come out +0
        out = np.ones(shape, dtype=bool)
        for axis in range(3):
            n = f.shape[axis]
            if n == 1:
                continue
            i = np.arange(n)
            num = np.take(f, np.minimum(i + 1, n - 1), axis=axis) - np.take(f, np.maximum(i - 1, 0), axis=axis)
            out &= ok(num) & ~((num == 0) & np.signbit(num))
        return out

    def see(k, f, v, args):
        nonlocal mask
        if f.op == "grad3d":
            mask &= numerators(args[0])
        m = ok(v)
        mask &= m.all(axis=-1) if m.ndim == 4 else m

    with np.errstate(all="ignore"):
        evaluate(dag, inputs, MeshWindow(x, y, z), on_value=see)
    return mask
