"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and
bench.py.  This module holds NO arithmetic of the method (no gradient, no
expression evaluation): only coordinates and velocity fields.

Recipe (stands in for the LLNL Rayleigh-Taylor DNS the
paper used, L154 / L348, which is not available):

* Coordinates (non-uniform, strictly increasing, L = 1, origin 0):
  - x, y: h_i = (L/n)(1 + 0.5 U(-1, 1)) from ``numpy.random.default_rng(seed)``
    (x seed 1, y seed 2), cumulative sum, rescaled so p_n = L;
  - z: sinh clustering towards the mixing layer at z = L/2,
    p_k = L/2 (1 + sinh(beta (2k/n - 1)) / sinh(beta)), beta = 1.5.
* RT-like velocity at cell centres (centre = midpoint of the bounding points,
  L154 / L223), computed in float64 and cast to T:
      u = E(z) * sum_{m=1..8} A_m sin(k_m . X + phi_m) + 1e-3 * noise
  E(z) = exp(-((z - 1/2) / 0.15)^2); per mode from default_rng(seed), in this
  order: a direction (3 normals, normalised), |k| ~ U[2 pi, 16 pi],
  phi ~ U[0, 2 pi); A = (|k| / 2 pi)^(-5/6).  Seeds u = 11, v = 12, w = 13.
  noise = a standard normal from a counter-based generator (splitmix64 of
  (seed, global cell index) -> Box-Muller), so any window of any size can be
  generated on any device without generating the rest of the mesh.
* Dyadic closed-form meshes: spacings drawn from {1, 2, 3} * 2^-6, a different
  permutation per axis, so every centre, difference and quotient of the
  closed-form fields is exact in float32 and float64.
"""

from __future__ import annotations

import math

import numpy as np
import torch

RT_SEEDS = {"u": 11, "v": 12, "w": 13}
NOISE_SEED = 99


# ----------------------------------------------------------------- coordinates
def coords_jitter(n: int, seed: int, L: float = 1.0) -> np.ndarray:
    rng = np.random.default_rng(seed)
    h = (L / n) * (1.0 + 0.5 * rng.uniform(-1.0, 1.0, n))
    p = np.concatenate([[0.0], np.cumsum(h)])
    p *= L / p[-1]
    p[-1] = L
    return p


def coords_sinh(n: int, beta: float = 1.5, L: float = 1.0) -> np.ndarray:
    k = np.arange(n + 1, dtype=np.float64)
    return 0.5 * L * (1.0 + np.sinh(beta * (2.0 * k / n - 1.0)) / math.sinh(beta))


def rt_coords(nx: int, ny: int, nz: int, dtype=np.float32):
    """Point coordinates (x, y, z) of the RT-like mesh, cast to T."""
    return (coords_jitter(nx, 1).astype(dtype), coords_jitter(ny, 2).astype(dtype),
            coords_sinh(nz).astype(dtype))


def dyadic_coords(n: int, seed: int, dtype=np.float64, origin: float = 0.0) -> np.ndarray:
    rng = np.random.default_rng(seed)
    h = rng.permutation(np.resize(np.array([1.0, 2.0, 3.0]), n)) * 2.0 ** -6
    p = origin + np.concatenate([[0.0], np.cumsum(h)])
    return p.astype(dtype)


def uniform_coords(n: int, h: float = 2.0 ** -5, dtype=np.float64) -> np.ndarray:
    return (np.arange(n + 1, dtype=np.float64) * h).astype(dtype)


def centres64(p: np.ndarray) -> np.ndarray:
    """Cell-centre positions in float64, for generating field VALUES only."""
    p = np.asarray(p, dtype=np.float64)
    return 0.5 * (p[:-1] + p[1:])


# -------------------------------------------------------------- RT-like field
def rt_modes(seed: int, nmodes: int = 8):
    rng = np.random.default_rng(seed)
    modes = []
    for _ in range(nmodes):
        d = rng.standard_normal(3)
        d /= np.linalg.norm(d)
        kmag = rng.uniform(2 * math.pi, 16 * math.pi)
        phi = rng.uniform(0.0, 2 * math.pi)
        amp = (kmag / (2 * math.pi)) ** (-5.0 / 6.0)
        modes.append((d * kmag, phi, amp))
    return modes


_M64 = (1 << 64) - 1


def _to_i64(v: int) -> int:
    v &= _M64
    return v - (1 << 64) if v >= (1 << 63) else v


_SM_A = _to_i64(0x9E3779B97F4A7C15)
_SM_B = _to_i64(0xBF58476D1CE4E5B9)
_SM_C = _to_i64(0x94D049BB133111EB)


def _lsr(x: torch.Tensor, s: int) -> torch.Tensor:
    return (x >> s) & ((1 << (64 - s)) - 1)


def _splitmix64(x: torch.Tensor) -> torch.Tensor:
    z = x + _SM_A
    z = (z ^ _lsr(z, 30)) * _SM_B
    z = (z ^ _lsr(z, 27)) * _SM_C
    return z ^ _lsr(z, 31)


def _noise(seed: int, gidx: torch.Tensor) -> torch.Tensor:
    """Standard normal per global cell index (counter-based, device-agnostic)."""
    base = gidx * 2 + (seed << 48)
    h1 = _splitmix64(base)
    h2 = _splitmix64(base + 1)
    u1 = (_lsr(h1, 11).to(torch.float64) + 1.0) * 2.0 ** -53    # (0, 1]
    u2 = _lsr(h2, 11).to(torch.float64) * 2.0 ** -53            # [0, 1)
    return torch.sqrt(-2.0 * torch.log(u1)) * torch.cos(2 * math.pi * u2)


def rt_velocity(comp: str, x, y, z, window=None, dtype=torch.float32,
                device="cpu", chunk_planes: int = 32) -> torch.Tensor:
    """Velocity component ``comp`` in {u, v, w} on the window
    (k0, k1, j0, j1, i0, i1) (global cell indices; default = whole mesh).
    Returns a contiguous tensor [k1-k0, j1-j0, i1-i0] of ``dtype``."""
    nx, ny, nz = len(x) - 1, len(y) - 1, len(z) - 1
    if window is None:
        window = (0, nz, 0, ny, 0, nx)
    k0, k1, j0, j1, i0, i1 = window
    cx = torch.tensor(centres64(x)[i0:i1], dtype=torch.float64, device=device)
    cy = torch.tensor(centres64(y)[j0:j1], dtype=torch.float64, device=device)
    czall = centres64(z)
    modes = rt_modes(RT_SEEDS[comp])
    out = torch.empty((k1 - k0, j1 - j0, i1 - i0), dtype=dtype, device=device)
    ii = torch.arange(i0, i1, device=device, dtype=torch.int64).view(1, 1, -1)
    jj = torch.arange(j0, j1, device=device, dtype=torch.int64).view(1, -1, 1)
    for kb in range(k0, k1, chunk_planes):
        ke = min(k1, kb + chunk_planes)
        cz = torch.tensor(czall[kb:ke], dtype=torch.float64, device=device).view(-1, 1, 1)
        acc = torch.zeros((ke - kb, j1 - j0, i1 - i0), dtype=torch.float64, device=device)
        for kv, phi, amp in modes:
            arg = (kv[0] * cx.view(1, 1, -1) + kv[1] * cy.view(1, -1, 1)) + (kv[2] * cz + phi)
            acc += amp * torch.sin(arg)
        env = torch.exp(-((cz - 0.5) / 0.15) ** 2)
        kk = torch.arange(kb, ke, device=device, dtype=torch.int64).view(-1, 1, 1)
        gidx = (kk * ny + jj) * nx + ii
        noise = _noise(NOISE_SEED * 4 + "uvw".index(comp), gidx)
        out[kb - k0:ke - k0] = (env * acc + 1e-3 * noise).to(dtype)
    return out


def rt_inputs(nx, ny, nz, dtype=np.float32, device="cpu", names=("u", "v", "w"),
              window=None):
    """(x, y, z, {name: tensor}) for the RT-like workload; names other than
    u/v/w reuse the u/v/w recipes in order (e.g. the intro's b = u, c = v)."""
    x, y, z = rt_coords(nx, ny, nz, dtype)
    tdt = torch.float32 if np.dtype(dtype) == np.float32 else torch.float64
    fields = {}
    for n_, comp in zip(names, ("u", "v", "w")):
        fields[n_] = rt_velocity(comp, x.astype(np.float64), y.astype(np.float64),
                                 z.astype(np.float64), window, tdt, device)
    return x, y, z, fields


# -------------------------------------------------------- closed-form fields
def closed_form(kind: str, x, y, z):
    """Velocity (u, v, w) or scalar fields at cell centres (float64 values;
    exact on dyadic meshes).  Returns dict name -> array[k, j, i]."""
    cx, cy, cz = centres64(x), centres64(y), centres64(z)
    Z, Y, X = np.meshgrid(cz, cy, cx, indexing="ij")
    if kind == "linear":                      # f = 3x - 2y + 5z
        return {"f": 3 * X - 2 * Y + 5 * Z}
    if kind == "quadratic":                   # f = x^2
        return {"f": X * X}
    if kind == "rotation":                    # v = Omega x (r - r0), Omega = 3 e_z
        om = 3.0
        x0, y0 = cx[len(cx) // 2], cy[len(cy) // 2]
        return {"u": -om * (Y - y0), "v": om * (X - x0), "w": np.zeros_like(X)}
    if kind == "strain":                      # u = a x, v = b y, w = -(a+b) z
        a, b = 2.0, -3.0
        return {"u": a * X, "v": b * Y, "w": -(a + b) * Z}
    if kind == "shear":                       # u = gamma y
        g = 2.0
        return {"u": g * Y, "v": np.zeros_like(X), "w": np.zeros_like(X)}
    raise ValueError(kind)
