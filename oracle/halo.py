"""Oracle: z-slab decomposition and ghost-plane maps.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper's distributed run hands each sub-grid to the framework "with these
ghost cells, allowing the gradient primitives to compute the proper values on
the boundaries of all sub-grids" (L255, L315).  grad3d has stencil radius 1
(reading R1), so one ghost plane per side suffices (reading R12).  The
B200 build splits the mesh into contiguous z-slabs, one per rank, in rank
order:

    nz_r = NZ // G + (1 if r < NZ % G else 0)
    k0_r = r * (NZ // G) + min(r, NZ % G)

Local plane numbering with one ghost plane per side: ghost 0, owned planes
1..nz_r, ghost nz_r + 1.  Rank r sends its first owned plane to r-1 and its
last owned plane to r+1, and receives into its ghost planes.
"""

from __future__ import annotations


def partition(NZ: int, G: int, r: int):
    """(k0, nz_r) of rank r; requires NZ >= G >= 1."""
    assert G >= 1 and NZ >= G and 0 <= r < G
    q, m = divmod(NZ, G)
    nz_r = q + (1 if r < m else 0)
    k0 = r * q + min(r, m)
    return k0, nz_r


def halo_map(NZ: int, k0: int, nz_r: int, rank: int, nranks: int,
             nx: int, ny: int, itemsize: int):
    """The 16-entry map of DESIGN.md section 6 / include/dfg.h."""
    k1 = k0 + nz_r
    has_lo = 1 if k0 > 0 else 0
    has_hi = 1 if k1 < NZ else 0
    return [
        rank, nranks, NZ, k0, k1, nz_r, has_lo, has_hi,
        rank - 1 if has_lo else -1,
        rank + 1 if has_hi else -1,
        1 if has_lo else -1,            # send_lo_local_plane
        nz_r if has_hi else -1,         # send_hi_local_plane
        0 if has_lo else -1,            # recv_lo_local_plane
        nz_r + 1 if has_hi else -1,     # recv_hi_local_plane
        nx * ny * itemsize,             # plane_bytes
        1,                              # halo_width
    ]
