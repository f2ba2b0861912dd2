"""B200-native dynamic derived-field generation (Harrison et al., SC 2012).

The compute path is libdfg.so (C++ host runtime + sm_100a CUDA kernels, see
include/dfg.h).  This package is its Python binding: the ``dfg_*`` functions
keep the C names and argument order, and ``Mesh`` / ``Plan`` are thin
handle owners on top of them.  PyTorch is used by callers only for device
memory and streams.
"""

from __future__ import annotations

from ._dfg import *  # noqa: F401,F403
from ._dfg import (DFG_F32, DFG_F64, DfgError, EXPORTS, LIB_PATH, STRATEGIES,  # noqa: F401
                   dfg_bind_field, dfg_compile, dfg_create_mesh, dfg_destroy_mesh, dfg_destroy_plan,
                   dfg_dump_dag, dfg_dump_kernel, dfg_execute, dfg_halo_map, dfg_plan_info, dfg_plan_stats,
                   dfg_plan_set_timing, dfg_reset_stats)


def _dtype_code(dtype) -> int:
    s = str(dtype)
    if s in ("float32", "torch.float32", "f32", "<class 'numpy.float32'>"):
        return DFG_F32
    if s in ("float64", "torch.float64", "f64", "<class 'numpy.float64'>"):
        return DFG_F64
    raise ValueError(f"unsupported dtype {dtype}")


class Mesh:
    """Owns a dfg_mesh.  x, y, z: point coordinates (numpy, T); for a z slab
    pass the GLOBAL z and (nz_global, z_offset, ghost)."""

    def __init__(self, x, y, z, nz_local=None, z_offset=0, ghost=0):
        import numpy as np
        x, y, z = (np.ascontiguousarray(a) for a in (x, y, z))
        assert x.dtype == y.dtype == z.dtype
        self.dtype = x.dtype
        self.nx, self.ny, self.nz_global = len(x) - 1, len(y) - 1, len(z) - 1
        self.nz = self.nz_global if nz_local is None else nz_local
        self.ghost = ghost
        self._coords = (x, y, z)
        self.handle = dfg_create_mesh(_dtype_code(x.dtype), self.nx, self.ny, self.nz, x, y, z,
                                      self.nz_global, z_offset, ghost)
        self._bound = {}

    @classmethod
    def block(cls, x, y, z, nx, ny, nz, i0, j0, k0, ghost=1, row_pitch=0, x_offset=0):
        """VisIt-style sub-grid of the global mesh with points x, y, z:
        local nx x ny x nz cells at (i0, j0, k0), one-cell ghost shell on all
        six faces filled by the caller (dfg_create_block); buffers
        T[nz+2][ny+2][row_pitch], owned cells from column x_offset
        (0: x_offset = ghost, row_pitch = x_offset + nx + ghost)."""
        import numpy as np
        from ._dfg import dfg_create_block
        self = cls.__new__(cls)
        x, y, z = (np.ascontiguousarray(a) for a in (x, y, z))
        self.dtype = x.dtype
        self.nx, self.ny, self.nz, self.nz_global = nx, ny, nz, len(z) - 1
        self.ghost = ghost
        self._coords = (x, y, z)
        self._bound = {}
        self.x_offset = x_offset or ghost
        self.row_pitch = row_pitch or self.x_offset + nx + ghost
        self.handle = dfg_create_block(_dtype_code(x.dtype), nx, ny, nz, x, y, z, len(x) - 1, len(y) - 1,
                                       len(z) - 1, i0, j0, k0, ghost, row_pitch, x_offset)
        return self

    def bind(self, name, buf, on_device=None):
        if on_device is None:
            on_device = bool(getattr(buf, "is_cuda", False))
        self._bound[name] = buf          # keep the borrowed buffer alive
        dfg_bind_field(self.handle, name, buf, on_device)

    def halo_map(self):
        return dfg_halo_map(self.handle)

    def peer_export(self) -> bytes:
        """Blob for the z neighbours' link_peers (bind the device fields first)."""
        from ._dfg import dfg_mesh_peer_export
        return dfg_mesh_peer_export(self.handle)

    def link_peers(self, lo_blob, hi_blob):
        """Read the neighbours' boundary planes in place (peer-memory halo)."""
        from ._dfg import dfg_mesh_link_peers
        dfg_mesh_link_peers(self.handle, lo_blob, hi_blob)

    def close(self):
        if self.handle:
            dfg_destroy_mesh(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Plan:
    """Owns a dfg_plan compiled from an expression on a Mesh."""

    def __init__(self, mesh: Mesh, expr: str, strategy="fused", dev_mem_cap=0):
        self.mesh = mesh
        self.handle = dfg_compile(mesh.handle, expr, strategy, dev_mem_cap)

    def execute(self, out, out_on_device=None, stream=None):
        if out_on_device is None:
            out_on_device = bool(getattr(out, "is_cuda", False))
        s = stream if (stream is None or isinstance(stream, int)) else stream.cuda_stream
        dfg_execute(self.handle, out, out_on_device, s)
        return out

    def stats(self):
        return dfg_plan_stats(self.handle)

    def set_timing(self, level: int):
        """0: no CUDA events, 1: execute interval (default), 2: also per fused launch."""
        dfg_plan_set_timing(self.handle, level)
        return self

    def reset_stats(self):
        dfg_reset_stats(self.handle)

    def info(self):
        return dfg_plan_info(self.handle)

    def dag(self):
        return dfg_dump_dag(self.handle)

    def schedule(self):
        from ._dfg import dfg_plan_schedule
        return dfg_plan_schedule(self.handle)

    def transfers(self):
        from ._dfg import dfg_plan_transfers
        return dfg_plan_transfers(self.handle)

    def kernel_source(self):
        return dfg_dump_kernel(self.handle)

    def close(self):
        if self.handle:
            dfg_destroy_plan(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def execute_blocks(plans, outs, stream=None):
    """One launch for fused plans of one network on several meshes (VisIt
    blocks of a device; dfg_execute_blocks).  outs: device tensors."""
    from ._dfg import dfg_execute_blocks
    s = stream if (stream is None or isinstance(stream, int)) else stream.cuda_stream
    dfg_execute_blocks([p.handle for p in plans], outs, s)
    return outs


PAPER_INPUTS = {"velmag": ("u", "v", "w"), "vortmag": ("u", "v", "w"), "qcrit": ("u", "v", "w"), "intro": ("b", "c")}


def paper_program(which: str) -> str:
    """The paper's program text (dfg_paper_program): velmag, vortmag, qcrit
    (Fig. 3, inputs u, v, w) or intro (L19, inputs b, c)."""
    from ._dfg import dfg_paper_program
    return dfg_paper_program(which)
