"""B200-native dynamic derived-field generation (Harrison et al., SC 2012).

The compute path is libdfg.so (C++ host runtime + sm_100a CUDA kernels, see
include/dfg.h).  This package is its Python binding: the ``dfg_*`` functions
keep the C names and argument order, and ``Mesh`` / ``Plan`` are thin
handle owners on top of them.  PyTorch is used by callers only for device
memory and streams.
"""

from __future__ import annotations

import sys

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


def _current_device():
    """The CUDA device current now (the one dfg_create_mesh takes), or None
    when torch or CUDA is absent."""
    torch = sys.modules.get("torch")
    if torch is None or not torch.cuda.is_available():
        return None
    return torch.cuda.current_device()


def _check_buffer(buf, dtype, numel, device, what):
    """Validate a torch tensor / numpy array before its raw pointer crosses
    the C ABI (which cannot see dtype, size, strides or device): contiguous,
    the mesh's element type, exactly the layout's element count (dfg.h) and,
    for a CUDA tensor, the mesh's device.  Plain integer pointers pass
    unchecked.  Raises ValueError."""
    import numpy as np
    if isinstance(buf, int) or buf is None:
        return
    if hasattr(buf, "is_contiguous"):                       # torch.Tensor
        if not buf.is_contiguous():
            raise ValueError(f"{what}: tensor is not contiguous")
        got = np.dtype(str(buf.dtype).replace("torch.", ""))
        n = buf.numel()
        if buf.is_cuda and device is not None and buf.device.index != device:
            raise ValueError(f"{what}: tensor on cuda:{buf.device.index}, mesh on cuda:{device}")
    elif isinstance(buf, np.ndarray):
        if not buf.flags["C_CONTIGUOUS"]:
            raise ValueError(f"{what}: array is not C-contiguous")
        got, n = buf.dtype, buf.size
    else:
        return
    if got != np.dtype(dtype):
        raise ValueError(f"{what}: dtype {got}, mesh type {np.dtype(dtype)}")
    if n != numel:
        raise ValueError(f"{what}: {n} elements, the layout needs {numel}")


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
        self.device = _current_device()
        # bound field layout T[nz_local + 2 ghost][ny][nx] (dfg.h)
        self.field_numel = (self.nz + 2 * ghost) * self.ny * self.nx
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
        self.device = _current_device()
        # T[nz + 2 ghost][ny + 2 ghost][row_pitch] (dfg_create_block)
        self.field_numel = (nz + 2 * ghost) * (ny + 2 * ghost) * self.row_pitch
        self.handle = dfg_create_block(_dtype_code(x.dtype), nx, ny, nz, x, y, z, len(x) - 1, len(y) - 1,
                                       len(z) - 1, i0, j0, k0, ghost, row_pitch, x_offset)
        return self

    def bind(self, name, buf, on_device=None):
        if on_device is None:
            on_device = bool(getattr(buf, "is_cuda", False))
        if buf is not None:
            _check_buffer(buf, self.dtype, self.field_numel, self.device, f"field '{name}'")
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
        self._out_numel = mesh.nz * mesh.ny * mesh.nx * self.info()["width"]   # T[nz][ny][nx](x4)

    def execute(self, out, out_on_device=None, stream=None):
        if out_on_device is None:
            out_on_device = bool(getattr(out, "is_cuda", False))
        m = self.mesh
        _check_buffer(out, m.dtype, self._out_numel, m.device, "output")
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

    def arith(self):
        """Quotient form, scale folding and the exactness domain: the inputs
        on which the results equal the literal network in T (dfg_plan_arith)."""
        from ._dfg import dfg_plan_arith
        return dfg_plan_arith(self.handle)

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


def probe_peer_transport(blobs, device: int, timeout: float = 120.0):
    """dfg_peer_probe on every neighbour blob, in a child process on CUDA
    device ``device`` (dfg.h: a transport that faults must not take the
    caller down).  Returns (ok, detail)."""
    import os
    import subprocess
    blobs = [b for b in blobs if b is not None]
    if not blobs:
        return True, "no neighbours"
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = ("import sys; sys.path.insert(0, sys.argv[1]); import torch; torch.cuda.set_device(int(sys.argv[2]))\n"
            "from paper_conf_sc_harrisonnmjc12_b200._dfg import dfg_peer_probe\n"
            "oks = [dfg_peer_probe(bytes.fromhex(h)) for h in sys.stdin.read().split()]\n"
            "print('probe', ' '.join(str(int(o)) for o in oks))\n")
    try:
        r = subprocess.run([sys.executable, "-c", code, root, str(device)], input=" ".join(b.hex() for b in blobs),
                           capture_output=True, text=True, timeout=timeout)
    except subprocess.TimeoutExpired:
        return False, "probe process timed out"
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("probe ")]
    if r.returncode != 0 or not lines:
        return False, f"probe process exit {r.returncode}: {(r.stderr or r.stdout).strip()[-300:]}"
    oks = lines[-1].split()[1:]
    if len(oks) != len(blobs) or any(o != "1" for o in oks):
        return False, f"probe read a wrong pattern ({' '.join(oks)})"
    return True, f"{len(blobs)} neighbour(s): TMA read through the IPC mapping returned the pattern"


PAPER_INPUTS = {"velmag": ("u", "v", "w"), "vortmag": ("u", "v", "w"), "qcrit": ("u", "v", "w"), "intro": ("b", "c")}


def paper_program(which: str) -> str:
    """The paper's program text (dfg_paper_program): velmag, vortmag, qcrit
    (Fig. 3, inputs u, v, w) or intro (L19, inputs b, c)."""
    from ._dfg import dfg_paper_program
    return dfg_paper_program(which)
