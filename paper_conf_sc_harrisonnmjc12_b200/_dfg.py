"""ctypes binding of libdfg.so (include/dfg.h) -- argument marshalling only.

Every function has the C name and C argument order; pointers may be given as
ints, numpy arrays or torch tensors (their data pointer is passed).  A
negative status raises ``DfgError`` with the library's message.  There is no
Python or CPU implementation of anything behind these names: if the shared
library is missing the import fails.
"""

from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libdfg.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
        "or `make -C paper_conf_sc_harrisonnmjc12_b200/csrc`; libdfg has no CPU fallback")

_lib = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)

DFG_ROUNDTRIP, DFG_STAGED, DFG_FUSED, DFG_STREAMED, DFG_REFERENCE, DFG_HYBRID = 0, 1, 2, 3, 4, 5
DFG_F32, DFG_F64 = 0, 1
STRATEGIES = {"roundtrip": DFG_ROUNDTRIP, "staged": DFG_STAGED, "fused": DFG_FUSED, "streamed": DFG_STREAMED,
              "reference": DFG_REFERENCE, "hybrid": DFG_HYBRID}
TRANSFER_KINDS = ("upload", "reload", "spill", "discard", "drop", "run", "sink_d2h", "sink_host", "sink_h2d")
STATUS = {0: "DFG_OK", -1: "DFG_E_INVALID", -2: "DFG_E_PARSE", -3: "DFG_E_UNDEFINED", -4: "DFG_E_TYPE",
          -5: "DFG_E_NOMEM", -6: "DFG_E_NVRTC", -7: "DFG_E_CUDA", -8: "DFG_E_NCCL", -9: "DFG_E_UNBOUND",
          -10: "DFG_E_UNSUPPORTED", -11: "DFG_E_RANGE"}


class DfgError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status
        self.name = STATUS.get(status, str(status))
        self.msg = msg


class dfg_stats(C.Structure):
    _fields_ = [(n, C.c_int64) for n in (
        "executes", "h2d_count", "d2h_count", "kernel_count", "h2d_bytes", "d2h_bytes", "halo_bytes",
        "dev_highwater_bytes", "predicted_highwater_bytes", "predicted_hbm_bytes", "predicted_pcie_bytes")] + [
        ("last_ms", C.c_double), ("kernel_ms_sum", C.c_double), ("kernel_launches_timed", C.c_int64)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


_P = C.c_void_p
_I64 = C.c_int64
_SIGS = {
    "dfg_version": (C.c_int, []),
    "dfg_last_error": (C.c_char_p, []),
    "dfg_create_mesh": (C.c_int, [C.c_int, _I64, _I64, _I64, _P, _P, _P, _I64, _I64, C.c_int, C.POINTER(_P)]),
    "dfg_create_block": (C.c_int, [C.c_int, _I64, _I64, _I64, _P, _P, _P, _I64, _I64, _I64, _I64, _I64, _I64,
                                   C.c_int, _I64, _I64, C.POINTER(_P)]),
    "dfg_destroy_mesh": (None, [_P]),
    "dfg_partition": (C.c_int, [_I64, C.c_int, C.c_int, C.POINTER(_I64), C.POINTER(_I64)]),
    "dfg_halo_map": (C.c_int, [_P, C.POINTER(_I64)]),
    "dfg_nccl_unique_id": (C.c_int, [_P]),
    "dfg_mesh_init_comm": (C.c_int, [_P, _P, C.c_int, C.c_int]),
    "dfg_mesh_link_local": (C.c_int, [_P, _P]),
    "dfg_mesh_peer_export": (C.c_int, [_P, _P, C.c_size_t]),
    "dfg_mesh_link_peers": (C.c_int, [_P, _P, _P]),
    "dfg_peer_probe": (C.c_int, [_P, C.POINTER(C.c_int)]),
    "dfg_bind_field": (C.c_int, [_P, C.c_char_p, _P, C.c_int]),
    "dfg_compile": (C.c_int, [_P, C.c_char_p, C.c_int, C.c_size_t, C.POINTER(_P)]),
    "dfg_destroy_plan": (None, [_P]),
    "dfg_execute": (C.c_int, [_P, _P, C.c_int, _P]),
    "dfg_execute_blocks": (C.c_int, [C.POINTER(_P), C.c_int, C.POINTER(_P), _P]),
    "dfg_plan_stats": (C.c_int, [_P, C.POINTER(dfg_stats)]),
    "dfg_reset_stats": (C.c_int, [_P]),
    "dfg_plan_set_timing": (C.c_int, [_P, C.c_int]),
    "dfg_plan_info": (C.c_int, [_P, C.POINTER(_I64)]),
    "dfg_plan_arith": (C.c_int, [_P, C.POINTER(_I64)]),
    "dfg_plan_schedule": (C.c_int, [_P, C.POINTER(C.c_int32), C.c_size_t, C.POINTER(C.c_size_t)]),
    "dfg_plan_transfers": (C.c_int, [_P, C.POINTER(C.c_int32), C.c_size_t, C.POINTER(C.c_size_t)]),
    "dfg_hybrid_model": (C.c_int, [C.c_char_p, C.POINTER(C.c_char_p), C.c_int, C.c_int, C.c_int64,
                                   C.POINTER(C.c_int32), C.c_size_t, C.POINTER(C.c_int32), C.c_size_t,
                                   C.POINTER(C.c_size_t), C.POINTER(_I64)]),
    "dfg_dump_dag": (C.c_int, [_P, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
    "dfg_dump_kernel": (C.c_int, [_P, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
    "dfg_dag_dump": (C.c_int, [C.c_char_p, C.POINTER(C.c_char_p), C.c_int, C.c_int, C.c_char_p, C.c_size_t,
                               C.POINTER(C.c_size_t)]),
    "dfg_model": (C.c_int, [C.c_char_p, C.POINTER(C.c_char_p), C.c_int, C.c_int, C.c_int, C.POINTER(_I64)]),
    "dfg_points3d_to_axes": (C.c_int, [C.c_int, _I64, _I64, _I64, _P, _P, _P, _P, _P, _P]),
    "dfg_div2_check": (C.c_int, [C.c_int, _P, _I64, C.c_int, _P, _P]),
    "dfg_paper_program": (C.c_int, [C.c_char_p, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
    "dfg_fused_source": (C.c_int, [C.c_char_p, C.POINTER(C.c_char_p), C.c_int, C.c_int, _I64, _I64, _I64, C.c_int,
                                   C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t), C.POINTER(C.c_int),
                                   C.POINTER(C.c_int)]),
}
EXPORTS = tuple(_SIGS)
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


def _check(status: int):
    if status != 0:
        raise DfgError(status, _lib.dfg_last_error().decode())


def _ptr(x):
    """Data pointer of an int / numpy array / torch tensor / None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    raise TypeError(type(x))


def _names(inputs):
    arr = (C.c_char_p * max(len(inputs), 1))(*[s.encode() for s in inputs])
    return arr, len(inputs)


def _text(fn, *args):
    need = C.c_size_t(0)
    st = fn(*args, None, 0, C.byref(need))
    if st not in (0, -11):
        _check(st)
    buf = C.create_string_buffer(need.value)
    _check(fn(*args, buf, need.value, C.byref(need)))
    return buf.value.decode()


# --------------------------------------------------------------- C names
def dfg_version() -> int:
    return _lib.dfg_version()


def dfg_last_error() -> str:
    return _lib.dfg_last_error().decode()


def dfg_create_mesh(dtype, nx, ny, nz_local, x, y, z, nz_global=None, z_offset=0, ghost=0):
    h = _P()
    _check(_lib.dfg_create_mesh(dtype, nx, ny, nz_local, _ptr(x), _ptr(y), _ptr(z),
                                nz_local if nz_global is None else nz_global, z_offset, ghost, C.byref(h)))
    return h.value


def dfg_create_block(dtype, nx, ny, nz, x, y, z, NX, NY, NZ, i0, j0, k0, ghost=1, row_pitch=0, x_offset=0):
    h = _P()
    _check(_lib.dfg_create_block(dtype, nx, ny, nz, _ptr(x), _ptr(y), _ptr(z), NX, NY, NZ, i0, j0, k0, ghost,
                                 row_pitch, x_offset, C.byref(h)))
    return h.value


def dfg_destroy_mesh(mesh):
    _lib.dfg_destroy_mesh(mesh)


def dfg_partition(nz_global, nranks, rank):
    off, n = _I64(), _I64()
    _check(_lib.dfg_partition(nz_global, nranks, rank, C.byref(off), C.byref(n)))
    return off.value, n.value


def dfg_halo_map(mesh):
    out = (_I64 * 16)()
    _check(_lib.dfg_halo_map(mesh, out))
    return list(out)


def dfg_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _check(_lib.dfg_nccl_unique_id(buf))
    return buf.raw


def dfg_mesh_init_comm(mesh, uid: bytes, rank, nranks):
    buf = C.create_string_buffer(bytes(uid), 128)
    _check(_lib.dfg_mesh_init_comm(mesh, buf, rank, nranks))


PEER_BLOB_BYTES = 4096


def dfg_mesh_peer_export(mesh) -> bytes:
    buf = C.create_string_buffer(PEER_BLOB_BYTES)
    _check(_lib.dfg_mesh_peer_export(mesh, buf, PEER_BLOB_BYTES))
    return buf.raw


def dfg_mesh_link_peers(mesh, lo_blob, hi_blob):
    def arg(b):
        return None if b is None else C.create_string_buffer(bytes(b), PEER_BLOB_BYTES)
    lo, hi = arg(lo_blob), arg(hi_blob)
    _check(_lib.dfg_mesh_link_peers(mesh, lo, hi))


def dfg_peer_probe(blob) -> bool:
    ok = C.c_int(0)
    _check(_lib.dfg_peer_probe(C.create_string_buffer(bytes(blob), PEER_BLOB_BYTES), C.byref(ok)))
    return bool(ok.value)


def dfg_mesh_link_local(lo, hi):
    _check(_lib.dfg_mesh_link_local(lo, hi))


def dfg_bind_field(mesh, name, ptr, on_device):
    _check(_lib.dfg_bind_field(mesh, name.encode(), _ptr(ptr), int(on_device)))


def dfg_compile(mesh, expr, strategy, dev_mem_cap=0):
    if isinstance(strategy, str):
        strategy = STRATEGIES[strategy]
    h = _P()
    _check(_lib.dfg_compile(mesh, expr.encode(), strategy, dev_mem_cap, C.byref(h)))
    return h.value


def dfg_destroy_plan(plan):
    _lib.dfg_destroy_plan(plan)


def dfg_execute(plan, out, out_on_device, cuda_stream=None):
    _check(_lib.dfg_execute(plan, _ptr(out), int(out_on_device), cuda_stream))


def dfg_plan_stats(plan) -> dict:
    st = dfg_stats()
    _check(_lib.dfg_plan_stats(plan, C.byref(st)))
    return st.as_dict()


def dfg_plan_set_timing(plan, level: int):
    _check(_lib.dfg_plan_set_timing(plan, int(level)))


def dfg_reset_stats(plan):
    _check(_lib.dfg_reset_stats(plan))


def dfg_plan_arith(plan) -> dict:
    out = (_I64 * 4)()
    _check(_lib.dfg_plan_arith(plan, out))
    return {"div_mode": ("ieee", "exact_normal", "fast")[out[0]], "fold": bool(out[1]), "div2_axes": out[2],
            "exact_domain": ("tolerance", "normal_range", "all_inputs")[out[3]]}


def dfg_plan_info(plan) -> dict:
    out = (_I64 * 14)()
    _check(_lib.dfg_plan_info(plan, out))
    keys = ("strategy", "width", "filters", "variant", "regs", "spill", "footprint_device", "footprint_host",
            "div2_axes", "rows_per_warp", "tile_w", "tile_h", "kz", "halo")
    return dict(zip(keys, list(out)))


def dfg_plan_transfers(plan) -> list:
    """DFG_HYBRID transfer schedule: [(kind name, ref)], ref = filter id or
    -1 - input index."""
    n = C.c_size_t(0)
    _check(_lib.dfg_plan_transfers(plan, None, 0, C.byref(n)))
    arr = (C.c_int32 * max(2 * n.value, 1))()
    _check(_lib.dfg_plan_transfers(plan, arr, n.value, C.byref(n)))
    return [(TRANSFER_KINDS[arr[2 * i]], int(arr[2 * i + 1])) for i in range(n.value)]


def dfg_hybrid_model(expr, inputs, host_mode, cap_units, order=None):
    """(events, high, h2d, d2h, h2d_units, d2h_units) of the hybrid planner."""
    arr, n_in = _names(inputs)
    ordp, n_ord = None, 0
    if order is not None:
        ordp = (C.c_int32 * max(len(order), 1))(*order)
        n_ord = len(order)
    n = C.c_size_t(0)
    out = (_I64 * 5)()
    _check(_lib.dfg_hybrid_model(expr.encode(), arr, n_in, int(host_mode), cap_units, ordp, n_ord, None, 0,
                                 C.byref(n), out))
    ev = (C.c_int32 * max(2 * n.value, 1))()
    _check(_lib.dfg_hybrid_model(expr.encode(), arr, n_in, int(host_mode), cap_units, ordp, n_ord, ev, n.value,
                                 C.byref(n), out))
    events = [(TRANSFER_KINDS[ev[2 * i]], int(ev[2 * i + 1])) for i in range(n.value)]
    return (events,) + tuple(int(v) for v in out)


def dfg_execute_blocks(plans, outs, stream=None):
    """plans: handles; outs: device tensors (or pointers), one per plan."""
    n = len(plans)
    ph = (_P * n)(*plans)
    oh = (_P * n)(*[_ptr(o) for o in outs])
    _check(_lib.dfg_execute_blocks(ph, n, oh, stream))


def dfg_plan_schedule(plan) -> list:
    n = C.c_size_t(0)
    _check(_lib.dfg_plan_schedule(plan, None, 0, C.byref(n)))
    arr = (C.c_int32 * max(n.value, 1))()
    _check(_lib.dfg_plan_schedule(plan, arr, n.value, C.byref(n)))
    return list(arr)[: n.value]


def dfg_dump_dag(plan) -> str:
    return _text(_lib.dfg_dump_dag, plan)


def dfg_dump_kernel(plan) -> str:
    return _text(_lib.dfg_dump_kernel, plan)


def dfg_dag_dump(expr, inputs, dtype=DFG_F32) -> str:
    arr, n = _names(inputs)
    return _text(_lib.dfg_dag_dump, expr.encode(), arr, n, dtype)


def dfg_model(expr, inputs, strategy, host_mode=True):
    if isinstance(strategy, str):
        strategy = STRATEGIES[strategy]
    arr, n = _names(inputs)
    out = (_I64 * 4)()
    _check(_lib.dfg_model(expr.encode(), arr, n, strategy, int(host_mode), out))
    return list(out)


def dfg_points3d_to_axes(x3, y3, z3):
    """numpy [nz+1][ny+1][nx+1] point arrays -> (x, y, z) 1-D axes (T)."""
    import numpy as np
    x3, y3, z3 = (np.ascontiguousarray(a) for a in (x3, y3, z3))
    assert x3.shape == y3.shape == z3.shape and x3.dtype == y3.dtype == z3.dtype
    pz, py, px = x3.shape
    x, y, z = np.empty(px, x3.dtype), np.empty(py, x3.dtype), np.empty(pz, x3.dtype)
    dt = DFG_F32 if x3.dtype == np.float32 else DFG_F64
    _check(_lib.dfg_points3d_to_axes(dt, px - 1, py - 1, pz - 1, _ptr(x3), _ptr(y3), _ptr(z3),
                                     _ptr(x), _ptr(y), _ptr(z)))
    return x, y, z


def dfg_paper_program(which):
    """The paper's program text: "velmag", "vortmag", "qcrit" (inputs u, v, w), "intro" (b, c)."""
    need = C.c_size_t(0)
    st = _lib.dfg_paper_program(which.encode(), None, 0, C.byref(need))
    if st not in (0, -11):
        _check(st)
    buf = C.create_string_buffer(need.value)
    _check(_lib.dfg_paper_program(which.encode(), buf, need.value, C.byref(need)))
    return buf.value.decode()


def dfg_div2_check(d, method=0):
    """numpy divisors (float32 / float64) -> (ok uint8[n], candidates tested int64[n])."""
    import numpy as np
    d = np.ascontiguousarray(d)
    ok = np.zeros(d.shape[0], np.uint8)
    tested = np.zeros(d.shape[0], np.int64)
    dt = DFG_F32 if d.dtype == np.float32 else DFG_F64
    _check(_lib.dfg_div2_check(dt, _ptr(d), d.shape[0], method, _ptr(ok), _ptr(tested)))
    return ok, tested


def dfg_fused_source(expr, inputs, dtype, nx, ny, nz, compile=False):
    """Returns (source, regs, spill)."""
    arr, n = _names(inputs)
    regs, spill = C.c_int(-1), C.c_int(-1)
    need = C.c_size_t(0)
    st = _lib.dfg_fused_source(expr.encode(), arr, n, dtype, nx, ny, nz, int(compile), None, 0, C.byref(need),
                               C.byref(regs), C.byref(spill))
    if st not in (0, -11):
        _check(st)
    buf = C.create_string_buffer(need.value)
    _check(_lib.dfg_fused_source(expr.encode(), arr, n, dtype, nx, ny, nz, 0, buf, need.value, C.byref(need),
                                 None, None))
    return buf.value.decode(), regs.value, spill.value
