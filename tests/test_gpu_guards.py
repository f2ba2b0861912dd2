"""Guard bands around every buffer the fused kernels touch (the pool has no
compute-sanitizer): inputs and outputs are views into larger allocations
whose margins hold a sentinel bit pattern; after an execute the margins must
be untouched and the inputs unchanged, on every kernel variant (TMA, row
class, cp.async tile, general, point-wise) and for blocks in one launch.
Offsets of 16 bytes keep the aligned paths; offsets of one element force the
unaligned ones (scalar stores, no tensor maps)."""
import numpy as np
import pytest
import torch

from dfg_testutil import run_oracle, assert_parity, tdtype
import synth

pytestmark = pytest.mark.gpu

SENT32 = 0x7FC0DEAD  # a NaN payload no kernel produces
SENT64 = 0x7FF8DEADBEEFDEAD


def _sentinel(T):
    return (np.uint32(SENT32) if T == np.float32 else np.uint64(SENT64))


def _guarded(shape, T, lead, tail, fill=None):
    """A [lead | shape | tail] allocation of T with sentinel margins; returns
    (whole, view)."""
    n = int(np.prod(shape))
    it = np.uint32 if T == np.float32 else np.uint64
    whole = torch.from_numpy(np.full(lead + n + tail, _sentinel(T), dtype=it).view(T)).cuda()
    view = whole[lead:lead + n].view(*shape)
    if fill is not None:
        view.copy_(torch.from_numpy(np.ascontiguousarray(fill)).cuda())
    return whole, view


def _margins_intact(whole, lead, n, T):
    it = torch.int32 if T == np.float32 else torch.int64
    bits = whole.view(it).cpu().numpy()
    s = np.int64(np.array(_sentinel(T)).view(np.int32 if T == np.float32 else np.int64))
    return bool((bits[:lead] == s).all() and (bits[lead + n:] == s).all())


CASES = [
    # shape, T, program, DFG_FUSED_KERNEL, element offset of every buffer, variant
    ((64, 20, 9), np.float32, "qcrit", None, 4, 1),       # TMA kernel
    ((67, 20, 9), np.float32, "qcrit", None, 4, 7),       # row-class kernel (P = 4)
    ((66, 8, 9), np.float32, "vortmag", None, 4, 7),      # row-class kernel (P = 2)
    ((66, 8, 9), np.float64, "qcrit", None, 2, 1),        # fp64, TMA kernel
    ((67, 8, 9), np.float64, "qcrit", None, 2, 7),        # fp64, row-class kernel
    ((64, 20, 9), np.float32, "qcrit", None, 1, 5),       # unaligned buffers: cp.async ring
    ((67, 21, 9), np.float32, "intro", "tile", 4, 5),     # cp.async ring
    ((67, 21, 9), np.float32, "qcrit", "general", 3, 2),  # z-marching columns
    ((67, 21, 9), np.float32, "velmag", None, 1, 3),      # point-wise, unaligned
]


@pytest.mark.parametrize("shape,T,prog,kernel,off,variant", CASES)
def test_guard_bands_single_mesh(shape, T, prog, kernel, off, variant, monkeypatch):
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    if kernel:
        monkeypatch.setenv("DFG_FUSED_KERNEL", kernel)
    names = dfg.PAPER_INPUTS[prog]
    nx, ny, nz = shape
    x, y, z, f = synth.rt_inputs(nx, ny, nz, dtype=T, names=names)
    f = {k: v.numpy() for k, v in f.items()}
    mesh = dfg.Mesh(x, y, z)
    keep = []
    for n in names:
        whole, view = _guarded((nz, ny, nx), T, off, 37, f[n])
        keep.append((whole, n))
        mesh.bind(n, view)
    src = dfg.paper_program(prog)
    plan = dfg.Plan(mesh, src, "fused")
    owhole, out = _guarded((nz, ny, nx), T, off, 41)
    plan.execute(out)
    torch.cuda.synchronize()
    assert plan.info()["variant"] == variant, plan.info()
    assert _margins_intact(owhole, off, nx * ny * nz, T), plan.info()
    for whole, n in keep:
        assert _margins_intact(whole, off, nx * ny * nz, T)
        got_in = whole[off:off + nx * ny * nz].cpu().numpy().reshape(nz, ny, nx)
        assert np.array_equal(got_in.view(np.uint8), np.ascontiguousarray(f[n]).view(np.uint8))
    assert_parity(out.cpu().numpy(), run_oracle(src, f, x, y, z))


@pytest.mark.parametrize("xo", [1, 4])
def test_guard_bands_blocks_one_launch(xo):
    """Packed (row-class kernel) and padded (TMA) ghost-shell blocks in one
    launch, every field and output a guarded view."""
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    T = np.float32
    shape, split = (64, 20, 14), (2, 2, 2)
    x, y, z, f = synth.rt_inputs(*shape, dtype=T)
    f = {k: v.numpy() for k, v in f.items()}
    pad = {n: np.pad(a, 1, mode="edge") for n, a in f.items()}
    src = dfg.paper_program("qcrit")
    whole_want = run_oracle(src, f, x, y, z)
    plans, outs, guards = [], [], []
    rp = 34 if xo == 1 else 40
    for a in range(2):
        for b in range(2):
            for c in range(2):
                i0, j0, k0 = 32 * a, 10 * b, 7 * c
                m = dfg.Mesh.block(x, y, z, 32, 10, 7, i0, j0, k0, ghost=1, row_pitch=rp, x_offset=xo)
                for n in "uvw":
                    buf = np.full((9, 12, rp), np.nan, T)
                    buf[:, :, xo - 1:xo + 33] = pad[n][k0:k0 + 9, j0:j0 + 12, i0:i0 + 34]
                    w, v = _guarded(buf.shape, T, 4, 29, buf)
                    guards.append((w, 4, buf.size))
                    m.bind(n, v)
                plans.append((dfg.Plan(m, src, "fused"), m, (i0, j0, k0)))
                w, o = _guarded((7, 10, 32), T, 4, 31)
                guards.append((w, 4, o.numel()))
                outs.append(o)
    dfg.execute_blocks([p for p, _, _ in plans], outs)
    torch.cuda.synchronize()
    assert plans[0][0].info()["variant"] == (8 if xo == 1 else 4)
    for w, lead, n in guards:
        assert _margins_intact(w, lead, n, T)
    got = np.empty_like(whole_want)
    for (p, m, (i0, j0, k0)), o in zip(plans, outs):
        got[k0:k0 + 7, j0:j0 + 10, i0:i0 + 32] = o.cpu().numpy()
    assert_parity(got, whole_want)
