"""The peer-memory z-slab halo on a one-GPU box.

tools/peer_ranks.py runs G ranks (processes) on cuda:0; each exports its slab
(CUDA IPC handles of its fields and step flags), links its z neighbours and
runs several time steps, rewriting its owned planes between executes.  The
fused kernel reads the neighbours' boundary planes in place through the IPC
mappings -- the code path of the NVLink case, same-device mappings only.  The
stitched slabs must equal the single-slab result of every step bit for bit,
and the ghost planes (NaN) must stay untouched on the in-place path.
"""
import json
import os
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args, env=None):
    cmd = [sys.executable, os.path.join(ROOT, "tools", "peer_ranks.py"), *map(str, args)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT,
                       env=None if env is None else dict(os.environ, **env))
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    return json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])


@pytest.mark.parametrize("inkernel", ["1", "0"])
@pytest.mark.parametrize("ranks,prog,dtype,nz", [(2, "qcrit", "f32", 29), (3, "qcrit", "f64", 29),
                                                 (4, "intro", "f32", 23), (3, "vortmag", "f32", 5),
                                                 (3, "qcrit", "f32", 3)])
def test_peer_slabs_match_single_slab(ranks, prog, dtype, nz, inkernel):
    """inkernel 1 (default): ONE launch per execute, the producers wait in
    the kernel for the neighbours' ready flags; 0: interior launch, stream
    waits, boundary-plane launches."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    line = _run("--ranks", ranks, "--n", 64, "--nz", nz, "--prog", prog, "--dtype", dtype, "--steps", 3,
                env={"DFG_PEER_INKERNEL": inkernel})
    assert line["bit_identical_to_single_slab"] and line["bit_identical_to_oracle"]
    assert line["halo_modes"] == [3] * ranks                  # read in place by the TMA kernel
    assert all(line["ghost_planes_untouched"])
    assert line["halo_fields"] == (1 if prog == "intro" else 3)   # stencil fields only (intro: b)
    # in-kernel waits: one launch; else the interior launch (when a slab has
    # interior planes) + one boundary launch per side
    for r_, k in enumerate(line["kernels_per_execute"]):
        nzl = nz // ranks + (r_ < nz % ranks)
        sides = (r_ > 0) + (r_ < ranks - 1)
        assert k == (1 if inkernel == "1" or nzl - sides <= 0 else 1 + sides)


def test_peer_copy_fallback_for_tile_layouts():
    """nx = 66 (rows not a multiple of 16 bytes): the tile kernel cannot read
    peers in place, so the two planes are copied through the mappings."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    line = _run("--ranks", 3, "--n", 40, "--nx", 66, "--nz", 17, "--steps", 2)
    assert line["bit_identical_to_single_slab"] and line["bit_identical_to_oracle"]
    assert line["halo_modes"] == [4, 4, 4]


def test_peer_probe_isolated():
    """dfg_peer_probe in a child process: a TMA read through the IPC mapping
    of an exported slab's probe block returns the exporter's pattern; a
    blob that is not an export fails in the child, not here."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import numpy as np
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    import synth
    x, y, z = synth.rt_coords(32, 16, 12, np.float32)
    m = dfg.Mesh(x, y, z, nz_local=6, z_offset=6, ghost=1)
    bufs = [torch.zeros((8, 16, 32), device="cuda") for _ in range(3)]
    for c, b in zip("uvw", bufs):
        m.bind(c, b)
    blob = m.peer_export()
    ok, detail = dfg.probe_peer_transport([blob, None], torch.cuda.current_device())
    assert ok, detail
    bad = bytearray(blob)
    bad[:8] = b"notablob"
    ok, detail = dfg.probe_peer_transport([bytes(bad)], torch.cuda.current_device())
    assert not ok and "DFG_E_INVALID" in detail


def test_bench_two_ranks_one_gpu():
    """`bench.py --gpus 2` launches its own two ranks (no torchrun wrapper);
    DFG_BENCH_ONE_GPU=1 puts both on cuda:0 (functional, not a timing): the
    line says n_gpus 2, the in-place halo passed its isolated probe on both
    ranks, and rank 0's slab boundary equals the oracle bit for bit."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, DFG_BENCH_ONE_GPU="1")
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK"):
        env.pop(k, None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup",
                        "3", "--size", "128", "--no-strategies"], capture_output=True, text=True, timeout=900,
                       cwd=ROOT, env=env)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    line = json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["config"]["one_gpu_functional_test"]
    mg = line["multi_gpu"]
    assert mg["halo_mode"] == "peer" and all(p["ok"] for p in mg["halo_probe"])
    assert mg["comm_ranks"] == [2, 2] and mg["comm_rank_of_rank"] == [0, 1]
    par = line["cpu_baseline"]["slab_boundary_parity"]
    assert par["cells_compared"] > 0 and par["mismatches"] == 0
