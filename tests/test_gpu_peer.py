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


def _run(*args):
    cmd = [sys.executable, os.path.join(ROOT, "tools", "peer_ranks.py"), *map(str, args)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    return json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])


@pytest.mark.parametrize("ranks,prog,dtype,nz", [(2, "qcrit", "f32", 29), (3, "qcrit", "f64", 29),
                                                 (4, "intro", "f32", 23), (3, "vortmag", "f32", 5),
                                                 (3, "qcrit", "f32", 3)])
def test_peer_slabs_match_single_slab(ranks, prog, dtype, nz):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    line = _run("--ranks", ranks, "--n", 64, "--nz", nz, "--prog", prog, "--dtype", dtype, "--steps", 3)
    assert line["bit_identical_to_single_slab"]
    assert line["halo_modes"] == [3] * ranks                  # read in place by the TMA kernel
    assert all(line["ghost_planes_untouched"])
    assert line["halo_fields"] == (1 if prog == "intro" else 3)   # stencil fields only (intro: b)
    # interior launch (when a slab has interior planes) + one boundary launch per side
    for r_, k in enumerate(line["kernels_per_execute"]):
        nzl = nz // ranks + (r_ < nz % ranks)
        sides = (r_ > 0) + (r_ < ranks - 1)
        assert k == (1 if nzl - sides <= 0 else 1 + sides)


def test_peer_copy_fallback_for_tile_layouts():
    """nx = 66 (rows not a multiple of 16 bytes): the tile kernel cannot read
    peers in place, so the two planes are copied through the mappings."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    line = _run("--ranks", 3, "--n", 40, "--nx", 66, "--nz", 17, "--steps", 2)
    assert line["bit_identical_to_single_slab"]
    assert line["halo_modes"] == [4, 4, 4]
