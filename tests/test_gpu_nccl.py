"""The library's NCCL z-slab path on a one-GPU box.

tools/nccl_two_ranks.py runs G ranks on cuda:0, each with its own
NCCL_HOSTID so that NCCL accepts them (it treats them as separate hosts and
uses its socket transport over loopback).  Everything above the transport is
the multi-GPU code: dfg_nccl_unique_id / dfg_mesh_init_comm, the grouped
send/recv of the ghost planes on the plan's side stream overlapped with the
interior planes, then the boundary-plane launches.  The stitched slab results
must equal the single-slab result bit for bit.
"""
import json
import os
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("ranks,overlap,prog,dtype", [(2, 1, "qcrit", "f32"), (3, 1, "qcrit", "f64"),
                                                      (3, 0, "vortmag", "f32"), (4, 1, "intro", "f32")])
def test_nccl_slabs_match_single_slab(ranks, overlap, prog, dtype):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    cmd = [sys.executable, os.path.join(ROOT, "tools", "nccl_two_ranks.py"), "--ranks", str(ranks), "--n", "64",
           "--nz", "29", "--prog", prog, "--overlap", str(overlap), "--dtype", dtype]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    line = json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["bit_identical_to_single_slab"] and line["bit_identical_to_oracle"] and line["halo_bytes_ok"]
    # interior launch + one boundary launch per halo side when overlapped
    want = [1 + (r_ > 0) + (r_ < ranks - 1) if overlap else 1 for r_ in range(ranks)]
    assert line["kernels_per_execute"] == want
