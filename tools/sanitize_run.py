"""Small end-to-end run of every strategy for compute-sanitizer (developer tool).

    compute-sanitizer --tool racecheck python tools/sanitize_run.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_harrisonnmjc12_b200 as dfg  # noqa: E402
import synth  # noqa: E402
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}


def main():
    shape = (132, 20, 13)
    for T, tt in ((np.float32, torch.float32), (np.float64, torch.float64)):
        x, y, z, f = synth.rt_inputs(*shape, dtype=T)
        mesh = dfg.Mesh(x, y, z)
        dev = {k: v.cuda() for k, v in f.items()}
        for k, v in dev.items():
            mesh.bind(k, v)
        out = torch.empty((shape[2], shape[1], shape[0]), dtype=tt, device="cuda")
        for prog in ("qcrit", "vortmag", "velmag"):
            for s in ("fused", "staged"):
                dfg.Plan(mesh, PAPER_PROGRAMS[prog][0], s).execute(out)
        dfg.Plan(mesh, "qcrit", "reference").execute(out)
        os.environ["DFG_KZ"] = "2"
        dfg.Plan(mesh, PAPER_PROGRAMS["qcrit"][0], "fused").execute(out)
        # the cp.async-filled ring (tile kernel), every tile shape, ragged rows
        for rpw in ("1", "2", "4"):
            os.environ["DFG_RPW"] = rpw
            os.environ["DFG_FUSED_KERNEL"] = "tile"
            dfg.Plan(mesh, PAPER_PROGRAMS["qcrit"][0], "fused").execute(out)
            os.environ.pop("DFG_FUSED_KERNEL")
            dfg.Plan(mesh, PAPER_PROGRAMS["qcrit"][0], "fused").execute(out)
        os.environ.pop("DFG_RPW")
        rx, ry, rz, rf = synth.rt_inputs(67, 21, 9, dtype=T)
        rmesh = dfg.Mesh(rx, ry, rz)
        rdev = {k: v.cuda() for k, v in rf.items()}
        for k, v in rdev.items():
            rmesh.bind(k, v)
        rout = torch.empty((9, 21, 67), dtype=tt, device="cuda")
        for prog in ("qcrit", "intro"):
            names = PAPER_PROGRAMS[prog][1]
            if prog == "intro":
                for nm, src_name in zip(names, ("u", "v")):
                    rmesh.bind(nm, rdev[src_name])
            dfg.Plan(rmesh, PAPER_PROGRAMS[prog][0], "fused").execute(rout)
        os.environ.pop("DFG_KZ")
        # streamed strategy from host fields (3-slot chunk ring, three streams)
        host = dfg.Mesh(x, y, z)
        for k, v in f.items():
            host.bind(k, v.numpy(), on_device=False)
        os.environ["DFG_STREAM_PLANES"] = "4"
        hout = np.empty((shape[2], shape[1], shape[0]), dtype=T)
        dfg.Plan(host, PAPER_PROGRAMS["qcrit"][0], "streamed").execute(hout, out_on_device=False)
        os.environ.pop("DFG_STREAM_PLANES")
        # three z-slabs linked in one process: halo exchange on the side stream
        # overlapped with the interior planes, then the boundary-plane launches
        slabs, keep = [], []
        for r in range(3):
            k0, nzr = dfg.dfg_partition(shape[2], 3, r)
            m = dfg.Mesh(x, y, z, nz_local=nzr, z_offset=k0, ghost=1)
            for k, v in f.items():
                buf = torch.zeros((nzr + 2,) + tuple(v.shape[1:]), dtype=tt, device="cuda")
                buf[1:nzr + 1] = v[k0:k0 + nzr].cuda()
                keep.append(buf)
                m.bind(k, buf)
            slabs.append(m)
        for r in range(2):
            dfg.dfg_mesh_link_local(slabs[r].handle, slabs[r + 1].handle)
        for m in slabs:
            o = torch.empty((m.nz, shape[1], shape[0]), dtype=tt, device="cuda")
            dfg.Plan(m, PAPER_PROGRAMS["qcrit"][0], "fused").execute(o)
        torch.cuda.synchronize()
    blocks_one_launch()
    print("sanitize run done")


def blocks_one_launch():
    """VisIt blocks of one device in one launch: packed ghost shells (the
    row-class kernel with its fixup warp, dfg_fused_rows_multi) and 16-byte
    padded shells (dfg_fused_tma_multi); 8 blocks of 32 x 10 x 7."""
    shape, split = (64, 20, 14), (2, 2, 2)
    x, y, z, f = synth.rt_inputs(*shape, dtype=np.float32)
    f = {k: v.numpy() for k, v in f.items()}
    pad = {n: np.pad(a, 1, mode="edge") for n, a in f.items()}
    for xo in (1, 4):
        plans, outs, keep = [], [], []
        for a in range(2):
            for b in range(2):
                for c in range(2):
                    i0, j0, k0 = 32 * a, 10 * b, 7 * c
                    rp = 34 if xo == 1 else 40
                    m = dfg.Mesh.block(x, y, z, 32, 10, 7, i0, j0, k0, ghost=1, row_pitch=rp, x_offset=xo)
                    for n in "uvw":
                        buf = np.zeros((9, 12, rp), np.float32)
                        buf[:, :, xo - 1:xo + 33] = pad[n][k0:k0 + 9, j0:j0 + 12, i0:i0 + 34]
                        t = torch.from_numpy(buf).cuda()
                        keep.append(t)
                        m.bind(n, t)
                    keep.append(m)
                    plans.append(dfg.Plan(m, PAPER_PROGRAMS["qcrit"][0], "fused"))
                    outs.append(torch.empty((7, 10, 32), device="cuda"))
        dfg.execute_blocks(plans, outs)
        torch.cuda.synchronize()
        print("blocks one launch, variant", plans[0].info()["variant"])


if __name__ == "__main__":
    main()
