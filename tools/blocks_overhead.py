"""Per-block launch overhead at the paper's VisIt block size (developer tool).

    python tools/blocks_overhead.py [--blocks 12] [--bx 192 --by 192 --bz 256]

Times B VisIt-style blocks (dfg_create_block, one-cell ghost shells) executed
one plan each, back to back on one stream, against one mesh holding the same
number of cells; prints one JSON line.
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_harrisonnmjc12_b200 as dfg  # noqa: E402
import synth  # noqa: E402
QCRIT = dfg.paper_program("qcrit")


def timeit(fn, iters=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters):
        fn()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / iters


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--blocks", type=int, default=12)
    ap.add_argument("--bx", type=int, default=192)
    ap.add_argument("--by", type=int, default=192)
    ap.add_argument("--bz", type=int, default=256)
    ap.add_argument("--pad", type=int, default=1, help="pad shell rows to a multiple of 16 bytes (TMA path)")
    a = ap.parse_args()
    print(json.dumps(measure(a.blocks, a.bx, a.by, a.bz, a.pad)))


def measure(B=12, bx=192, by=192, bz=256, pad=1):
    """B blocks of bx x by x bz stacked in z, one-cell ghost shells: one plan
    per block back to back, all blocks in one launch (dfg_execute_blocks) and
    one mesh of the same cells; returns a dict (times in ms)."""
    class a:  # noqa: N801
        pass
    a.pad = pad
    NZ = bz * B                       # blocks stacked in z: global mesh bx x by x (bz*B)
    x, y, z = synth.rt_coords(bx, by, NZ, np.float32)
    x64, y64, z64 = (v.astype(np.float64) for v in (x, y, z))
    plans, outs, keep = [], [], []
    for b in range(B):
        k0 = b * bz
        xo = 4 if a.pad else 1                       # first owned column (16-byte aligned when padded)
        rp = (xo + bx + 1 + 3) // 4 * 4 if a.pad else bx + 2
        m = dfg.Mesh.block(x, y, z, bx, by, bz, 0, 0, k0, ghost=1, row_pitch=rp, x_offset=xo)
        for c in "uvw":
            # ghost shell filled from the global field (clamped at the mesh ends)
            kk = np.clip(np.arange(k0 - 1, k0 + bz + 1), 0, NZ - 1)
            jj = np.clip(np.arange(-1, by + 1), 0, by - 1)
            ii = np.clip(np.arange(-1, bx + 1), 0, bx - 1)
            f = synth.rt_velocity(c, x64, y64, z64, (int(kk.min()), int(kk.max()) + 1, 0, by, 0, bx),
                                  torch.float32, "cuda")
            f = f[torch.as_tensor(kk - kk.min(), device="cuda")][:, torch.as_tensor(jj, device="cuda")][
                :, :, torch.as_tensor(ii, device="cuda")]
            f = torch.nn.functional.pad(f, (xo - 1, rp - (xo + bx + 1))).contiguous()
            keep.append(f)
            m.bind(c, f)
        p = dfg.Plan(m, QCRIT, "fused")
        o = torch.empty((bz, by, bx), dtype=torch.float32, device="cuda")
        plans.append(p)
        outs.append(o)
        keep.append(m)

    def blocks():
        for p, o in zip(plans, outs):
            p.execute(o)

    t_blocks = timeit(blocks)
    blocks_variant = plans[0].info()["variant"]
    t_batched = timeit(lambda: dfg.execute_blocks(plans, outs))
    batched_variant = plans[0].info()["variant"]
    whole = dfg.Mesh(x, y, z)
    wf = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for c, f in wf.items():
        whole.bind(c, f)
    wp = dfg.Plan(whole, QCRIT, "fused")
    wo = torch.empty((NZ, by, bx), dtype=torch.float32, device="cuda")
    t_whole = timeit(lambda: wp.execute(wo))
    same = bool(torch.equal(torch.cat(outs), wo))
    cells = bx * by * NZ
    res = {"blocks": B, "block": [bx, by, bz], "row_pitch": rp, "x_offset": xo, "cells": cells, "ms_blocks": t_blocks,
           "ms_batched": t_batched, "batched_variant": batched_variant,
           "gcells_s_batched": cells / t_batched / 1e6,
           "ms_one_mesh": t_whole, "overhead": t_blocks / t_whole - 1,
           "blocks_variant": blocks_variant, "bit_identical": same,
           "gcells_s_blocks": cells / t_blocks / 1e6, "gcells_s_one_mesh": cells / t_whole / 1e6}
    for p in plans + [wp]:
        p.close()
    return res


if __name__ == "__main__":
    main()
