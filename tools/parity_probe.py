"""Full-size parity probe (developer tool): fused Q on the 1024^3 bench mesh
against the oracle on a block, per fused-body variant, listing mismatching
cells with their bits.

    python tools/parity_probe.py [--planes 123] [--rows 512]
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
from oracle import evaluate as oev  # noqa: E402
from oracle.lang import QCRIT, build_dag  # noqa: E402

N = 1024


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--planes", type=int, default=123)
    ap.add_argument("--rows", type=int, default=512)
    ap.add_argument("--k0", type=int, default=100)
    ap.add_argument("--j0", type=int, default=200)
    args = ap.parse_args()
    x, y, z = synth.rt_coords(N, N, N, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    bufs = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for c, b in bufs.items():
        mesh.bind(c, b)
    k0, j0, P, R = args.k0, args.j0, args.planes, args.rows
    win = (k0 - 1, k0 + P + 1, j0 - 1, j0 + R + 1, 0, N)
    f = {c: bufs[c][win[0]:win[1], win[2]:win[3], :].cpu().numpy() for c in "uvw"}
    dag = build_dag(QCRIT, ("u", "v", "w"), "f32")
    res, valid = oev.evaluate(dag, f, oev.MeshWindow(x, y, z, i0=0, j0=win[2], k0=win[0]))
    want = res[1:-1, 1:-1, :]
    out = torch.empty((N, N, N), device="cuda")
    report = {}
    for conf in ({}, {"DFG_FUSED_VARIANT": "ieee"}, {"DFG_FUSED_VARIANT": "markstein"}, {"DFG_SCALE_FOLD": "0"},
                 {"DFG_DIV2": "0"}, {"DFG_FUSED_KERNEL": "general"}):
        for k in ("DFG_FUSED_VARIANT", "DFG_SCALE_FOLD", "DFG_DIV2", "DFG_FUSED_KERNEL"):
            os.environ.pop(k, None)
        os.environ.update(conf)
        plan = dfg.Plan(mesh, QCRIT, "fused")
        plan.execute(out)
        torch.cuda.synchronize()
        got = out[k0:k0 + P, j0:j0 + R, :].cpu().numpy()
        bad = np.argwhere(got.view(np.uint32) != want.view(np.uint32))
        cells = []
        for kk, jj, ii in bad[:12]:
            g, w = got[kk, jj, ii], want[kk, jj, ii]
            cells.append({"k": int(k0 + kk), "j": int(j0 + jj), "i": int(ii), "gpu": float(g), "oracle": float(w),
                          "gpu_hex": float(g).hex(), "oracle_hex": float(w).hex(),
                          "ulps": int(abs(int(g.view(np.int32)) - int(w.view(np.int32))))})
        report[json.dumps(conf)] = {"mismatches": int(len(bad)), "cells": cells, "info": plan.info()}
        print(json.dumps({"conf": conf, "mismatches": int(len(bad)), "first": cells[:6]}), flush=True)
        plan.close()
    json.dump(report, open(os.path.join(ROOT, "gpurun_out", "parity_probe.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
