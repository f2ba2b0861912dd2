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
from oracle.lang import PAPER_PROGRAMS  # noqa: E402


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
        os.environ.pop("DFG_KZ")
        torch.cuda.synchronize()
    print("sanitize run done")


if __name__ == "__main__":
    main()
