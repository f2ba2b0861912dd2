"""Row-copy fused kernel vs the cp.async tile ring and the TMA kernel on
layouts the tensor maps cannot take (developer tool): one JSON line.

    python tools/rows_probe.py [--n 1022] [--iters 20]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1022)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--kernels", default="rows,tile")
    a = ap.parse_args()
    n = a.n
    x, y, z = synth.rt_coords(n, n, n, np.float32)
    x64, y64, z64 = (v.astype(np.float64) for v in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    f = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for c, t in f.items():
        mesh.bind(c, t)
    src = dfg.paper_program("qcrit")
    res = {"n": n}
    ref = None
    for k in a.kernels.split(","):
        os.environ["DFG_FUSED_KERNEL"] = k
        p = dfg.Plan(mesh, src, "fused").set_timing(2)
        o = torch.empty((n, n, n), device="cuda")
        for _ in range(3):
            p.execute(o)
        torch.cuda.synchronize()
        p.reset_stats()
        for _ in range(a.iters):
            p.execute(o)
        st = p.stats()
        ms = st["kernel_ms_sum"] / max(1, st["kernel_launches_timed"])
        res[k] = {"variant": p.info()["variant"], "kernel_ms": ms, "gcells_s": n ** 3 / ms / 1e6,
                  "algorithmic_gb_s": 16 * n ** 3 / ms / 1e6, "regs": p.info()["regs"]}
        if ref is None:
            ref = o.clone()
        else:
            res[k]["bit_identical_to_first"] = bool(torch.equal(o, ref))
        p.close()
        del o
    os.environ.pop("DFG_FUSED_KERNEL", None)
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
