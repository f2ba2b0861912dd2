"""Small-mesh timing of the fused kernel (developer tool, not the bench).

    python tools/small_mesh.py [--n 192] [--configs "K=V,..;.."]

Times one fused execute per run after three L2 conditions: `dirty` (write a
512 MB buffer: L2 full of dirty lines whose write-back lands inside the timed
kernel), `clean` (write 512 MB, then read another 512 MB: L2 cold and clean),
`warm` (no flush).  Trimmed mean of 9 runs, CUDA events on the current stream
recorded behind a short device sleep (host launch latency not timed), and the
library's own events around the kernel launch (`kernel_us`).
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
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}

KNOBS = ("DFG_FUSED_VARIANT", "DFG_NCW", "DFG_STAGES", "DFG_KZ", "DFG_FUSED_KERNEL", "DFG_CTAS", "DFG_ROWS_PER_WARP")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=192)
    ap.add_argument("--runs", type=int, default=9)
    ap.add_argument("--exprs", default="velmag,vortmag,qcrit")
    ap.add_argument("--configs", default="")
    args = ap.parse_args()
    n = args.n
    x, y, z = synth.rt_coords(n, n, n, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    bufs = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for c, b in bufs.items():
        mesh.bind(c, b)
    big_w = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    big_r = torch.ones(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    out = torch.empty((n, n, n), dtype=torch.float32, device="cuda")
    confs = [dict(kv.split("=") for kv in c.split(",") if kv) for c in args.configs.split(";")] if args.configs else [{}]
    for expr in args.exprs.split(","):
        src = PAPER_PROGRAMS[expr][0]
        for conf in confs:
            for k in KNOBS:
                os.environ.pop(k, None)
            os.environ.update(conf)
            plan = dfg.Plan(mesh, src, "fused")
            for _ in range(3):
                plan.execute(out)
            res = {}
            for mode in ("dirty", "clean", "warm"):
                ts, ks = [], []
                for _ in range(args.runs):
                    if mode != "warm":
                        big_w.zero_()
                    if mode == "clean":
                        big_r.sum()
                    torch.cuda.synchronize()
                    # keep the GPU busy while the host enqueues: e0 then fires right
                    # before the kernel, so host launch latency is not timed
                    torch.cuda._sleep(200000)
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    plan.execute(out)
                    e1.record()
                    e1.synchronize()
                    ts.append(e0.elapsed_time(e1))
                    ks.append(plan.stats()["last_ms"])
                ts = sorted(ts)[1:-1]
                ms = sum(ts) / len(ts)
                ks = sorted(ks)[1:-1]
                kms = sum(ks) / len(ks)
                res[mode] = {"us": round(ms * 1e3, 2), "gcells_s": round(n ** 3 / ms / 1e6, 1),
                             "tb_s": round(16 * n ** 3 / ms / 1e9, 3),
                             "kernel_us": round(kms * 1e3, 2), "kernel_tb_s": round(16 * n ** 3 / kms / 1e9, 3)}
            info = plan.info()
            print(json.dumps({"expr": expr, "conf": conf, "kernel": info["variant"], "regs": info["regs"], **res}),
                  flush=True)
            plan.close()


if __name__ == "__main__":
    main()
