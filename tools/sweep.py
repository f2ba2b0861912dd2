"""Parameter sweep of the fused kernel (developer tool, not the bench).

    python tools/sweep.py [--n 1024] [--iters 200] [--expr qcrit]

For each configuration (environment variables read by dfg_compile /
dfg_execute: DFG_FUSED_VARIANT, DFG_NCW, DFG_STAGES, DFG_KZ) compiles a
plan on the same device-resident 1024^3 inputs and times `iters` back-to-back
executes with CUDA events; prints one JSON line per configuration with the
median SM clock seen by nvidia-smi during the timed loop.
"""
import argparse
import itertools
import json
import os
import subprocess
import sys
import threading

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_harrisonnmjc12_b200 as dfg  # noqa: E402
import synth  # noqa: E402
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}


def clocks(stop, out):
    while not stop.is_set():
        r = subprocess.run(["nvidia-smi", "--id=0", "--query-gpu=clocks.sm,power.draw",
                            "--format=csv,noheader,nounits"], capture_output=True, text=True).stdout.strip()
        try:
            a, b = r.split(",")
            out.append((float(a), float(b)))
        except Exception:
            pass
        stop.wait(0.05)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1024)
    ap.add_argument("--iters", type=int, default=200)
    ap.add_argument("--expr", default="qcrit")
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--configs", default="")
    args = ap.parse_args()
    n = args.n
    T = np.float32 if args.dtype == "f32" else np.float64
    tt = torch.float32 if T == np.float32 else torch.float64
    src, names = PAPER_PROGRAMS[args.expr]
    x, y, z = synth.rt_coords(n, n, n, T)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    bufs = {nm: synth.rt_velocity(c, x64, y64, z64, None, tt, "cuda") for nm, c in zip(names, "uvw")}
    for k, v in bufs.items():
        mesh.bind(k, v)
    out = torch.empty((n, n, n), dtype=tt, device="cuda")
    ref = None
    if args.configs:
        confs = [dict(kv.split("=") for kv in c.split(",") if kv) for c in args.configs.split(";")]
    else:
        confs = [dict(DFG_FUSED_VARIANT=v, DFG_NCW=str(w)) for v, w in itertools.product(
            ["exact", "fast", "ieee"], [15, 7])]
    nbytes = (len(names) + 1) * np.dtype(T).itemsize
    for conf in confs:
        for k in ("DFG_FUSED_VARIANT", "DFG_NCW", "DFG_STAGES", "DFG_KZ", "DFG_FUSED_KERNEL", "DFG_CTAS"):
            os.environ.pop(k, None)
        os.environ.update(conf)
        plan = dfg.Plan(mesh, src, "fused")
        for _ in range(5):
            plan.execute(out)
        torch.cuda.synchronize()
        if ref is None:
            ref = out.clone()
        same = bool(torch.equal(ref, out))
        samples = []
        stop = threading.Event()
        th = threading.Thread(target=clocks, args=(stop, samples), daemon=True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        th.start()
        e0.record()
        for _ in range(args.iters):
            plan.execute(out)
        e1.record()
        e1.synchronize()
        stop.set()
        th.join()
        ms = e0.elapsed_time(e1) / args.iters
        info = plan.info()
        sm = float(np.median([s[0] for s in samples])) if samples else None
        pw = float(np.median([s[1] for s in samples])) if samples else None
        print(json.dumps({"conf": conf, "ms": round(ms, 4), "gcells_s": round(n ** 3 / ms / 1e6, 1),
                          "tb_s": round(nbytes * n ** 3 / ms / 1e9, 3), "regs": info["regs"],
                          "variant": info["variant"], "same_as_first": same, "sm_mhz": sm, "power_w": pw}),
              flush=True)
        plan.close()


if __name__ == "__main__":
    main()
