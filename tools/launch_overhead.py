"""Launch overhead of one execute on a tiny mesh (developer tool).

    python tools/launch_overhead.py [--n 32]

For device sleeps of 0, 0.1 and 1 ms before the first event (so the host
enqueues behind a busy GPU), times a torch zero_() and fused VelMag / Q
executes between CUDA events, plus the library's own kernel events.
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_harrisonnmjc12_b200 as dfg  # noqa: E402
import synth  # noqa: E402
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=32)
    args = ap.parse_args()
    n = args.n
    x, y, z = synth.rt_coords(n, n, n, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    bufs = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for c, b in bufs.items():
        mesh.bind(c, b)
    out = torch.empty((n, n, n), dtype=torch.float32, device="cuda")
    lvl = int(os.environ.get("DFG_TIMING_LEVEL", "1"))
    plans = {e: dfg.Plan(mesh, PAPER_PROGRAMS[e][0], "fused").set_timing(lvl) for e in ("velmag", "qcrit")}
    ops = {"torch_zero": lambda: out.zero_()}
    for e, p in plans.items():
        ops[e] = p.execute if False else (lambda p=p: p.execute(out))
    for _ in range(5):
        for f in ops.values():
            f()
    torch.cuda.synchronize()
    for sleep in (0, 200_000, 2_000_000):
        for name, f in ops.items():
            ev, kv, host = [], [], []
            for _ in range(20):
                torch.cuda.synchronize()
                if sleep:
                    torch.cuda._sleep(sleep)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                t0 = time.perf_counter()
                f()
                host.append((time.perf_counter() - t0) * 1e6)
                e1.record()
                e1.synchronize()
                ev.append(e0.elapsed_time(e1) * 1e3)
                if name in plans and lvl >= 1:
                    kv.append(plans[name].stats()["last_ms"] * 1e3)
            rec = {"sleep_cycles": sleep, "op": name, "event_us": round(float(np.median(ev)), 2),
                   "host_call_us": round(float(np.median(host)), 2)}
            if kv:
                rec["kernel_event_us"] = round(float(np.median(kv)), 2)
            print(json.dumps(rec), flush=True)
    # amortized: 200 back-to-back calls on the default and on a side stream
    side = torch.cuda.Stream()
    for sname, st in (("default", None), ("side", side)):
        for name, f in ops.items():
            ctx = torch.cuda.stream(st) if st is not None else torch.cuda.stream(torch.cuda.current_stream())
            with ctx:
                if name in plans:
                    g = (lambda p=plans[name]: p.execute(out, stream=torch.cuda.current_stream()))
                else:
                    g = f
                torch.cuda.synchronize()
                torch.cuda._sleep(20_000_000)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(200):
                    g()
                e1.record()
                e1.synchronize()
                rec = {"amortized_stream": sname, "op": name, "us_per_call": round(e0.elapsed_time(e1) * 1e3 / 200, 2)}
                rec["timing_level"] = lvl
                print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
