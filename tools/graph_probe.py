"""Staged strategy with and without CUDA-graph replay (DFG_GRAPH): host time
per execute call (enqueue only) and device time per execute, back to back,
for VortMag / Q at 32^3 (config 1) and 192^3 (config 2).  One JSON line per case."""
import json, os, sys, time
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import numpy as np, torch
import paper_conf_sc_harrisonnmjc12_b200 as dfg
import synth
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}

for n in (32, 192):
    x, y, z = synth.rt_coords(n, n, n, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    f = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for prog in ("vortmag", "qcrit"):
        res = {}
        for g in ("1", "0"):
            os.environ["DFG_GRAPH"] = g
            mesh = dfg.Mesh(x, y, z)
            for c in "uvw":
                mesh.bind(c, f[c])
            plan = dfg.Plan(mesh, PAPER_PROGRAMS[prog][0], "staged").set_timing(0)
            out = torch.empty((n, n, n), device="cuda")
            for _ in range(3):
                plan.execute(out)
            torch.cuda.synchronize()
            iters = 200 if n == 32 else 50
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda._sleep(50_000_000)            # keep the device busy: host time is enqueue only
            t0 = time.perf_counter()
            e0.record()
            for _ in range(iters):
                plan.execute(out)
            e1.record()
            host_us = (time.perf_counter() - t0) / iters * 1e6
            e1.synchronize()
            res["graph" if g == "1" else "stream"] = {"host_us_per_execute": round(host_us, 1),
                                                       "device_us_per_execute": round(e0.elapsed_time(e1) / iters * 1e3, 1)}
            plan.close()
            mesh.close()
        print(json.dumps({"n": n, "prog": prog, **res}), flush=True)
os.environ.pop("DFG_GRAPH", None)
