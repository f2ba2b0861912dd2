"""Sustained power / SM clock / time per launch of fused kernels at 1024^3
(1.5 s back-to-back per case, NVML sampled).  Context for DESIGN section 5:
which work the 1 kW board cap charges."""
import json, os, sys, time
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import numpy as np, torch
import paper_conf_sc_harrisonnmjc12_b200 as dfg
import synth
from bench import ClockSampler
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}

n = int(os.environ.get("N", "1024"))
x, y, z = synth.rt_coords(n, n, n, np.float32)
x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
f = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
out = torch.empty((n, n, n), dtype=torch.float32, device="cuda")
mesh = dfg.Mesh(x, y, z)
for c in "uvw":
    mesh.bind(c, f[c])


def run(name, fn, secs=1.5):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter(); k = 0
    with ClockSampler(0) as cs:
        e0.record()
        while time.perf_counter() - t0 < secs:
            for _ in range(20):
                fn()
            k += 20
            torch.cuda.synchronize()
        e1.record(); e1.synchronize()
    ms = e0.elapsed_time(e1) / k
    s = cs.summary()
    print(json.dumps({"case": name, "ms": round(ms, 4), "gcells_s": round(n ** 3 / ms / 1e6, 1),
                      "sm_mhz": s["sm_mhz"], "power_w": s["power_w"], "reasons": s["reasons"]}), flush=True)


cases = sys.argv[1:] or ["copy", "velmag", "vortmag", "qcrit", "qcrit_fast", "qcrit_ref"]
for c in cases:
    if c == "copy":
        a = torch.empty(n ** 3 * 3, dtype=torch.float32, device="cuda"); b = torch.empty(n ** 3, dtype=torch.float32, device="cuda")
        # 12 B read + 4 B written per cell, like the fused kernels: 3 reads summed into one output
        run("copy3to1 (torch sum of 3 planes)", lambda: torch.sum(a.view(3, -1), 0, out=b))
        del a, b
        continue
    env = {}
    prog, strat = c, "fused"
    if c.endswith("_fast"):
        prog, env = c[:-5], {"DFG_FUSED_VARIANT": "fast"}
    if c.endswith("_ref"):
        prog, strat = c[:-4], "reference"
    for k, v in env.items():
        os.environ[k] = v
    for k, v in [kv.split("=") for kv in os.environ.get("EXTRA", "").split(",") if "=" in kv]:
        os.environ[k] = v
    try:
        plan = dfg.Plan(mesh, PAPER_PROGRAMS[prog][0] if strat == "fused" else prog, strat)
    finally:
        for k in env:
            os.environ.pop(k, None)
    run(c + (" " + os.environ.get("EXTRA", "") if os.environ.get("EXTRA") else ""), lambda: plan.execute(out))
    plan.close()
