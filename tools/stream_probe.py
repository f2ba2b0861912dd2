"""Streamed strategy (host buffers, 1024^3 Q) vs chunk height (DFG_STREAM_PLANES):
wall time per execute and fraction of the pinned-copy PCIe bound."""
import json, os, sys, time
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import numpy as np, torch
import paper_conf_sc_harrisonnmjc12_b200 as dfg
import synth
QCRIT = dfg.paper_program("qcrit")

n = 1024
x, y, z = synth.rt_coords(n, n, n, np.float32)
x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
host = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda").cpu().pin_memory() for c in "uvw"}
hout = torch.empty((n, n, n), dtype=torch.float32).pin_memory()
for planes in [p for p in (sys.argv[1:] or ["0", "32", "16", "8"])]:
    if planes == "0":
        os.environ.pop("DFG_STREAM_PLANES", None)
    else:
        os.environ["DFG_STREAM_PLANES"] = planes
    mesh = dfg.Mesh(x, y, z)
    for c in "uvw":
        mesh.bind(c, host[c], on_device=False)
    plan = dfg.Plan(mesh, QCRIT, "streamed")
    plan.execute(hout, out_on_device=False)
    t0 = time.perf_counter()
    for _ in range(3):
        plan.execute(hout, out_on_device=False)
    ms = (time.perf_counter() - t0) / 3 * 1e3
    print(json.dumps({"planes": planes or "default", "ms": round(ms, 1)}), flush=True)
    plan.close()
    mesh.close()
