"""One execute per bench configuration, for an ncu launch capture (developer tool).

    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,\\
        smsp__sass_thread_inst_executed.sum -k "regex:dfg|k_" --csv --log-file gpurun_out/cfg.csv \\
        python tools/ncu_configs.py > gpurun_out/cfg_order.json
    python tools/ncu_configs.py --summarize gpurun_out/cfg.csv gpurun_out/cfg_order.json > profiles/r02_configs.md

Each case compiles its plan, then executes once (ncu replays the launches
itself); the order file lists (case, cells, algorithmic bytes per cell, dfg
launches) so the summary can attribute every captured launch.
"""
import csv
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run():
    import torch
    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    import synth
    cases = [("Q fp32 192^3 fused (config 2)", "qcrit", 192, "f32", "fused"),
             ("Q fp32 192^3 staged (config 2)", "qcrit", 192, "f32", "staged"),
             ("Q fp32 512^3 fused (config 3)", "qcrit", 512, "f32", "fused"),
             ("intro fp32 768^3 fused (config 5)", "intro", 768, "f32", "fused"),
             ("VelMag fp32 768^3 fused (config 5)", "velmag", 768, "f32", "fused"),
             ("VortMag fp32 768^3 fused (config 5)", "vortmag", 768, "f32", "fused"),
             ("Q fp32 768^3 fused (config 5)", "qcrit", 768, "f32", "fused"),
             ("Q fp64 768^3 fused (config 5)", "qcrit", 768, "f64", "fused"),
             ("Q fp32 1024^3 fused (bench headline)", "qcrit", 1024, "f32", "fused"),
             ("Q fp32 1022^3 fused, row-class kernel", "qcrit", 1022, "f32", "fused")]
    order = []
    for label, prog, n, dt, strat in cases:
        npt, tt = (np.float32, torch.float32) if dt == "f32" else (np.float64, torch.float64)
        x, y, z = synth.rt_coords(n, n, n, npt)
        x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
        names = dfg.PAPER_INPUTS[prog]
        mesh = dfg.Mesh(x, y, z)
        flds = {nm: synth.rt_velocity(c, x64, y64, z64, None, tt, "cuda") for nm, c in zip(names, "uvw")}
        for nm, t in flds.items():
            mesh.bind(nm, t)
        if strat == "staged":
            os.environ["DFG_GRAPH"] = "0"   # plain launches (ncu sees each filter's kernel)
        plan = dfg.Plan(mesh, dfg.paper_program(prog), strat).set_timing(0)
        out = torch.empty((n, n, n), dtype=tt, device="cuda")
        plan.execute(out)
        torch.cuda.synchronize()
        st = plan.stats()
        nb = (len(names) + 1) * np.dtype(npt).itemsize
        order.append({"case": label, "cells": n ** 3, "fused_bytes_per_cell": nb,
                      "predicted_device_bytes": st["predicted_hbm_bytes"], "launches": st["kernel_count"],
                      "variant": plan.info()["variant"]})
        plan.close()
        mesh.close()
        del flds, out
        torch.cuda.empty_cache()
    print(json.dumps(order))


def summarize(csv_path, order_path):
    rows = list(csv.reader(open(csv_path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr, data = rows[hi], rows[hi + 1:]
    iI, iN, iM, iU, iV = (hdr.index(k) for k in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
    launches = {}
    for r in data:
        if ("dfg" not in r[iN] and "k_" not in r[iN]) or "verify_div2" in r[iN]:
            continue   # torch's kernels (input generation), the mesh's divisor check (not a step)
        d = launches.setdefault(int(r[iI]), {"name": r[iN].split("(")[0]})
        v = float(r[iV].replace(",", ""))
        unit = r[iU]
        if r[iM] == "gpu__time_duration.sum":
            v *= {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}.get(unit, 1.0)
        elif unit in ("Gbyte", "GB"):
            v *= 1e9
        elif unit in ("Mbyte", "MB"):
            v *= 1e6
        elif unit in ("Kbyte", "KB"):
            v *= 1e3
        d[r[iM]] = v
    ids = sorted(launches)
    order = json.load(open(order_path))
    print("# Per-configuration ncu accounting (round 2)\n")
    print("`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,"
          "smsp__sass_thread_inst_executed.sum --clock-control none -k \"regex:dfg|k_\"` over "
          "`tools/ncu_configs.py` (one execute per case, cold L2, launches serialised).  Predicted "
          "bytes: the library's model (fused: inputs + output once; staged: every filter's operands "
          "and result).\n")
    print("| case | kernel(s) | launches | ms | DRAM GB (read + write) | predicted GB | measured / predicted | "
          "thread instr / cell | GB/s (DRAM) |")
    print("|---|---|---|---|---|---|---|---|---|")
    pos = 0
    for o in order:
        ls = [launches[i] for i in ids[pos:pos + o["launches"]]]
        pos += o["launches"]
        ms = sum(l.get("gpu__time_duration.sum", 0) for l in ls)
        b = sum(l.get("dram__bytes_read.sum", 0) + l.get("dram__bytes_write.sum", 0) for l in ls)
        inst = sum(l.get("smsp__sass_thread_inst_executed.sum", 0) for l in ls)
        names = sorted({l["name"] for l in ls})
        pred = o["predicted_device_bytes"]
        print(f"| {o['case']} | {', '.join(names)[:60]} | {len(ls)} | {ms:.3f} | {b / 1e9:.3f} | {pred / 1e9:.3f} | "
              f"{b / pred:.3f} | {inst / o['cells']:.1f} | {b / (ms * 1e-3) / 1e9:.0f} |")


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--summarize":
        summarize(sys.argv[2], sys.argv[3])
    else:
        run()
