"""Summaries of ncu output for profiles/ (developer tool).

    python tools/summarize_ncu.py launches <launches.csv> <out.csv>
        every dfg kernel launch of an `ncu --metrics gpu__time_duration.sum`
        log (torch launches -- synthetic input generation -- are only totalled)
    python tools/summarize_ncu.py traffic <prof.ncu-rep> <n>
        writes profiles/traffic.json (DRAM read+write bytes per launch of the
        profiled dfg_fused_tma launch) for bench.py's roofline.traffic
"""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def launches(src, dst):
    rows = list(csv.reader(open(src)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr, data = rows[hi], rows[hi + 1:]
    iN, iV, iU = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "nsecond": 1e-6, "ms": 1.0, "msecond": 1.0}
    dfg, other, n_other = [], 0.0, 0
    for r in data:
        ms = float(r[iV].replace(",", "")) * scale.get(r[iU], 1.0)
        if "dfg" in r[iN]:
            dfg.append((r[0], r[iN].split("(")[0][:60], ms))
        else:
            other += ms
            n_other += 1
    tot = sum(d[2] for d in dfg)
    with open(dst, "w") as f:
        f.write("# ncu --metrics gpu__time_duration.sum --clock-control none (cold, serialised launches)\n")
        f.write(f"# {len(dfg)} dfg launches, {tot:.3f} ms; {n_other} torch launches (input generation) "
                f"{other:.3f} ms, not part of the timed step\n")
        f.write("ID,kernel,ms,share_of_dfg_time\n")
        for i, k, ms in dfg:
            f.write(f"{i},{k},{ms:.4f},{ms / tot:.4f}\n")
    print(f"{len(dfg)} dfg launches -> {dst}")


def traffic(rep, n):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, vals = rows[0], rows[2]
    get = lambda k: float(vals[hdr.index(k)].replace(",", ""))
    unit = rows[1][hdr.index("dram__bytes_read.sum")]
    mult = {"Gbyte": 1e9, "Mbyte": 1e6, "byte": 1.0, "Kbyte": 1e3}[unit]
    tb = (get("dram__bytes_read.sum") + get("dram__bytes_write.sum")) * mult
    d = {"n": int(n), "kernel": "dfg_fused_tma", "report": os.path.basename(rep),
         "dram_bytes_per_launch": tb, "duration_ms": get("gpu__time_duration.sum")}
    json.dump(d, open(os.path.join(ROOT, "profiles", "traffic.json"), "w"), indent=1)
    print(d)


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        traffic(sys.argv[2], sys.argv[3])
