"""Config-2 roundtrip timings (developer tool): the paper's roundtrip strategy
at n^3 fp32 for VelMag / VortMag / Q with the config-2 protocol of bench.py.

    python tools/roundtrip_probe.py [n]
"""
import json
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch  # noqa: E402
import paper_conf_sc_harrisonnmjc12_b200 as dfg  # noqa: E402
import synth  # noqa: E402
from bench import _strategies_at  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 192
for prog in ("velmag", "vortmag", "qcrit"):
    r = _strategies_at(dfg, synth, torch, n, dfg.paper_program(prog), ("fused", "roundtrip"), 7)
    rt = r["roundtrip"]
    print(json.dumps({"n": n, "prog": prog, "roundtrip_ms": round(rt["ms"], 3),
                      "bit_identical_to_fused": rt["bit_identical_to_fused"], "pcie_bytes": rt["pcie_bytes"]}))
