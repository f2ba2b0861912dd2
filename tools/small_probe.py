"""Config-2 style timing of the fused kernel on small meshes (device time
behind a sleep, clean-cold L2, 7-run trimmed mean) -- for tile / CTA shape
experiments via DFG_NCW / DFG_CTAS / DFG_RPW / DFG_STAGES."""
import json, os, sys
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import torch
import paper_conf_sc_harrisonnmjc12_b200 as dfg
import synth
from bench import _strategies_at
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}

for n in [int(a) for a in (sys.argv[1:] or ["192", "256"])]:
    for prog in ("vortmag", "qcrit"):
        r = _strategies_at(dfg, synth, torch, n, PAPER_PROGRAMS[prog][0], ("fused",), 7)["fused"]
        print(json.dumps({"n": n, "prog": prog, "env": {k: v for k, v in os.environ.items() if k.startswith("DFG_")},
                          "us": round(r["ms"] * 1e3, 2), "parity_bad": r["oracle_parity"]["mismatches"]}), flush=True)
