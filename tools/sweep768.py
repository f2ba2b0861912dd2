"""Config 5 sweep only (768^3, fp32 + fp64, fused): prints one JSON line."""
import json, os, sys
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import torch
import paper_conf_sc_harrisonnmjc12_b200 as dfg
import synth
from bench import complexity_sweep

res = complexity_sweep(dfg, synth, torch)
print(json.dumps({k: {"ms": round(v["kernel_ms"], 4), "gbs": round(v["algorithmic_gb_per_s"])} for k, v in res.items()}))
