"""Config-2 floor probe (developer tool): what does a plain 3-read / 1-write
streaming op cost on an n^3 fp32 mesh under the config-2 protocol (L2 flushed
and clean, enqueued behind a device sleep, 7 runs, trimmed mean)?  Printed
beside the library's fused VelMag / VortMag / Q at the same size, so the
small-mesh gap can be split into "any 16 B/cell stream at this size" and
"the stencil kernel's own overhead".

    python tools/small_floor.py 192 256 384
"""
import json, os, sys
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import torch
import paper_conf_sc_harrisonnmjc12_b200 as dfg
import synth
from bench import _strategies_at

PROGS = {k: dfg.paper_program(k) for k in ("velmag", "vortmag", "qcrit")}


def timed(fn, runs=7):
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    clean = torch.ones(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    t = []
    for _ in range(runs):
        flush.zero_()
        clean.sum()
        torch.cuda.synchronize()
        torch.cuda._sleep(2_000_000)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        t.append(e0.elapsed_time(e1))
    t = sorted(t)[1:-1]
    return sum(t) / len(t)


for n in [int(a) for a in (sys.argv[1:] or ["192", "256"])]:
    u, v, w, o = (torch.rand((n, n, n), device="cuda") for _ in range(4))
    ms = timed(lambda: torch.addcmul(u, v, w, out=o))
    print(json.dumps({"n": n, "op": "torch.addcmul (3 reads, 1 write)", "us": round(ms * 1e3, 2),
                      "gb_per_s": round(16 * n ** 3 / (ms * 1e-3) / 1e9, 1)}), flush=True)
    ms = timed(lambda: o.copy_(u))
    print(json.dumps({"n": n, "op": "torch copy_ (1 read, 1 write)", "us": round(ms * 1e3, 2),
                      "gb_per_s": round(8 * n ** 3 / (ms * 1e-3) / 1e9, 1)}), flush=True)
    del u, v, w, o
    torch.cuda.empty_cache()
    for prog, src in PROGS.items():
        r = _strategies_at(dfg, synth, torch, n, src, ("fused",), 7)["fused"]
        print(json.dumps({"n": n, "op": f"fused {prog}", "us": round(r["ms"] * 1e3, 2),
                          "gb_per_s": round(16 * n ** 3 / (r["ms"] * 1e-3) / 1e9, 1),
                          "parity_bad": r["oracle_parity"]["mismatches"]}), flush=True)
