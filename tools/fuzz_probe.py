"""Print the cells where a fused plan differs from the oracle for one
program (developer tool).  python tools/fuzz_probe.py 'src' nx ny nz f32|f64 [variant]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import synth  # noqa: E402
from dfg_testutil import run_lib, run_oracle  # noqa: E402

src, nx, ny, nz, dt = sys.argv[1].replace("\\n", "\n"), *map(int, sys.argv[2:5]), sys.argv[5]
if len(sys.argv) > 6:
    os.environ["DFG_FUSED_VARIANT"] = sys.argv[6]
T = np.float32 if dt == "f32" else np.float64
x, y, z, f = synth.rt_inputs(nx, ny, nz, dtype=T)
f = {k: v.numpy() for k, v in f.items()}
want = run_oracle(src, f, x, y, z)
got, plan, *_ = run_lib(src, f, x, y, z, "fused", return_plan=True)
u = np.uint32 if T == np.float32 else np.uint64
bad = (got.view(u) != want.view(u)) & ~(np.isnan(got) & np.isnan(want))
print("variant", plan.info()["variant"], "arith", plan.arith(), "mismatches", int(bad.sum()), "of", bad.size)
for idx in list(zip(*np.nonzero(bad)))[:10]:
    print(idx, repr(got[idx]), repr(want[idx]))
