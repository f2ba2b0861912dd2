"""Write tests/golden/dag_*.txt from the ORACLE (oracle.lang) only.

Run:  python tools/make_golden.py
The dumps are pinned independently by tests/test_oracle_lang.py (Table II,
filter counts, head/tail structure of the completed Fig. 3C network).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle.lang import PAPER_PROGRAMS, build_dag  # noqa: E402

for name, (src, inputs) in PAPER_PROGRAMS.items():
    for dt in ("f32", "f64"):
        path = os.path.join(ROOT, "tests", "golden", f"dag_{name}_{dt}.txt")
        with open(path, "w") as f:
            f.write(build_dag(src, inputs, dt).dump())
        print("wrote", path)
