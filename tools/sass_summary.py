"""SASS summaries of the kernels on the hot path (host only, developer tool).

    python tools/sass_summary.py > profiles/r02_sass.md

Generated fused kernels (the library's own generator, dfg_fused_source, for
the bench meshes) are compiled with nvcc for sm_100a with the NVRTC options
of csrc/jit.cpp; the per-primitive staged kernels come from the library's
object file (csrc/build/kernels.cu.o).  Per kernel: registers, spills and the
count of the instructions that prove the design (UTMALDG: TMA tensor loads,
UBLKCP: bulk copies, LDGSTS: cp.async, SYNCS: mbarrier operations, FFMA2 /
FADD2: paired FP32, LDS / STS / STG: shared / global traffic; static counts
of the SASS text, not executions).
"""
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_harrisonnmjc12_b200 as dfg  # noqa: E402

OPTS = ["-gencode", "arch=compute_100a,code=sm_100a", "-std=c++17", "--fmad=false", "-ftz=false",
        "-prec-div=true", "-prec-sqrt=true", "-cubin", "-Xptxas", "-v"]
OPS = ["UTMALDG", "UBLKCP", "LDGSTS", "SYNCS", "FFMA2", "FADD2", "FFMA", "FADD", "FMUL", "DFMA", "DADD", "DMUL",
       "LDS", "STS", "LDG", "STG", "SHFL", "BAR"]


def sass_counts(cubin, fn):
    out = subprocess.run(["cuobjdump", "-sass", "-fun", fn, cubin], capture_output=True, text=True).stdout
    ops = re.findall(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P[0-9T]\s+)?([A-Z0-9_]+)", out)
    cnt = {o: 0 for o in OPS}
    for o in ops:
        if o in cnt:
            cnt[o] += 1
    return cnt, len(ops)


def ptxas_info(log):
    info, fn = {}, None
    for line in log.splitlines():
        m = re.search(r"entry function '([^']+)'", line)
        if m:
            fn = m.group(1)
        m = re.search(r"Used (\d+) registers", line)
        if m and fn:
            info.setdefault(fn, {})["regs"] = int(m.group(1))
        m = re.search(r"(\d+) bytes spill stores", line)
        if m and fn:
            info.setdefault(fn, {})["spill"] = int(m.group(1))
    return info


def main():
    rows = []
    # (the packed-shell case: the paper's 192 x 192 x 256 block with its one-cell x
    # offset runs the row-class kernel; forced here since the source has no pitch)
    cases = [("qcrit", 0, (1024, 1024, 1024)), ("qcrit", 1, (768, 768, 768)), ("qcrit", 0, (192, 192, 256)),
             ("qcrit", 0, (1022, 1022, 1022)), ("vortmag", 0, (768, 768, 768)), ("intro", 0, (768, 768, 768)),
             ("velmag", 0, (768, 768, 768)), ("qcrit packed shells", 0, (192, 192, 256)),
             ("qcrit packed shells", 1, (192, 192, 256))]
    with tempfile.TemporaryDirectory() as td:
        for name, dt, dims in cases:
            prog = name.split()[0]
            src = dfg.paper_program(prog)
            if "packed" in name:
                os.environ["DFG_FUSED_KERNEL"] = "rows"
            code, _, _ = dfg.dfg_fused_source(src, dfg.PAPER_INPUTS[prog], dt, *dims)
            os.environ.pop("DFG_FUSED_KERNEL", None)
            cu = os.path.join(td, "k.cu")
            open(cu, "w").write(code)
            cub = os.path.join(td, "k.cubin")
            r = subprocess.run(["nvcc"] + OPTS + ["-o", cub, cu], capture_output=True, text=True)
            info = ptxas_info(r.stderr + r.stdout)
            for fn in ("dfg_fused_tma", "dfg_fused_rows", "dfg_fused_tile", "dfg_fused_general", "dfg_fused_pointwise"):
                if fn not in info:
                    continue
                cnt, tot = sass_counts(cub, fn)
                rows.append((f"{name} {'f32' if dt == 0 else 'f64'} {'x'.join(map(str, dims))}", fn, info[fn], cnt, tot))
    obj = os.path.join(ROOT, "paper_conf_sc_harrisonnmjc12_b200", "csrc", "build", "kernels.cu.o")
    fns = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True).stdout
    for fn in sorted(set(re.findall(r"Function : (\S+)", fns))):
        if "grad3d" in fn or "binary" in fn:
            cnt, tot = sass_counts(obj, fn)
            name = subprocess.run(["c++filt", fn], capture_output=True, text=True).stdout.strip()
            name = re.sub(r"\(anonymous namespace\)::|dfg::kern::", "", name).split("(")[0]
            rows.append(("staged primitive", name, {}, cnt, tot))
    print("# SASS summaries (static instruction counts; `tools/sass_summary.py`)\n")
    print("| case | kernel | regs | spill B | SASS | " + " | ".join(OPS) + " |")
    print("|---|---|---|---|---|" + "---|" * len(OPS))
    for case, fn, info, cnt, tot in rows:
        print(f"| {case} | {fn} | {info.get('regs', '')} | {info.get('spill', '')} | {tot} | "
              + " | ".join(str(cnt[o]) for o in OPS) + " |")


if __name__ == "__main__":
    main()
