"""Debug: which cells of the one-launch multi-block tile kernel differ."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
sys.path.insert(0, os.path.join(os.path.dirname(__file__), "..", "tests"))
import numpy as np, torch
import paper_conf_sc_harrisonnmjc12_b200 as dfg
import synth
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}
from dfg_testutil import run_lib

shape = (62, 30, 20); split = tuple(int(c) for c in os.environ.get("SPLIT", "222"))
x, y, z, f = synth.rt_inputs(*shape, dtype=np.float32, names=("u", "v", "w"))
f = {k: v.numpy() for k, v in f.items()}
src = PAPER_PROGRAMS[sys.argv[1] if len(sys.argv) > 1 else "qcrit"][0]
whole = run_lib(src, f, x, y, z, "fused")
cuts = [np.linspace(0, n, s + 1).astype(int) for n, s in zip(shape, split)]
pad = {n: np.pad(a, 1, mode="edge") for n, a in f.items()}
blocks = []
for a in range(split[0]):
    for b in range(split[1]):
        for c in range(split[2]):
            i0, i1 = cuts[0][a], cuts[0][a + 1]; j0, j1 = cuts[1][b], cuts[1][b + 1]; k0, k1 = cuts[2][c], cuts[2][c + 1]
            bx = i1 - i0; padded = os.environ.get("PITCH") == "padded"; xo = 4 if padded else 1; rp = (xo + bx + 1 + 3) // 4 * 4 + 4 if padded else bx + 2
            m = dfg.Mesh.block(x, y, z, bx, j1 - j0, k1 - k0, i0, j0, k0, ghost=1, row_pitch=rp, x_offset=xo)
            keep = []
            for n in ("u", "v", "w"):
                buf = np.full((k1 - k0 + 2, j1 - j0 + 2, rp), np.nan, np.float32)
                buf[:, :, xo - 1:xo + bx + 1] = pad[n][k0:k1 + 2, j0:j1 + 2, i0:i1 + 2]
                t = torch.from_numpy(buf).cuda(); keep.append(t); m.bind(n, t)
            p = dfg.Plan(m, src, "fused")
            o = torch.full((k1 - k0, j1 - j0, bx), float("nan"), device="cuda")
            blocks.append((p, o, (k0, k1, j0, j1, i0, i1), m, keep))
dfg.execute_blocks([b[0] for b in blocks], [b[1] for b in blocks])
torch.cuda.synchronize()
print("variant", blocks[0][0].info())
for bi, (p, o, (k0, k1, j0, j1, i0, i1), _, _) in enumerate(blocks):
    g = o.cpu().numpy(); w = whole[k0:k1, j0:j1, i0:i1]
    bad = np.argwhere(~(g == w))
    print(f"block {bi} k{k0}:{k1} j{j0}:{j1} i{i0}:{i1} bad {len(bad)} of {g.size}")
    if len(bad):
        print("  planes", np.unique(bad[:, 0]), "rows", np.unique(bad[:, 1])[:20], "cols", np.unique(bad[:, 2])[:40])
        kk, jj, ii = bad[0]; print("  first", bad[0], g[kk, jj, ii], w[kk, jj, ii])
