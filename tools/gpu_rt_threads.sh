python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
nproc
for t in 32 16 8 4; do DFG_HOST_THREADS=$t timeout 600 python -c "
import sys, json, torch, os; sys.path.insert(0, '.')
import paper_conf_sc_harrisonnmjc12_b200 as dfg, synth, bench
PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}
for name in ('vortmag', 'qcrit'):
    r = bench._strategies_at(dfg, synth, torch, 192, PAPER_PROGRAMS[name][0], ('roundtrip',), 5)
    print(os.environ['DFG_HOST_THREADS'], name, round(r['roundtrip']['ms'], 2))
"; done
