python -c "import __graft_entry__ as g; g.build()" >/dev/null
for e in "" "DFG_NCW=7,DFG_CTAS=2" "DFG_NCW=7,DFG_CTAS=2,DFG_RPW=2" "DFG_RPW=2" "DFG_STAGES=10" "DFG_NCW=12" "DFG_NCW=7,DFG_CTAS=2,DFG_STAGES=5"; do
  EXTRA=$e timeout 100 python tools/power_probe.py qcrit 2>&1 | tail -1
done > gpurun_out/sweep1.log
