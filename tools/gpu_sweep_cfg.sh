# A/B of fused-kernel build options on the 1024^3 Q bench workload (power_probe: 1.5 s back to back per case)
python -c "import __graft_entry__ as g; g.build()" >/dev/null
for e in ${CASES:-"" "DFG_XPAIR=1" "" "DFG_XPAIR=1"}; do
  EXTRA=$e timeout 100 python tools/power_probe.py qcrit 2>&1 | tail -1
done > gpurun_out/sweep_cfg.log
