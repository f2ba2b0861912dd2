# A/B of two fused_tma.cuh versions (gpurun_out/ab/fused_tma_{old,new}.cuh) on the
# 1024^3 bench workload: power_probe cases, alternating builds.
C=paper_conf_sc_harrisonnmjc12_b200/csrc
for round in 1 2; do
  for v in old new; do
    cp gpurun_out/ab/fused_tma_$v.cuh $C/fused_tma.cuh
    python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
    echo "== $v round $round"
    timeout 200 python tools/power_probe.py ${CASES:-qcrit vortmag} 2>&1 | grep case
  done
done > gpurun_out/ab.log
cp gpurun_out/ab/fused_tma_new.cuh $C/fused_tma.cuh
