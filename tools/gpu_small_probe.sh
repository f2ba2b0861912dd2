# tile-shape experiments on small and mid-size meshes (tools/small_probe.py)
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for e in ${CASES:-"_" "DFG_NCW=12"}; do
  env $( [ "$e" = "_" ] || echo $e ) timeout 300 python tools/small_probe.py ${SIZES:-192 256} 2>&1 | grep '"n"'
done > gpurun_out/small.log
