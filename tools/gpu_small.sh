python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python tools/small_mesh.py --configs ";DFG_NCW=12" > gpurun_out/small2.log 2>&1
cat gpurun_out/small2.log
