python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows_per_warp or tile_shape or fast_variant or visit_blocks or parity_paper or z_chunking" > gpurun_out/rpw_tests.log 2>&1; echo tests=$?
tail -3 gpurun_out/rpw_tests.log
timeout 600 python tools/small_mesh.py --configs ";DFG_RPW=1;DFG_RPW=4" > gpurun_out/small3.log 2>&1
cat gpurun_out/small3.log
