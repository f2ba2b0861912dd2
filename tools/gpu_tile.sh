python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tile or tma_and_general or visit_blocks or parity_paper" > gpurun_out/tile_tests.log 2>&1; echo tests=$?
tail -15 gpurun_out/tile_tests.log
timeout 300 python tools/sweep.py --n 1022 --iters 100 --configs ";DFG_FUSED_KERNEL=general" > gpurun_out/tile_perf.log 2>&1
timeout 300 python tools/sweep.py --n 1024 --iters 100 --configs ";DFG_FUSED_KERNEL=tile" >> gpurun_out/tile_perf.log 2>&1
cat gpurun_out/tile_perf.log
