python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/blocks_overhead.py --pad 0 > gpurun_out/blocks_perf8.log 2>&1; tail -1 gpurun_out/blocks_perf8.log
timeout 300 python tools/rows_probe.py --n 1022 > gpurun_out/rows_probe8.log 2>&1; tail -1 gpurun_out/rows_probe8.log
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "rows_kernel or visit_blocks or extreme or tile_kernel" > gpurun_out/rows_tests8.log 2>&1; echo tests=$?; tail -1 gpurun_out/rows_tests8.log
