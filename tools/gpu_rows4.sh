python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows or extreme or visit_blocks or tile_kernel" > gpurun_out/rows_tests4.log 2>&1; echo tests=$?
tail -3 gpurun_out/rows_tests4.log
for p in 0; do timeout 300 python tools/blocks_overhead.py --pad $p; done > gpurun_out/blocks_perf4.log 2>&1
cat gpurun_out/blocks_perf4.log
timeout 300 python tools/rows_probe.py --n 1022 > gpurun_out/rows_probe4.log 2>&1; tail -1 gpurun_out/rows_probe4.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_rows_multi -c 1 -o gpurun_out/prof_r02_rows_blocks python tools/blocks_overhead.py --pad 0 > gpurun_out/ncu_rows4.log 2>&1; echo ncu=$?
