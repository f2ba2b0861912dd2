python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_rows_multi -c 1 -o gpurun_out/prof_r02_rows_blocks9 python tools/blocks_overhead.py --pad 0 > gpurun_out/ncu_rows9.log 2>&1; echo ncu=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_rows -c 1 -o gpurun_out/prof_r02_rows1022_9 python tools/rows_probe.py --n 1022 --iters 1 --kernels rows >> gpurun_out/ncu_rows9.log 2>&1; echo ncu=$?
