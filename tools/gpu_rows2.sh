python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows or extreme or visit_blocks" > gpurun_out/rows_tests2.log 2>&1; echo tests=$?
tail -5 gpurun_out/rows_tests2.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_rows -c 1 -o gpurun_out/prof_r02_rows1022 python tools/rows_probe.py --n 1022 --iters 1 --kernels rows > gpurun_out/ncu_rows.log 2>&1; echo ncu1=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused -c 1 -o gpurun_out/prof_r02_tile1022 python tools/rows_probe.py --n 1022 --iters 1 --kernels tile >> gpurun_out/ncu_rows.log 2>&1; echo ncu2=$?
tail -3 gpurun_out/ncu_rows.log
