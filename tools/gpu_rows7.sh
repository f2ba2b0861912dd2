python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_rows -c 1 -o gpurun_out/prof_r02_rows8 python tools/rows_probe.py --n 1022 --iters 1 --kernels rows > gpurun_out/ncu_rows8.log 2>&1; echo ncu=$?
