python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
DFG_DEBUG=1 timeout 300 python tools/rows_probe.py --n 1022 --kernels rows > gpurun_out/rows_probe5.log 2>&1; tail -3 gpurun_out/rows_probe5.log
DFG_DEBUG=1 timeout 300 python tools/blocks_overhead.py --pad 0 > gpurun_out/blocks_perf5.log 2>&1; tail -3 gpurun_out/blocks_perf5.log
