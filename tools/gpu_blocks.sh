python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "visit_blocks or tile" > gpurun_out/blocks_tests.log 2>&1; echo tests=$?
tail -3 gpurun_out/blocks_tests.log
for p in 0 1; do timeout 300 python tools/blocks_overhead.py --pad $p; done > gpurun_out/blocks_perf.log 2>&1
cat gpurun_out/blocks_perf.log
