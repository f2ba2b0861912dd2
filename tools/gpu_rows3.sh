python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows or extreme or visit_blocks or tile_kernel" > gpurun_out/rows_tests3.log 2>&1; echo tests=$?
tail -5 gpurun_out/rows_tests3.log
for p in 0; do timeout 300 python tools/blocks_overhead.py --pad $p; done > gpurun_out/blocks_perf3.log 2>&1
cat gpurun_out/blocks_perf3.log
timeout 300 python tools/rows_probe.py --n 1022 > gpurun_out/rows_probe3.log 2>&1; tail -2 gpurun_out/rows_probe3.log
timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -x -q -k "test_rows_kernel and qcrit and float32 and (67 or 197 or 258)" > gpurun_out/rows_memcheck3.log 2>&1; echo memcheck=$?
grep -E "ERROR SUMMARY|passed|failed" gpurun_out/rows_memcheck3.log | tail -3
