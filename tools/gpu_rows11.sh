python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows_kernel or visit_blocks or extreme or tile_kernel or tma_and_general" > gpurun_out/rows_tests11.log 2>&1; echo tests=$?; tail -1 gpurun_out/rows_tests11.log
timeout 300 python tools/blocks_overhead.py --pad 0 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('packed', d['gcells_s_batched'], d['batched_variant'], d['bit_identical'])"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_rows_multi -c 1 -o gpurun_out/prof_r02_rows_blocks11 python tools/blocks_overhead.py --pad 0 > gpurun_out/ncu_rows11.log 2>&1; echo ncu=$?
