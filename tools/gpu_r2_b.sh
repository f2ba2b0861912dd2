python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows_kernel or visit_blocks or extreme or tile_kernel or tma_and_general" > gpurun_out/rows_tests12.log 2>&1; echo tests=$?; tail -1 gpurun_out/rows_tests12.log
timeout 300 python tools/blocks_overhead.py --pad 0 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('packed', d['gcells_s_batched'], d['batched_variant'], d['bit_identical'])"
timeout 300 python tools/rows_probe.py --n 1022 --kernels rows | tail -1
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__sass_thread_inst_executed.sum --clock-control none -k "regex:dfg|k_" --csv --log-file gpurun_out/r02_cfg.csv python tools/ncu_configs.py > gpurun_out/r02_cfg_order.json 2> gpurun_out/r02_cfg.err; echo cfg=$?
python tools/ncu_configs.py --summarize gpurun_out/r02_cfg.csv gpurun_out/r02_cfg_order.json > gpurun_out/r02_configs.md; echo sum=$?
