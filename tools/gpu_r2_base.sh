nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
lscpu | head -20 > gpurun_out/lscpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/bench0.log 2>gpurun_out/bench0.err; echo bench=$?
tail -c 300 gpurun_out/bench0.log
