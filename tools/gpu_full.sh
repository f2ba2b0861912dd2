# full GPU suite, smoke, default bench, and the launch list of the bench command (dfg kernels)
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1800 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.log 2>gpurun_out/bench.err; echo bench=$?
tail -c 400 gpurun_out/bench.log
TAG=${TAG:-r01i}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:dfg --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-strategies \
  > gpurun_out/${TAG}_launches_bench.log 2>&1; echo launches=$?
