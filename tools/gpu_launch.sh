python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/launch_overhead.py > gpurun_out/launch.log 2>&1
cat gpurun_out/launch.log
