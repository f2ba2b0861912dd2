python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python tools/parity_probe.py > gpurun_out/parity_probe.log 2>&1; echo probe=$?
cat gpurun_out/parity_probe.log | cut -c1-1500
