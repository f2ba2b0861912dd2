python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for a in "1 0" "1 3" "1 1" "1 -3" "1 5" "3 4" "3 1" "3 -3"; do timeout 30 tools/tma_probe $a; done > gpurun_out/tma_probe.log 2>&1
cat gpurun_out/tma_probe.log
timeout 900 python -m pytest tests/ -x -q -m gpu > gpurun_out/pytest_gpu2.log 2>&1; echo tests=$?
tail -3 gpurun_out/pytest_gpu2.log
for n in 32 64 96; do timeout 300 python tools/small_mesh.py --n $n --exprs velmag,qcrit; done > gpurun_out/small4.log 2>&1
cat gpurun_out/small4.log
