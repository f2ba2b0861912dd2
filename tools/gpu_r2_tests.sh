# round 2: targeted GPU tests first (fast fail), then the full GPU suite
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python -m pytest tests/test_gpu_peer.py tests/test_gpu_nccl.py -x -q -m gpu > gpurun_out/pytest_multi.log 2>&1; echo multi=$?
tail -5 gpurun_out/pytest_multi.log
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "graph_replay or odd_plane or zslab or highwater or streamed" > gpurun_out/pytest_sel.log 2>&1; echo sel=$?
tail -5 gpurun_out/pytest_sel.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_gpu.log
