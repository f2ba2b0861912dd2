python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/peer_ranks.py --ranks 2 --n 64 --nz 29 > gpurun_out/peer1.log 2>&1; echo peer=$?
tail -30 gpurun_out/peer1.log
timeout 900 python -m pytest tests/test_gpu_peer.py -x -q > gpurun_out/peer_tests.log 2>&1; echo tests=$?
tail -30 gpurun_out/peer_tests.log
