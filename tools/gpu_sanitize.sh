python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for t in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $t python tools/sanitize_run.py > gpurun_out/san_$t.log 2>&1; echo $t=$?
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|hazard|sanitize run done" gpurun_out/san_$t.log | tail -3
done
timeout 900 compute-sanitizer --tool memcheck --target-processes all python tools/peer_ranks.py --ranks 2 --n 64 --nz 13 --steps 2 > gpurun_out/san_peer.log 2>&1; echo peer_memcheck=$?
grep -E "ERROR SUMMARY|bit_identical" gpurun_out/san_peer.log | tail -4
