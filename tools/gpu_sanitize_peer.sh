python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for t in memcheck racecheck; do
  for r in 0 1; do
    timeout 600 compute-sanitizer --tool $t python tools/peer_ranks.py --ranks 2 --n 64 --nz 13 --steps 2 --as-rank $r --port 29733 > gpurun_out/san_peer_${t}_r$r.log 2>&1 &
  done
  wait
  for r in 0 1; do echo "$t rank $r:"; grep -E "SUMMARY|bit_identical" gpurun_out/san_peer_${t}_r$r.log | tail -2; done
done
