# A/B of the cp.async-filled tile kernel: .ab/fused_tma_{old,new}.cuh (inside the snapshot: gpurun_out/ does not travel) on
# ragged (1022^3) and forced-tile (1024^3) meshes and packed VisIt shells
C=paper_conf_sc_harrisonnmjc12_b200/csrc
for v in new old; do
  cp .ab/fused_tma_$v.cuh $C/fused_tma.cuh
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
  echo "== $v"
  timeout 300 python tools/sweep.py --n 1022 --iters 100 --configs ";" 2>&1 | tail -2
  timeout 300 python tools/sweep.py --n 1024 --iters 100 --configs "DFG_FUSED_KERNEL=tile" 2>&1 | tail -2
  timeout 300 python tools/blocks_overhead.py --pad 0 2>&1 | tail -1
done > gpurun_out/ab_tile.log
cp .ab/fused_tma_new.cuh $C/fused_tma.cuh
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1


