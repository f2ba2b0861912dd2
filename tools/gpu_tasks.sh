#!/usr/bin/env bash
# GPU-box task runner (developer tool): `gpurun -- 'bash tools/gpu_tasks.sh TASK [TASK ...]'`.
# Every task writes its logs under gpurun_out/ (merged back by gpurun).
#   full      smoke(), the whole GPU suite, a driver-like bench line
#   tests     the GPU suite only
#   bench     bench.py --steps 20 --warmup 3 (the driver's form)
#   launches  ncu launch list of the bench command (per-launch times, TAG prefix)
#   profile   ncu --set full of the headline kernel (dfg_fused_tma, fused Q 1024^3 fp32)
#   configs   ncu DRAM bytes / instructions per bench configuration -> gpurun_out/r02_configs.md
#   rows      row-class kernel: parity, packed VisIt blocks and 1022^3 timings, one full capture
#   small     config-2 tile / CTA sweep of the 192^3 fused kernel
#   multi     the multi-rank tests (peer / NCCL slabs on one GPU, bench --gpus 2)
#   sanitize  compute-sanitizer memcheck / racecheck / synccheck / initcheck on the pipelines
#             (closed on the round-2 GPU pool: the runs print the pool's notice and exit)
#   sanitize_peer  memcheck + racecheck of the peer halo, each rank under its own sanitizer
set -u
TAG=${TAG:-r02}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { echo build failed; exit 1; }
for task in "$@"; do
  case $task in
  full)
    python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
    timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
    tail -3 gpurun_out/pytest_gpu.log
    timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2> gpurun_out/bench.err; echo bench=$?
    tail -c 300 gpurun_out/bench.log ;;
  tests)
    timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
    tail -3 gpurun_out/pytest_gpu.log ;;
  bench)
    timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2> gpurun_out/bench.err; echo bench=$?
    tail -c 300 gpurun_out/bench.log ;;
  launches)
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:dfg -c 400 --csv \
      --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline \
      --no-strategies > gpurun_out/${TAG}_launches_bench.log 2>&1; echo launches=$? ;;
  profile)
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_tma -s 3 -c 1 \
      -o gpurun_out/prof_${TAG} -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-strategies \
      > gpurun_out/prof_${TAG}.log 2>&1; echo profile=$? ;;
  configs)
    timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__sass_thread_inst_executed.sum \
      --clock-control none -k "regex:dfg|k_" --csv --log-file gpurun_out/${TAG}_cfg.csv python tools/ncu_configs.py \
      > gpurun_out/${TAG}_cfg_order.json 2> gpurun_out/${TAG}_cfg.err; echo configs=$?
    python tools/ncu_configs.py --summarize gpurun_out/${TAG}_cfg.csv gpurun_out/${TAG}_cfg_order.json \
      > gpurun_out/${TAG}_configs.md ;;
  rows)
    timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows_kernel or visit_blocks or extreme or tile_kernel" \
      > gpurun_out/rows_tests.log 2>&1; echo rows_tests=$?; tail -1 gpurun_out/rows_tests.log
    timeout 300 python tools/blocks_overhead.py --pad 0 > gpurun_out/rows_blocks.log 2>&1; tail -1 gpurun_out/rows_blocks.log
    timeout 300 python tools/rows_probe.py --n 1022 > gpurun_out/rows_1022.log 2>&1; tail -1 gpurun_out/rows_1022.log
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_rows_multi -c 1 \
      -o gpurun_out/prof_${TAG}_rows_blocks -f python tools/blocks_overhead.py --pad 0 > gpurun_out/ncu_rows.log 2>&1
    echo rows_profile=$? ;;
  small)
    for e in "" "DFG_CTAS=2 DFG_NCW=8" "DFG_CTAS=2 DFG_NCW=7" "DFG_KZ=16" "DFG_KZ=24" "DFG_STAGES=4" "DFG_NCW=8" "DFG_RPW=4"; do
      env $e timeout 300 python tools/small_probe.py 192 2>/dev/null | grep qcrit
    done > gpurun_out/${TAG}_small.log; cat gpurun_out/${TAG}_small.log ;;
  multi)
    timeout 1500 python -m pytest tests/test_gpu_peer.py tests/test_gpu_nccl.py -q -m gpu > gpurun_out/pytest_multi.log 2>&1
    echo multi=$?; tail -3 gpurun_out/pytest_multi.log ;;
  sanitize)
    for t in memcheck racecheck synccheck initcheck; do
      timeout 900 compute-sanitizer --tool $t python tools/sanitize_run.py > gpurun_out/san_$t.log 2>&1; echo $t=$?
      grep -E "ERROR SUMMARY|RACECHECK SUMMARY|hazard|sanitize run done" gpurun_out/san_$t.log | tail -3
    done ;;
  sanitize_peer)
    for t in memcheck racecheck; do
      for r in 0 1; do
        timeout 600 compute-sanitizer --tool $t python tools/peer_ranks.py --ranks 2 --n 64 --nz 13 --steps 2 \
          --as-rank $r --port 29733 > gpurun_out/san_peer_${t}_r$r.log 2>&1 &
      done
      wait
      for r in 0 1; do echo "$t rank $r:"; grep -E "SUMMARY|bit_identical" gpurun_out/san_peer_${t}_r$r.log | tail -2; done
    done ;;
  *) echo "unknown task $task" ;;
  esac
done
