# ncu evidence for profiles/: launch list of the bench command, one full
# capture of the top kernel (dfg_fused_tma, fused Q 1024^3 fp32)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
TAG=${TAG:-r01h}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:dfg -c 400 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-strategies \
  > gpurun_out/${TAG}_launches_bench.log 2>&1; echo launches=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfg_fused_tma -s 3 -c 1 \
  -o gpurun_out/prof_${TAG} -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-strategies \
  > gpurun_out/prof_${TAG}.log 2>&1; echo full=$?
ls -la gpurun_out/
