python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for l in 0 1 2; do DFG_TIMING_LEVEL=$l timeout 300 python tools/launch_overhead.py | grep amortized; done > gpurun_out/launch3.log 2>&1
cat gpurun_out/launch3.log
timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline > gpurun_out/bench2.log 2>gpurun_out/bench2.err; echo bench=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench2.log').read().strip().splitlines()[-1])
print(d['value'], d['roofline']['frac'], d['clocks'])
c=d['strategies']['config2_192']
for e in c:
  if isinstance(c[e], dict): print(e, {k:(v['ms'] if isinstance(v,dict) and 'ms' in v else None) for k,v in c[e].items()})
"
