python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python bench.py > gpurun_out/bench3.log 2>gpurun_out/bench3.err; echo bench=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench3.log').read().strip().splitlines()[-1])
print(d['value'], d['roofline']['frac'], d['clocks']); print(json.dumps(d['cpu_baseline']))"
tail -3 gpurun_out/bench3.err
bash tools/gpu_sanitize_peer.sh
