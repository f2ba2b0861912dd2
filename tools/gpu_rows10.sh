python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do DFG_RPW=$r timeout 300 python tools/blocks_overhead.py --pad 0 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rpw', $r, d['gcells_s_batched'], d['batched_variant'], d['bit_identical'])"; done
for r in 1 2; do DFG_RPW=$r timeout 300 python tools/blocks_overhead.py --pad 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('padded rpw', $r, d['gcells_s_batched'], d['batched_variant'], d['bit_identical'])"; done
