python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
C="DFG_FUSED_VARIANT=exact;DFG_FUSED_VARIANT=fast;DFG_NCW=7,DFG_CTAS=2;DFG_NCW=7,DFG_CTAS=2,DFG_STAGES=5;DFG_NCW=11;DFG_NCW=12;DFG_STAGES=10;DFG_STAGES=4;DFG_FUSED_VARIANT=exact"
timeout 600 python tools/sweep.py --iters 300 --configs "$C" > gpurun_out/sweep1.log 2>&1
timeout 300 python tools/sweep.py --iters 300 --expr vortmag --configs "DFG_FUSED_VARIANT=exact" >> gpurun_out/sweep1.log 2>&1
timeout 300 python tools/sweep.py --iters 300 --expr velmag --configs "DFG_FUSED_VARIANT=exact" >> gpurun_out/sweep1.log 2>&1
cat gpurun_out/sweep1.log
