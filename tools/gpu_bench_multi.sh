python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for H in peer nccl; do
DFG_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 2 --steps 5 --warmup 3 --size 256 --halo $H > gpurun_out/bench_multi_$H.log 2> gpurun_out/bench_multi_$H.err; echo multi_$H=$?
tail -c 1500 gpurun_out/bench_multi_$H.log
tail -5 gpurun_out/bench_multi_$H.err
done
