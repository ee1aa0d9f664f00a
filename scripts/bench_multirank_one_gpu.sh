# the N = 2 / 4 bench path (torchrun, one rank per process, p2p transport) on the one GPU a
# gpurun box has: every rank shares the device, so the numbers are not scaling data -- this
# (SF_BENCH_SHARED_GPU=1: every rank on cuda:0) checks that the multi-rank launch, exchanges, max-over-ranks timing and JSON line work
for n in 2 4; do
SF_BENCH_SHARED_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus $n --steps 3 --warmup 3 --quick > gpurun_out/bench_n$n.json 2> gpurun_out/bench_n$n.err
echo "N=$n rc=$?"; head -c 600 gpurun_out/bench_n$n.json; echo
done
