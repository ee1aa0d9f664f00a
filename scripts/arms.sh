python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
nproc; free -g | head -2
( time timeout 900 python bench.py --impl reference --steps 2 --warmup 1 ) > gpurun_out/ref.json 2> gpurun_out/ref.err
tail -4 gpurun_out/ref.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 3 --warmup 3 --quick > gpurun_out/trun.json 2> gpurun_out/trun.err
echo "torchrun exit $?"; tail -3 gpurun_out/trun.err
