cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r1
timeout 900 python -m pytest tests -m gpu -q -k "headline_builds or multigpu_readiness" > gpurun_out/r1/t_new.log 2>&1; echo "new rc=$?" >> gpurun_out/r1/t_new.log
timeout 300 python scripts/pair_headroom.py 256 512 > gpurun_out/r1/headroom.txt 2>&1
timeout 300 python scripts/e2e_phases.py > gpurun_out/r1/e2e.txt 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/r1/bench.json 2> gpurun_out/r1/bench.err
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r1/t_all.log 2>&1; echo "all rc=$?" >> gpurun_out/r1/t_all.log
tail -3 gpurun_out/r1/t_new.log gpurun_out/r1/t_all.log; cat gpurun_out/r1/headroom.txt gpurun_out/r1/e2e.txt
