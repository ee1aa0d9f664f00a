cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
timeout 900 python -m pytest tests -m gpu -q -x -k "coarse or dead_peer" > gpurun_out/r2/t.log 2>&1; echo "rc=$?" >> gpurun_out/r2/t.log
timeout 600 python scripts/coarse_ab.py > gpurun_out/r2/coarse_ab.txt 2>&1
tail -3 gpurun_out/r2/t.log; cat gpurun_out/r2/coarse_ab.txt
