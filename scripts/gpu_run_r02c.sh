cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r3
for k in 0 1; do
SF_COARSE_KERNEL=$k timeout 300 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r3/v64_k$k.csv python scripts/vcycle_once_n.py 64 > gpurun_out/r3/v64_k$k.log 2>&1
done
python scripts/launch_list.py gpurun_out/r3/v64_k0.csv > gpurun_out/r3/v64_k0.txt 2>&1
python scripts/launch_list.py gpurun_out/r3/v64_k1.csv > gpurun_out/r3/v64_k1.txt 2>&1
