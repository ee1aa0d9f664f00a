cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r5
for m in 8 1; do echo "SF_GSRB_MIND=$m"; SF_GSRB_MIND=$m timeout 300 python scripts/coarse_ab.py 64 128 256; done > gpurun_out/r5/mind_ab.txt 2>&1
for m in 8 1; do SF_GSRB_MIND=$m SF_COARSE_KERNEL=1 timeout 300 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r5/v64_m$m.csv python scripts/vcycle_once_n.py 64 > /dev/null 2>&1; python scripts/launch_list.py gpurun_out/r5/v64_m$m.csv > gpurun_out/r5/v64_m$m.txt; done
cat gpurun_out/r5/mind_ab.txt gpurun_out/r5/v64_m1.txt
