cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r4
timeout 300 python scripts/coarse_ab.py 64 128 > gpurun_out/r4/coarse_ab.txt 2>&1
SF_COARSE_KERNEL=1 timeout 300 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r4/v64.csv python scripts/vcycle_once_n.py 64 > /dev/null 2>&1
python scripts/launch_list.py gpurun_out/r4/v64.csv > gpurun_out/r4/v64.txt
SF_COARSE_KERNEL=1 timeout 300 ncu --profile-from-start off -k regex:coarse --set full --import-source on --clock-control none -o gpurun_out/r4/coarse python scripts/vcycle_once_n.py 64 > /dev/null 2>&1
python scripts/ncu_lines.py gpurun_out/r4/coarse.ncu-rep 0 30 > gpurun_out/r4/coarse_lines.txt 2>&1
cat gpurun_out/r4/coarse_ab.txt gpurun_out/r4/v64.txt gpurun_out/r4/coarse_lines.txt
