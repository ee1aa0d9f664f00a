# coarse V-cycle kernel: parity tests, solve A/B, warm launch lists of one V-cycle
set -x
timeout 900 python -m pytest tests/test_gpu_coarse.py -x -q 2>&1 | tail -5
timeout 300 python scripts/coarse_ab.py 64 128 256 2>&1
for n in 64 128; do
timeout 300 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/vc_warm_$n.csv python scripts/vcycle_once_n.py $n > /dev/null 2>&1
python scripts/launch_list.py gpurun_out/vc_warm_$n.csv
done
timeout 300 ncu --profile-from-start off -k regex:coarse_vcycle --set full --import-source on --warp-sampling-interval 0 --clock-control none --cache-control none -o gpurun_out/coarse_full -f python scripts/vcycle_once_n.py 64 > /dev/null 2>&1
