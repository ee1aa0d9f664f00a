# coarse V-cycle kernel: parity, solve timings, warm launch list
timeout 900 python -m pytest tests/test_gpu_coarse.py tests/test_gpu_parity.py -x -q 2>&1 | tail -2
python scripts/small_pair_ab.py default
timeout 300 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/vc_warm_64.csv python scripts/vcycle_once_n.py 64 > /dev/null 2>&1
python scripts/launch_list.py gpurun_out/vc_warm_64.csv | grep coarse
