timeout 600 python -m pytest tests/test_gpu_coarse.py -x -q 2>&1 | tail -1
python scripts/small_pair_ab.py default
SF_GSRB_W4=0 python scripts/small_pair_ab.py t32
SF_GSRB_W4=0 SF_GSRB_DEPTH=4 python scripts/small_pair_ab.py t32-d4
SF_GSRB_W4=0 SF_GSRB_DEPTH=2 python scripts/small_pair_ab.py t32-d2
SF_GSRB_DEPTH=2 python scripts/small_pair_ab.py w4-d2
SF_GSRB_DEPTH=1 python scripts/small_pair_ab.py w4-d1
timeout 300 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/vc_warm_64.csv python scripts/vcycle_once_n.py 64 > /dev/null 2>&1
python scripts/launch_list.py gpurun_out/vc_warm_64.csv
