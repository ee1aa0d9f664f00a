#!/bin/bash
# full ncu capture of the fused pair (512^3, 256^3) + launch list of bench.py's timed region
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gsrb_pair -s 2 -c 1 \
   -o gpurun_out/prof_gsrb_pf3_512 -f python scripts/prof_gsrb.py 512 3 fused > gpurun_out/ncu_pf3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gsrb_pair -s 2 -c 1 \
   -o gpurun_out/prof_gsrb_pf3_256 -f python scripts/prof_gsrb.py 256 3 fused >> gpurun_out/ncu_pf3.log 2>&1
SF_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/bench_launches.csv python bench.py --steps 2 --warmup 1 --quick > gpurun_out/bench_launches_run.log 2>&1
tail -c 400 gpurun_out/bench_launches_run.log
