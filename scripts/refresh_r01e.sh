#!/bin/bash
# Evidence refresh (device loop + PDL + 3-CTA default + live roofline): bench line, timed-region
# solve launch list with DRAM bytes, e2e probe, ncu full of the 512^3 pair (unchanged kernel,
# now PDL-launched) for the committed source-level profile.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench exit $?"
SF_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/bench_launches.csv python bench.py --steps 1 --warmup 3 --quick > gpurun_out/bench_launches_run.log 2>&1
echo "timed-region launch list exit $?"
timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
   --log-file gpurun_out/solve_launches.csv python scripts/solve_profile.py 512 0 > gpurun_out/solve_launches.log 2>&1
echo "solve launch list exit $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gsrb_pair -s 2 -c 1 \
   -o gpurun_out/prof_gsrb_v14_512 -f python scripts/prof_gsrb.py 512 3 fused > gpurun_out/ncu_v14_512.log 2>&1
echo "ncu pair 512 exit $?"
python scripts/e2e_probe.py 512 > gpurun_out/e2e_probe.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gsrb_pair -s 2 -c 1 \
   -o gpurun_out/prof_gsrb_v14_256 -f python scripts/prof_gsrb.py 256 3 fused > gpurun_out/ncu_v14_256.log 2>&1
echo "ncu pair 256 exit $?"
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -1 gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
