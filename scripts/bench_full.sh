#!/bin/bash
# bench line + launch list of exactly the timed region (bench's own command)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?" >> gpurun_out/bench.err
SF_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/bench_launches.csv python bench.py --steps 1 --warmup 3 --quick > gpurun_out/bench_launches_run.log 2>&1
tail -2 gpurun_out/bench.err
