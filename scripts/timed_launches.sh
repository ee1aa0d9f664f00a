python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
SF_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
   --log-file gpurun_out/bench_launches.csv python bench.py --steps 1 --warmup 3 --quick > gpurun_out/bench_launches_run.log 2>&1
