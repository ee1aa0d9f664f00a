#!/bin/bash
# Round-2 evidence run on one B200 (gpurun): GPU tests, bench line, reference
# arm, launch list of the timed region, ncu capture of the dominant kernel,
# oracle table, e2e phases, headroom / coarse A/Bs.  Outputs under gpurun_out/ev/.
cd ${GRAFT_REPO_ROOT:-.}; mkdir -p gpurun_out/ev
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/ev/build.log 2>&1
what=${1:-all}
if [[ $what == all || $what == tests ]]; then
  timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/ev/tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/ev/tests.log
  tail -3 gpurun_out/ev/tests.log
fi
if [[ $what == all || $what == bench ]]; then
  timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/ev/bench.json 2> gpurun_out/ev/bench.err; echo "bench rc=$?"
  timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/ev/reference.json 2> gpurun_out/ev/reference.err; echo "ref rc=$?"
fi
if [[ $what == all || $what == ncu ]]; then
  SF_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
     --log-file gpurun_out/ev/bench_launches.csv python bench.py --steps 1 --warmup 3 --quick > gpurun_out/ev/bench_launches_run.log 2>&1
  python scripts/launch_summary.py gpurun_out/ev/bench_launches.csv > gpurun_out/ev/bench_launches_summary.txt 2>&1
  timeout 900 ncu -k regex:gsrb_pair_tma --launch-skip 6 --launch-count 1 --set full --import-source on --clock-control none \
     -f -o gpurun_out/ev/prof_gsrb_512 python scripts/prof_gsrb.py 512 > gpurun_out/ev/prof_gsrb_512.log 2>&1
  python scripts/ncu_summary.py gpurun_out/ev/prof_gsrb_512.ncu-rep > gpurun_out/ev/ncu_gsrb_pair_512.txt 2>&1
  python scripts/ncu_lines.py gpurun_out/ev/prof_gsrb_512.ncu-rep 0 25 >> gpurun_out/ev/ncu_gsrb_pair_512.txt 2>&1
  timeout 900 ncu -k regex:gsrb_pair_tma --launch-skip 6 --launch-count 1 --set full --import-source on --clock-control none \
     -f -o gpurun_out/ev/prof_gsrb_256 python scripts/prof_gsrb.py 256 > gpurun_out/ev/prof_gsrb_256.log 2>&1
  python scripts/ncu_summary.py gpurun_out/ev/prof_gsrb_256.ncu-rep > gpurun_out/ev/ncu_gsrb_pair_256.txt 2>&1
fi
if [[ $what == all || $what == oracle ]]; then
  timeout 1200 python scripts/oracle_table.py > gpurun_out/ev/oracle_table.json 2> gpurun_out/ev/oracle_table.err; echo "oracle rc=$?"
fi
if [[ $what == all || $what == probes ]]; then
  timeout 300 python scripts/e2e_phases.py > gpurun_out/ev/e2e_phases.txt 2>&1
  timeout 300 python scripts/pair_headroom.py 256 512 > gpurun_out/ev/pair_headroom.txt 2>&1
  timeout 300 python scripts/pair_sustained.py 512 > gpurun_out/ev/pair_sustained.txt 2>&1
  timeout 300 python scripts/pair_sustained.py 256 >> gpurun_out/ev/pair_sustained.txt 2>&1
  timeout 600 python scripts/coarse_ab.py > gpurun_out/ev/coarse_ab.txt 2>&1
  timeout 600 python scripts/solve_sizes.py > gpurun_out/ev/solve_sizes.txt 2>&1
fi
