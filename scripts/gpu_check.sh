#!/bin/bash
# One gpurun call: build, GPU tests, smoke, bench, ncu launch list + full capture.
# Usage (from the repo root on the GPU box): bash scripts/gpu_check.sh [tests|bench|ncu|all]
set -u
what=${1:-all}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || echo BUILD_FAILED
if [[ $what == tests || $what == all ]]; then
  timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
  echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke.log
fi
if [[ $what == bench || $what == all ]]; then
  timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
  echo "bench exit $?" >> gpurun_out/bench.err
fi
if [[ $what == ncu || $what == all ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
     --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 0 --quick > gpurun_out/ncu_launch_run.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:gsrb_pair -s 2 -c 1 \
     -o gpurun_out/prof_gsrb_pair -f python bench.py --steps 1 --warmup 0 --quick > gpurun_out/ncu_full_run.log 2>&1
fi
tail -3 gpurun_out/pytest_gpu.log gpurun_out/smoke.log gpurun_out/bench.err 2>/dev/null
cat gpurun_out/bench.json 2>/dev/null | head -c 3000
