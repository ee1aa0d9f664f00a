#!/bin/bash
# quick GPU iteration: build, fused-kernel parity subset, timing of fused pairs (both RPW)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { echo BUILD_FAILED; tail gpurun_out/build.log; }
for r in 1; do
  echo "RPW=$r"
  SF_GSRB_RPW=$r timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "${1:-gsrb or fused or decomposition or c3 or vcycle or solve}" 2>&1 | tail -3
  for n in 256 512; do SF_GSRB_RPW=$r timeout 120 python scripts/prof_gsrb.py $n 4 fused; done
done
