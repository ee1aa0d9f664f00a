#!/bin/bash
# per-kernel device times of one eager 512^3 V-cycle and F-cycle (INTERP pairs, PL interpolation)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/vc_launches.csv \
   python scripts/prof_variants.py 512 fcycle > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/vc_launches.csv | head -12
for i in 1 2; do timeout 300 python scripts/variant_time.py 512; done
