#!/bin/bash
# A/B/C of several builds (ab/libsf_<tag>.so) in one session: ncu time + DRAM of one eager
# 512^3 V-cycle per build, then alternating event timings of V-cycle and solve
tags=${@:-old new}
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for v in $tags; do
  SF_LIB=ab/libsf_$v.so timeout 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/ab_$v.csv \
     python scripts/prof_variants.py 512 vcycle > /dev/null 2>&1
  echo "== $v (ncu, one V-cycle)"; python scripts/launch_summary.py gpurun_out/ab_$v.csv | sed -n 2,7p
done
for i in 1 2; do for v in $tags; do
  echo "== $v"; SF_LIB=ab/libsf_$v.so timeout 300 python scripts/variant_time.py 512 | tail -2
done; done
