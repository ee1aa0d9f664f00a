#!/bin/bash
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for st in 0 1; do
  SF_GSRB_STREAM=$st python -m paper_conf_ipps_zhangdmwbf17_b200.build --force > /dev/null 2>&1
  echo "== STREAM=$st"
  timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "gsrb or fused or decomposition or c3 or solve" 2>&1 | tail -1
  for n in 256 512; do python scripts/prof_gsrb.py $n 4 fused; done
  for n in 256 512; do
    timeout 300 ncu --metrics $M --clock-control none -k regex:gsrb_pair -s 2 -c 1 --csv python scripts/prof_gsrb.py $n 3 fused 2>/dev/null | grep -E '"(dram__)' | awk -F'","' -v c="n=$n" '{print c, $(NF-2), $NF}'
  done
done
