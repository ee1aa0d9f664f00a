#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct
for cfg in "256 0" "512 0"; do
  set -- $cfg
  SF_GSRB_DEPTH=$2 timeout 300 ncu --metrics $M --clock-control none -k regex:gsrb_pair -s 2 -c 1 --csv \
    python scripts/prof_gsrb.py $1 3 fused 2>/dev/null | grep -E '"(gpu__|dram__|lts__)' | awk -F'","' -v c="n=$1 d=$2" '{print c, $(NF-2), $(NF-1), $NF}'
done
