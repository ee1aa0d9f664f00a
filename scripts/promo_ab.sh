#!/bin/bash
# A/B of fused-pair variants: TMA L2 promotion, and the 32x8 2-CTA/SM build (SF_GSRB_W4=1)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for cfg in "SF_TMA_PROMO=256" "SF_TMA_PROMO=128" "SF_TMA_PROMO=0" "SF_GSRB_W4=1" "SF_GSRB_W4=1 SF_TMA_PROMO=128"; do
  echo "== $cfg"
  for n in 128 256 512; do env $cfg python scripts/prof_gsrb.py $n 4 fused; done
  for n in 256 512; do
    env $cfg timeout 300 ncu --metrics $M --clock-control none -k regex:gsrb_pair -s 2 -c 1 --csv python scripts/prof_gsrb.py $n 3 fused 2>/dev/null | grep -E '"(dram__)' | awk -F'","' -v c="n=$n" '{print c, $(NF-2), $NF}'
  done
done
SF_GSRB_W4=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "gsrb or fused or chunk or decomposition or vcycle or c2_solve or max_cycles" 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "chunk" 2>&1 | tail -2
