#!/bin/bash
# ncu capture of the fused GSRB pair at 256^3 and 512^3 (+ a timing line)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
tag=${1:-v1}
for n in 256 512; do
  python scripts/prof_gsrb.py $n 4 fused >> gpurun_out/prof_timing_$tag.txt 2>&1
  python scripts/prof_gsrb.py $n 4 colour >> gpurun_out/prof_timing_$tag.txt 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gsrb_pair -s 2 -c 1 \
   -o gpurun_out/prof_gsrb_${tag}_512 -f python scripts/prof_gsrb.py 512 3 fused > gpurun_out/ncu_$tag.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gsrb_pair -s 2 -c 1 \
   -o gpurun_out/prof_gsrb_${tag}_256 -f python scripts/prof_gsrb.py 256 3 fused >> gpurun_out/ncu_$tag.log 2>&1
cat gpurun_out/prof_timing_$tag.txt
