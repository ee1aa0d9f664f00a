#!/bin/bash
# chunk-depth sweep of the fused pair at 128^3/256^3 (32x8 two-CTA build) and 512^3 (32x16)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for n in 128 256; do for d in 0 256 128 86 64 43 32 22 16; do
  if [ $d -gt $n ]; then continue; fi
  echo -n "n=$n depth=$d "; SF_GSRB_DEPTH=$d timeout 120 python scripts/prof_gsrb.py $n 4 fused
done; done
for d in 0 512 256 171 128; do echo -n "n=512 depth=$d "; SF_GSRB_DEPTH=$d timeout 120 python scripts/prof_gsrb.py 512 4 fused; done
