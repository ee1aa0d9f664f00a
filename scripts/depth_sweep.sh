#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for n in 256; do for d in 0 16 21 26 32 43 52 64 86 128 256; do
  if [ $d -gt $n ]; then continue; fi
  echo -n "depth=$d "; SF_GSRB_DEPTH=$d timeout 120 python scripts/prof_gsrb.py $n 4 fused
done; done
