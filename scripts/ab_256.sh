#!/bin/bash
# A/B of fused-pair builds at 256^3 and 128^3 (ab/libsf_<tag>.so), alternating
for i in 1 2 3; do for v in ${@:-base pf4}; do
  echo "== $v"; for n in 256 128; do SF_LIB=ab/libsf_$v.so timeout 120 python scripts/prof_gsrb.py $n 4 fused; done
done; done
