#!/bin/bash
# A/B two builds of libsf in one session (ab/libsf_old.so, ab/libsf_new.so), alternating
n=${1:-512}
for i in 1 2 3; do
  for v in old new; do
    echo "== $v"; SF_LIB=ab/libsf_$v.so timeout 300 python scripts/variant_time.py $n
    SF_LIB=ab/libsf_$v.so timeout 120 python scripts/prof_gsrb.py 256 4 fused
  done
done
