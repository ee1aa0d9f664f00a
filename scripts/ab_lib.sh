#!/bin/bash
# A/B two builds of libsf in one session (ab/libsf_old.so, ab/libsf_new.so), alternating
for i in 1 2 3; do
  for v in old new; do
    echo "== $v"; SF_LIB=ab/libsf_$v.so timeout 300 python scripts/variant_time.py ${1:-512}
  done
done
