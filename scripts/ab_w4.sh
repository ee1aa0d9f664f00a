#!/bin/bash
# 512^3: 32x16/1 CTA (default) vs the 32x8 build forced (SF_GSRB_W4=1); V-cycle + solve per build
for i in 1 2; do for v in ${@:-base m3pf2}; do
  echo "== $v"; SF_LIB=ab/libsf_$v.so timeout 120 python scripts/prof_gsrb.py 512 3 fused
  echo "   (W4=1)"; SF_GSRB_W4=1 SF_LIB=ab/libsf_$v.so timeout 120 python scripts/prof_gsrb.py 512 3 fused
  SF_LIB=ab/libsf_$v.so timeout 300 python scripts/variant_time.py 512 | tail -2
  SF_LIB=ab/libsf_$v.so timeout 300 python scripts/variant_time.py 256 | tail -2
done; done
