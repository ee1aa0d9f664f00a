#!/bin/bash
# A/B of programmatic dependent launch (SF_PDL=1 default vs 0), same build, alternating
for i in 1 2; do for v in 0 1; do
  echo "== SF_PDL=$v"
  SF_PDL=$v timeout 300 python scripts/coarse_cost.py | grep -E "n=  64|n= 256"
  SF_PDL=$v timeout 300 python scripts/variant_time.py 512 | tail -2
done; done
