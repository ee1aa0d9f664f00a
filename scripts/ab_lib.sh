#!/bin/bash
# A/B of library builds (SF_VARIANT builds, build.py) on one GPU: the fused
# pair alone and with its operands L2-resident (scripts/pair_headroom.py),
# interleaved twice.  usage: scripts/ab_lib.sh name [name ...]  (base = libsf.so)
cd ${GRAFT_REPO_ROOT:-.}
P=paper_conf_ipps_zhangdmwbf17_b200
for rep in 1 2; do
  for v in base "$@"; do
    if [[ $v == base ]]; then lib=$P/libsf.so; else lib=$P/libsf_$v.so; fi
    echo "== $v (rep $rep)"
    SF_LIB=$lib timeout 300 python scripts/pair_headroom.py 256 512
  done
done
