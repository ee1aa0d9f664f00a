#!/bin/bash
# Sustained-load (power-capped) A/B of the fused pair: library builds
# (SF_VARIANT, build.py) and/or environment settings, interleaved 3x.
# usage: scripts/ab_sustained.sh "label:VAR=val:variant" ...  (variant "base" = libsf.so)
cd ${GRAFT_REPO_ROOT:-.}
P=paper_conf_ipps_zhangdmwbf17_b200
for rep in 1 2 3; do
  for spec in "$@"; do
    IFS=: read label envs v <<< "$spec"
    lib=$P/libsf.so; [[ $v != base ]] && lib=$P/libsf_$v.so
    echo -n "$label: "
    env $envs SF_LIB=$lib timeout 120 python scripts/pair_sustained.py 512
  done
done
