#!/bin/bash
# ncu --set full of the RESID and INTERP fused-pair variants at 512^3
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
tag=${1:-v11}
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
   -k 'regex:gsrb_pair_tma_kernel<.bool.1' -c 1 \
   -o gpurun_out/prof_resid_${tag}_512 -f python scripts/prof_variants.py 512 solve > gpurun_out/ncu_resid_$tag.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
   -k 'regex:gsrb_pair_tma_kernel<.bool.0, .bool.1' -c 6 \
   -o gpurun_out/prof_interp_${tag}_512 -f python scripts/prof_variants.py 512 vcycle > gpurun_out/ncu_interp_$tag.log 2>&1
for f in gpurun_out/ncu_resid_$tag.log gpurun_out/ncu_interp_$tag.log; do tail -n 3 $f; done
