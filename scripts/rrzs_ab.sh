#!/bin/bash
# A/B: z-streamed residual_restrict (SF_RR_ZS=1, default) vs the per-plane kernel; INTERP 2-step prefetch
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "vcycle or fcycle or solve or decomposition or overlap or chunk" 2>&1 | grep -E "^E|passed|failed" | head -5
for zs in 1 0; do
  echo "== SF_RR_ZS=$zs"
  SF_RR_ZS=$zs timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
     --log-file gpurun_out/vc_$zs.csv python scripts/prof_variants.py 512 vcycle > /dev/null 2>&1
  python scripts/launch_summary.py gpurun_out/vc_$zs.csv | head -8
  SF_RR_ZS=$zs timeout 300 python scripts/variant_time.py 512
done
