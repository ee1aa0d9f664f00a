python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "vcycle or fcycle or solve or decomposition or overlap or chunk or interpolate" 2>&1 | grep -E "^E|passed|failed" | head -5
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/vc_new.csv python scripts/prof_variants.py 512 vcycle > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/vc_new.csv | head -8
for i in 1 2; do timeout 300 python scripts/variant_time.py 512; done
