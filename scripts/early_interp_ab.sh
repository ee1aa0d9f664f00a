# the P0-fused pair started early under the coarse cluster V-cycle (TMA prologue before
# griddepcontrol.wait) vs the previous build (dbg/libsf_base.so)
timeout 1500 python -m pytest tests/test_gpu_coarse.py tests/test_gpu_parity.py tests/test_gpu_headline_builds.py tests/test_gpu_measurement.py -x -q 2>&1 | grep -E "FAILED|passed|failed" | head -5
for r in 1 2; do
SF_LIB=dbg/libsf_base.so python scripts/small_pair_ab.py base
python scripts/small_pair_ab.py early-interp
done
