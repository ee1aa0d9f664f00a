# the coarse cluster V-cycle launched early (PDL trigger in the residual + restriction before it,
# constant operands staged before griddepcontrol.wait) vs the previous build (dbg/libsf_base.so)
timeout 900 python -m pytest tests/test_gpu_coarse.py tests/test_gpu_parity.py -x -q 2>&1 | tail -1
for r in 1 2; do
SF_LIB=dbg/libsf_base.so python scripts/small_pair_ab.py base
python scripts/small_pair_ab.py early-coarse
done
