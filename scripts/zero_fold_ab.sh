# the BRES scalar reset folded into the P0-fused pair (no zero_bits launch): GPU suite, timings
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | grep -E "FAILED|passed|failed" | head -5
for r in 1 2; do
SF_LIB=dbg/libsf_base.so python scripts/small_pair_ab.py base
python scripts/small_pair_ab.py zero-folded
done
