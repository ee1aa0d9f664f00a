timeout 600 python -m pytest tests/test_gpu_cc_tma.py tests/test_gpu_parity.py -x -q -k "cc or laplacian or jacobi" 2>&1 | tail -2
for n in 256 512; do python scripts/cc_time.py $n; SF_CC_TMA=0 python scripts/cc_time.py $n; done
