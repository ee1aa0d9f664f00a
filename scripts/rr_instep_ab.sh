# in-step A/B of the fused pair + residual + restriction (gsrb_rr.cu, dbg/libsf_rr.so built
# with -DSF_WITH_RR, enabled by SF_RR=1) against the shipped separate launches
SF_LIB=dbg/libsf_rr.so SF_RR=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "vcycle or solve or rr" 2>&1 | tail -1
for r in 1 2; do
for cfg in "SF_LIB=dbg/libsf_rr.so SF_RR=0" "SF_LIB=dbg/libsf_rr.so SF_RR=1"; do
env $cfg python bench.py --steps 10 --warmup 3 --quick 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); print('bench', '$cfg', round(d['ms_per_step'],2), d['clocks']['sm_mhz'], {k:round(v['ms'],3) for k,v in d['roofline']['live_per_variant'].items()})"
done; done
