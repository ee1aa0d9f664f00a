timeout 900 python -m pytest tests/test_gpu_headline_builds.py tests/test_gpu_parity.py -x -q 2>&1 | tail -2
for n in 256 512; do python scripts/interp_time.py $n; python scripts/interp_time.py $n; done
python bench.py --steps 10 --warmup 3 --quick 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); print('bench', d['ms_per_step'], d['clocks']['sm_mhz'], {k:round(v['ms'],3) for k,v in d['roofline']['live_per_variant'].items()})"
SF_INTERP_T32=0 python bench.py --steps 10 --warmup 3 --quick 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); print('bench w4-interp', d['ms_per_step'], d['clocks']['sm_mhz'], {k:round(v['ms'],3) for k,v in d['roofline']['live_per_variant'].items()})"
