timeout 900 python -m pytest tests/test_gpu_headline_builds.py tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q 2>&1 | tail -2
for r in 1 2; do
for lib in dbg/libsf_base.so paper_conf_ipps_zhangdmwbf17_b200/libsf.so; do
  SF_LIB=$lib python scripts/interp_nocorr.py 512
  SF_LIB=$lib python scripts/interp_nocorr.py 256
done; done
for lib in dbg/libsf_base.so paper_conf_ipps_zhangdmwbf17_b200/libsf.so dbg/libsf_base.so paper_conf_ipps_zhangdmwbf17_b200/libsf.so; do
SF_LIB=$lib python bench.py --steps 10 --warmup 3 --quick 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); print('bench', '$lib', round(d['ms_per_step'],2), d['clocks']['sm_mhz'], {k:round(v['ms'],3) for k,v in d['roofline']['live_per_variant'].items()})"
done
