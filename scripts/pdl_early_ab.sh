# A/B: griddepcontrol.launch_dependents right after griddepcontrol.wait in every kernel
# (dbg/libsf_early.so, -DSF_PDL_EARLY) vs the shipped library
SF_LIB=dbg/libsf_early.so timeout 900 python -m pytest tests/test_gpu_coarse.py tests/test_gpu_parity.py -x -q 2>&1 | tail -1
for r in 1 2; do
python scripts/small_pair_ab.py shipped
SF_LIB=dbg/libsf_early.so python scripts/small_pair_ab.py early
done
for lib in paper_conf_ipps_zhangdmwbf17_b200/libsf.so dbg/libsf_early.so paper_conf_ipps_zhangdmwbf17_b200/libsf.so dbg/libsf_early.so; do
SF_LIB=$lib python bench.py --steps 10 --warmup 3 --quick 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); print('bench', '$lib', round(d['ms_per_step'],2), d['clocks']['sm_mhz'], round(d['vcycle']['ms'],3), round(d['fcycle']['ms'],3))"
done
