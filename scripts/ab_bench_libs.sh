#!/bin/bash
# same-session A/B of builds (ab/libsf_<tag>.so) on the bench step (--quick): ms per solve,
# in-step fused-pair ms (live timer) and SM clock
for i in 1 2 3; do for v in ${@:-base hint}; do
  r=$(SF_LIB=ab/libsf_$v.so timeout 300 python bench.py --steps 5 --warmup 3 --quick 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],2), round(d['roofline']['launch_ms'],4), d['clocks']['sm_mhz'])")
  echo "$v: ms/step, in-step pair ms, sm_mhz = $r"
done; done
