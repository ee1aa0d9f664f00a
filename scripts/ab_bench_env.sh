#!/bin/bash
# same-session A/B of an environment switch on the bench step (--quick):
#   bash scripts/ab_bench_env.sh VAR "valA valB"
var=$1; vals=${2:-"0 1"}
for i in 1 2 3; do for v in $vals; do
  r=$(env $var=$v timeout 300 python bench.py --steps 5 --warmup 3 --quick 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],2), round(d['roofline']['launch_ms'],4), d['clocks']['sm_mhz'])")
  echo "$var=$v: ms/step, in-step pair ms, sm_mhz = $r"
done; done
