#!/bin/bash
# same-session A/B of the solve step (bench.py --quick): PDL and device loop on/off
for i in 1 2; do
  for cfg in "1 1" "0 1" "1 0" "0 0"; do set -- $cfg
    v=$(SF_PDL=$1 SF_DEVICE_LOOP=$2 timeout 300 python bench.py --steps 5 --warmup 3 --quick 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],2), d['clocks']['sm_mhz'])")
    echo "PDL=$1 DEVICE_LOOP=$2: ms/step, sm_mhz = $v"
  done
done
