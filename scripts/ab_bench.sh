#!/bin/bash
# In-step A/B of library builds (SF_VARIANT, build.py) and/or environment
# settings: bench.py --quick lines interleaved; step time, cycles, clock and the
# live per-variant pair times.
# usage: scripts/ab_bench.sh reps "label:VAR=val:variant" ...  (variant "base" = libsf.so)
cd ${GRAFT_REPO_ROOT:-.}; mkdir -p gpurun_out
P=paper_conf_ipps_zhangdmwbf17_b200
reps=$1; shift
for rep in $(seq $reps); do
  for spec in "$@"; do
    IFS=: read label envs v <<< "$spec"
    lib=$P/libsf.so; [[ $v != base ]] && lib=$P/libsf_$v.so
    env $envs SF_LIB=$lib timeout 600 python bench.py --steps 10 --warmup 3 --quick > gpurun_out/bench_$label.json 2>gpurun_out/bench_$label.err
    python - $label <<'PY'
import json,sys
try:
    d=json.loads(open(f"gpurun_out/bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
except Exception as e:
    print(sys.argv[1], "FAILED", e); sys.exit(0)
r=d["roofline"]
print(sys.argv[1], "ms/step %.2f" % d["ms_per_step"], "cyc", d["config"].get("cycles_per_solve"), "clk", d["clocks"]["sm_mhz"], "frac %.3f" % r["frac"],
      {k: round(v["ms"], 4) for k, v in r["live_per_variant"].items()}, flush=True)
PY
  done
done
