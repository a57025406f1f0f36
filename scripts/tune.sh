#!/bin/bash
# Parameter sweep of the tuning knobs (FSGC_* env vars) on the default bench.
# Usage: gpurun -- 'bash scripts/tune.sh "<VAR=a VAR2=b>;<VAR=c>;..." [workload] [steps]'
CONFIGS=${1:-""}
WL=${2:-internet}
STEPS=${3:-100}
mkdir -p gpurun_out
IFS=';' read -ra CS <<< "$CONFIGS"
for c in "${CS[@]}"; do
  out=$(env $c timeout 300 python bench.py --workload $WL --steps $STEPS --warmup 5 --no-e2e --no-cpu-baseline 2>&1 | tail -1)
  echo "$c :: $(echo "$out" | python -c 'import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; o=d["roofline_other_kernels"]; print("step_ms=%.4f main=%s %.4f ms  other=%s" % (d["ms_per_step"], r["kernel"][:14], r["kernel_ms"], [(x["kernel"][:14], round(x["kernel_ms"],4)) for x in o]))' 2>&1 | tail -1)"
done
