#!/bin/bash
# support-pass large-table variants (FSGC_SUP_BIG) on RMAT-22: counts must agree
OUT=gpurun_out; mkdir -p $OUT
for m in 0 1 2; do
  FSGC_SUP_BIG=$m timeout 300 python bench.py --workload rmat22 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/supbig_$m.json 2>$OUT/supbig_$m.err
  echo "mode $m rc=$?"
  python - $OUT/supbig_$m.json <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
ks = [d["roofline"]] + d.get("roofline_other_kernels", [])
print(d["ms_per_step"], [(k["kernel"][:20], round(k["kernel_ms"], 2)) for k in ks], d["config"]["counts"]["diamond"])
PY
done
