#!/bin/bash
# large-table cap experiment (FSGC_SUP_CAP_BIG): counts must equal the default's
OUT=gpurun_out; mkdir -p $OUT
TAG=r01p
for cap in 4096 2048; do
  FSGC_SUP_CAP_BIG=$cap timeout 400 python -m pytest tests/test_gpu.py -m gpu -x -q -k "wedge_hash or sharded_support or rmat16_closed" > $OUT/pytest_cap${cap}_$TAG.log 2>&1; echo "pytest cap $cap rc=$?"; tail -1 $OUT/pytest_cap${cap}_$TAG.log
done
for cap in 1024 2048 4096; do
  FSGC_SUP_CAP_BIG=$cap timeout 300 python bench.py --workload rmat22 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/cap${cap}_rmat22.json 2>$OUT/cap${cap}_rmat22.err
  echo "rmat22 cap $cap rc=$?"
  python - $OUT/cap${cap}_rmat22.json <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
ks = [d["roofline"]] + d.get("roofline_other_kernels", [])
print(d["ms_per_step"], [(k["kernel"][:20], round(k["kernel_ms"], 2)) for k in ks], d["config"]["counts"]["4-tailed-triangle"])
PY
done
for cap in 4096 1024; do
  FSGC_SUP_CAP_BIG=$cap timeout 300 python scripts/rmat26_probe.py 26 "triangle,1-tailed-triangle" > $OUT/cap${cap}_rmat26.log 2>&1; echo "rmat26 cap $cap rc=$?"; tail -2 $OUT/cap${cap}_rmat26.log
done
