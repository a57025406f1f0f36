#!/bin/bash
OUT=gpurun_out
TAG=${1:-r02n}
timeout 1500 python bench.py --no-per-config --steps 3 --warmup 2 --e2e-steps 1 ${BARGS} > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
tail -12 $OUT/bench_$TAG.err
python - <<'PY'
import json,sys
d=json.loads(open(f"gpurun_out/bench_{sys.argv[1] if len(sys.argv)>1 else 'r02n'}.json").readline())
print({k: d[k] for k in ("value","ms_per_step","edges_per_s")}, d["roofline"]["kernel"], d["roofline"]["frac"], d.get("cpu_baseline"))
PY
