#!/bin/bash
# r02 GPU check: full GPU suite, the default bench line, listing-kernel probes
TAG=${1:-r02a}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $OUT/gpu_$TAG.txt
if [ "${SKIP_TESTS:-0}" != "1" ]; then
  timeout ${TTIMEOUT:-1200} python -m pytest tests -m gpu -x -q ${TESTK:+-k "$TESTK"} > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log
  tail -3 $OUT/pytest_gpu_$TAG.log
fi
if [ "${SKIP_BENCH:-0}" != "1" ]; then
  timeout ${BTIMEOUT:-1200} python bench.py ${BENCHARGS} > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
  head -c 4000 $OUT/bench_$TAG.json; echo; tail -5 $OUT/bench_$TAG.err
fi
if [ -n "$PROBES" ]; then SKIP_TESTS=1 bash scripts/probe_r02.sh $TAG; fi
