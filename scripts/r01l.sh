#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
SKIP_NCU_FULL=1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu_r01l.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_r01l.log; tail -3 $OUT/pytest_gpu_r01l.log
timeout 400 python bench.py > $OUT/bench_r01l_internet.json 2> $OUT/bench_r01l_internet.err; echo "bench rc=$?"; head -c 600 $OUT/bench_r01l_internet.json; echo
timeout 300 python scripts/rmat26_probe.py 24 > $OUT/probe24.log 2>&1; echo "probe24 rc=$?"; cat $OUT/probe24.log | tail -8
timeout 700 python scripts/rmat26_probe.py 26 > $OUT/probe26.log 2>&1; echo "probe26 rc=$?"; cat $OUT/probe26.log | tail -8
