#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
TAG=r01r
timeout 600 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu.py::test_rmat26_full_size_wedge_hash_equals_merge > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log; tail -3 $OUT/pytest_gpu_$TAG.log
timeout 150 python scripts/rmat26_probe.py 20 "tricore+1f;tricore+3f" > $OUT/probe20_$TAG.log 2>&1; echo "probe20 rc=$?"; tail -5 $OUT/probe20_$TAG.log
timeout 200 python bench.py --workload pl10m --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_${TAG}_pl10m.json 2>$OUT/bench_${TAG}_pl10m.err; echo "pl10m rc=$?"; head -c 300 $OUT/bench_${TAG}_pl10m.json
