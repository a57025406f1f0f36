#!/bin/bash
OUT=gpurun_out
TAG=${1:-r02r}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu_$TAG.txt
timeout 2400 python bench.py ${BARGS} > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
tail -30 $OUT/bench_$TAG.err
