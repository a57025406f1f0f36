#!/bin/bash
# One gpurun call: GPU tests, the default bench, the ncu launch list and one
# full ncu capture of the dominant kernel.  Usage (from the repo root):
#   gpurun --timeout 1500 -- 'bash scripts/gpu_check.sh [tag] [workload]'
TAG=${1:-r01}
WL=${2:-internet}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $OUT/gpu_$TAG.txt
if [ "${SKIP_TESTS:-0}" != "1" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log
  tail -3 $OUT/pytest_gpu_$TAG.log
fi
timeout 600 python bench.py --workload $WL > $OUT/bench_${TAG}_$WL.json 2> $OUT/bench_${TAG}_$WL.err; echo "bench rc=$?"
cat $OUT/bench_${TAG}_$WL.json | head -c 3000; echo
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $OUT/launches_${TAG}_$WL.csv python bench.py --workload $WL --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'support_kernel|edge_fc_kernel|core_kernel' -s 8 -c 2 \
  -o $OUT/prof_${TAG}_$WL -f python bench.py --workload $WL --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_full_${TAG}.log 2>&1; echo "ncu full rc=$?"
ls -la $OUT
