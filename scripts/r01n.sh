#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
TAG=r01n
timeout 600 python -m pytest tests/test_gpu.py -m gpu -x -q -k rmat26 > $OUT/pytest_rmat26_$TAG.log 2>&1; echo "pytest26 rc=$?"; tail -3 $OUT/pytest_rmat26_$TAG.log
timeout 900 python bench.py --workload rmat26 --steps 3 --warmup 3 --no-cpu-baseline > $OUT/bench_${TAG}_rmat26.json 2> $OUT/bench_${TAG}_rmat26.err; echo "bench rc=$?"; head -c 2500 $OUT/bench_${TAG}_rmat26.json; tail -3 $OUT/bench_${TAG}_rmat26.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $OUT/launches_${TAG}_rmat26.csv python bench.py --workload rmat26 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'support_hash_kernel|support_kernel|edge_fc_kernel' -c 4 \
  -o $OUT/prof_${TAG}_rmat26 -f python scripts/one_count.py rmat26 triangle,1-tailed-triangle,2-tailed-triangle,3-tailed-triangle,4-tailed-triangle 1 > $OUT/ncu_full_${TAG}_rmat26.log 2>&1; echo "ncu full rc=$?"
for r in $OUT/prof_${TAG}_*.ncu-rep; do
  ncu -i $r --page raw --csv > ${r%.ncu-rep}_raw.csv 2>/dev/null
  rm -f $r
done
ls -la $OUT | tail -5
