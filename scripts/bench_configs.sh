#!/bin/bash
# Bench lines for the non-default workloads (BASELINE configs) + their ncu
# launch lists.  Usage: gpurun -- 'bash scripts/bench_configs.sh TAG "wl1 wl2 ..."'
TAG=${1:-r01}
WLS=${2:-"pl2k pl10m rmat22 rmat16"}
mkdir -p gpurun_out
for wl in $WLS; do
  case $wl in
    pl2k) ARGS="--steps 50 --warmup 5";;
    *) ARGS="--steps 3 --warmup 3 --no-cpu-baseline";;
  esac
  timeout 900 python bench.py --workload $wl $ARGS > gpurun_out/bench_${TAG}_$wl.json 2> gpurun_out/bench_${TAG}_$wl.err
  echo "$wl rc=$?"; head -c 400 gpurun_out/bench_${TAG}_$wl.json; echo
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${TAG}_$wl.csv python bench.py --workload $wl --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  echo "$wl ncu rc=$?"
done
