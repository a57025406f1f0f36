#!/bin/bash
mkdir -p gpurun_out
timeout 300 python scripts/debug_support.py 20 16 > gpurun_out/dbg9_sup20.txt 2>&1; echo "sup20 rc=$?"; tail -2 gpurun_out/dbg9_sup20.txt
for sc in 20 22; do
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/l9_$sc.csv python scripts/one_count.py rmat${sc}x 1-tailed-triangle 2 > /dev/null 2>&1
python scripts/launch_agg.py gpurun_out/l9_$sc.csv 3
done
