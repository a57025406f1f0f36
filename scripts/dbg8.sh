#!/bin/bash
mkdir -p gpurun_out
timeout 300 python scripts/debug_support.py 20 16 > gpurun_out/dbg8_sup20.txt 2>&1; echo "sup20 rc=$?"; tail -3 gpurun_out/dbg8_sup20.txt
for sc in 20 22; do
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/l8_$sc.csv python scripts/one_count.py rmat${sc}x 1-tailed-triangle 2 > /dev/null 2>&1
python scripts/launch_agg.py gpurun_out/l8_$sc.csv 4
done
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_q8.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_q8.log
