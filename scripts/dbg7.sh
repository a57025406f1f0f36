#!/bin/bash
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:support_hash_kernel -c 1 -o gpurun_out/prof_hash20b -f python scripts/one_count.py rmat20x 1-tailed-triangle 1 > gpurun_out/ncu7.log 2>&1; echo "ncu rc=$?"; tail -3 gpurun_out/ncu7.log
