#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
bash scripts/sweep_supbig.sh
timeout 240 python scripts/rmat26_probe.py 20 "tricore+1f;tricore+6f;c4core+1f" > $OUT/probe20.log 2>&1; echo "probe20 rc=$?"; tail -8 $OUT/probe20.log
timeout 400 python scripts/rmat26_probe.py 26 "triangle;1-tailed-triangle,2-tailed-triangle,3-tailed-triangle,4-tailed-triangle" > $OUT/probe26e.log 2>&1; echo "probe26e rc=$?"; tail -8 $OUT/probe26e.log
