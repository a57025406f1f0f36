#!/bin/bash
mkdir -p gpurun_out
python scripts/e2e_breakdown.py internet > gpurun_out/e2e_bd.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "sharded or distributed or internet or pl2k or fig2" > gpurun_out/pytest_q1.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_q1.log
timeout 400 python scripts/debug_rmat.py 14,16,18,20,22 triangle,diamond,1-tailed-triangle,2-tailed-triangle,3-tailed-triangle,4-tailed-triangle > gpurun_out/dbg_edge.txt 2>&1; echo "edge rc=$?"
EF=8 timeout 400 python scripts/debug_rmat.py 12,14,16 clique4,diamondcore+1f,k4core+1f,k4core+2f,k4core+4f,k4core+6f,diamondcore+2f > gpurun_out/dbg_gen.txt 2>&1; echo "gen rc=$?"
cat gpurun_out/e2e_bd.txt
