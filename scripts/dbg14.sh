#!/bin/bash
mkdir -p gpurun_out
FSGC_VENN_INFO=1 timeout 300 python scripts/one_count.py pl10m fig4 1 2>&1 | tail -2
FSGC_VENN_INFO=1 timeout 300 python scripts/one_count.py rmat16 k4core+1f,k4core+2f,k4core+3f,k4core+4f,k4core+5f,k4core+6f 1 2>&1 | tail -2
FSGC_VENN_WARP_TERMS=100000 timeout 300 python scripts/one_count.py rmat16 k4core+1f,k4core+2f,k4core+3f,k4core+4f,k4core+5f,k4core+6f 1 2>&1 | tail -1
FSGC_VENN_WARP_TERMS=1 timeout 300 python scripts/one_count.py rmat16 k4core+1f,k4core+2f,k4core+3f,k4core+4f,k4core+5f,k4core+6f 1 2>&1 | tail -1
FSGC_NO_VENN_TERMS=1 timeout 300 python scripts/one_count.py rmat16 k4core+1f,k4core+2f,k4core+3f,k4core+4f,k4core+5f,k4core+6f 1 2>&1 | tail -1
timeout 300 python scripts/one_count.py rmat16 diamondcore+1f 1 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_q14.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_q14.log
