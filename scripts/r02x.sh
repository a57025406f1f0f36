#!/bin/bash
OUT=gpurun_out
TAG=${1:-r02x}
export FSGC_VENN_INFO=1
timeout 300 python scripts/one_count.py rmat20x triangle/tricore,tricore+1f,tricore+2f,2-tailed-triangle/tricore,3-tailed-triangle/tricore,4-tailed-triangle/tricore,diamond/tricore 3 > $OUT/probe_$TAG.log 2>&1
timeout 600 python scripts/one_count.py rmat26 triangle/tricore,tricore+1f,tricore+2f,2-tailed-triangle/tricore,3-tailed-triangle/tricore,4-tailed-triangle/tricore,diamond/tricore 1 >> $OUT/probe_$TAG.log 2>&1
cut -c1-250 $OUT/probe_$TAG.log
timeout 900 python -m pytest tests -m gpu -x -q -k "triangle or tri or rmat_hubs or z_tiers" > $OUT/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_$TAG.log
[ "${NCU:-1}" = "1" ] && SKIP=2 bash scripts/ncu_r02.sh $TAG rmat20x triangle/tricore,tricore+1f,tricore+2f,2-tailed-triangle/tricore,3-tailed-triangle/tricore,4-tailed-triangle/tricore,diamond/tricore list_ 1
