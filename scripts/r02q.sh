#!/bin/bash
OUT=gpurun_out
TAG=${1:-r02q}
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
timeout 300 python scripts/one_count.py rmat20x $P26 3 > $OUT/probe_$TAG.log 2>&1
timeout 300 python scripts/one_count.py rmat20x triangle/tricore 3 >> $OUT/probe_$TAG.log 2>&1
timeout 300 python scripts/one_count.py rmat22 triangle,1-tailed-triangle 3 >> $OUT/probe_$TAG.log 2>&1
timeout 300 python scripts/one_count.py pl10m fig4 3 >> $OUT/probe_$TAG.log 2>&1
cut -c1-250 $OUT/probe_$TAG.log
timeout 1500 python -m pytest tests -m gpu -x -q ${TESTK:+-k "$TESTK"} > $OUT/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_$TAG.log
