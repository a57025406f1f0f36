#!/bin/bash
OUT=gpurun_out
TAG=${1:-r02f}
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
timeout 300 python scripts/one_count.py rmat20x $P26 3 > $OUT/probe_$TAG.log 2>&1
timeout 300 python scripts/one_count.py rmat20x triangle/tricore 3 >> $OUT/probe_$TAG.log 2>&1
cat $OUT/probe_$TAG.log
if [ "${NCU:-1}" = "1" ]; then SKIP=2 bash scripts/ncu_r02.sh $TAG rmat20x $P26 'list_' 2; fi
