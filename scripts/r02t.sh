#!/bin/bash
OUT=gpurun_out
TAG=${1:-r02t}
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
export FSGC_VENN_INFO=1
timeout 300 python scripts/one_count.py rmat20x $P26 3 > $OUT/probe_$TAG.log 2>&1
timeout 300 python scripts/one_count.py rmat20x triangle/tricore 3 >> $OUT/probe_$TAG.log 2>&1
timeout 600 python scripts/one_count.py rmat26 $P26 1 >> $OUT/probe_$TAG.log 2>&1
cut -c1-250 $OUT/probe_$TAG.log
timeout 900 python -m pytest tests -m gpu -x -q -k "${TESTK:-triangle or tri or venn or rmat_hubs or pl2k or small_patterns or z_tiers or wedge or sharded}" > $OUT/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_$TAG.log
