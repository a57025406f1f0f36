#!/bin/bash
# support-pass timings (RMAT-20 / 22 / 26) + the support-algorithm GPU tests
OUT=gpurun_out
TAG=${1:-probe}
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
timeout 300 python scripts/one_count.py rmat20x triangle 3 > $OUT/probe_$TAG.log 2>&1
timeout 300 python scripts/one_count.py rmat22 triangle 3 >> $OUT/probe_$TAG.log 2>&1
timeout 600 python scripts/one_count.py rmat26 $P26 1 >> $OUT/probe_$TAG.log 2>&1
cut -c1-200 $OUT/probe_$TAG.log
timeout 1500 python -m pytest tests -m gpu -x -q -k "${TESTK:-support or wedge or small_patterns or pl2k or internet or rmat_hubs or sharded or k_tailed or venn or z_tiers or fc_paths}" > $OUT/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_$TAG.log
