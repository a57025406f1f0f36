#!/bin/bash
# triangle-core pass timings (configs[4] set on RMAT-20 / RMAT-26, Fig. 4 on
# pl10m) + the triangle-core GPU tests: one gpurun call per kernel change
OUT=gpurun_out
TAG=${1:-probe}
timeout 300 python scripts/one_count.py rmat20x triangle/tricore,tricore+1f,tricore+2f,2-tailed-triangle/tricore,3-tailed-triangle/tricore,4-tailed-triangle/tricore,diamond/tricore 3 > $OUT/probe_$TAG.log 2>&1
timeout 600 python scripts/one_count.py rmat26 triangle/tricore,tricore+1f,tricore+2f,2-tailed-triangle/tricore,3-tailed-triangle/tricore,4-tailed-triangle/tricore,diamond/tricore 1 >> $OUT/probe_$TAG.log 2>&1
timeout 300 python scripts/one_count.py pl10m fig4 3 >> $OUT/probe_$TAG.log 2>&1
cut -c1-200 $OUT/probe_$TAG.log
timeout 900 python -m pytest tests -m gpu -x -q -k "${TESTK:-triangle or tri or rmat_hubs or z_tiers or venn}" > $OUT/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_$TAG.log
