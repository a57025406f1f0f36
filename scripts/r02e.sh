#!/bin/bash
OUT=gpurun_out
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
export FSGC_VENN_INFO=1
timeout 300 python scripts/one_count.py rmat20x $P26 3 > $OUT/probe_r02e.log 2>&1
timeout 300 python scripts/one_count.py rmat20x triangle/tricore 3 >> $OUT/probe_r02e.log 2>&1
timeout 300 python scripts/one_count.py pl10m fig4 3 >> $OUT/probe_r02e.log 2>&1
cat $OUT/probe_r02e.log
timeout 1200 python -m pytest tests -m gpu -x -q -k "${TESTK:-triangle or tri or venn or rmat_hubs or pl2k or small_patterns or fig2 or rmat16}" > $OUT/pytest_r02e.log 2>&1; echo "pytest rc=$?"; tail -5 $OUT/pytest_r02e.log
