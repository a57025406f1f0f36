#!/bin/bash
# ncu full capture of the triangle-core listing kernels on RMAT-20 with the
# configs[4] pattern set (+ timings without ncu first)
OUT=gpurun_out
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
timeout 300 python scripts/one_count.py rmat20x $P26 3 > $OUT/probe_r02c.log 2>&1; echo "rc=$?" >> $OUT/probe_r02c.log
FSGC_VENN_INFO=1 timeout 300 python scripts/one_count.py rmat22 $P26 2 >> $OUT/probe_r02c.log 2>&1; echo "rc=$?" >> $OUT/probe_r02c.log
cat $OUT/probe_r02c.log
bash scripts/ncu_r02.sh r02c rmat20x $P26 'list_' 4
