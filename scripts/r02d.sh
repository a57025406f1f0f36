#!/bin/bash
# which fc path the triangle-core pass takes, and the cost per pattern
OUT=gpurun_out
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
run() { echo "== $*" >> $OUT/probe_r02d.log; env "$@" >> $OUT/probe_r02d.log 2>&1; }
export FSGC_VENN_INFO=1
run timeout 300 python scripts/one_count.py rmat20x $P26 3
run FSGC_NO_Z_TERMS=1 timeout 300 python scripts/one_count.py rmat20x $P26 3
run FSGC_NO_VENN_TERMS=1 timeout 300 python scripts/one_count.py rmat20x $P26 3
for p in triangle/tricore tricore+1f 4-tailed-triangle/tricore tricore+2f diamond/tricore; do
  run timeout 300 python scripts/one_count.py rmat20x $p 3
done
cat $OUT/probe_r02d.log
