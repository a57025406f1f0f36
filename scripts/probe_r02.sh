#!/bin/bash
# r02 probe: parity subset + timings of the listing kernels
OUT=gpurun_out
TAG=${1:-r02}
if [ "${SKIP_TESTS:-0}" != "1" ]; then
timeout 900 python -m pytest tests -m gpu -x -q -k "${TESTK:-rmat_hubs or venn or pl2k or sharded or wedge_hash or small_patterns or hub_bitmaps or fig2 or degenerate}" > $OUT/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
tail -3 $OUT/pytest_$TAG.log
fi
IFS=';' read -ra SPECS <<< "${PROBES:-rmat20x triangle,tricore+1f,tricore+2f;rmat20x tricore+3f;pl10m fig4;rmat22 triangle,tricore+1f;rmat26 triangle,tricore+1f,tricore+2f}"
for spec in "${SPECS[@]}"; do
  set -- $spec
  timeout ${PTIMEOUT:-300} python scripts/one_count.py $1 $2 3 >> $OUT/probe_$TAG.log 2>&1; echo "$spec rc=$?" >> $OUT/probe_$TAG.log
done
cat $OUT/probe_$TAG.log
