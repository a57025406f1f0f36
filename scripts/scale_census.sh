#!/bin/bash
# configs[2] / configs[4] core-size census: counts and times of the 4-vertex
# cores (general core kernel) across RMAT scales, clique4 / diamond on RMAT-22
OUT=gpurun_out
TAG=${1:-r02s}
python scripts/census.py 14 16 18 20 22 26 > $OUT/census_$TAG.log 2>&1
cat $OUT/census_$TAG.log
for sc in 14 16 18; do
  for p in cycle4 c4core+2f c4core+4f clique4 k4core+1f k4core+3f k4core+6f diamondcore+1f diamondcore+3f; do
    echo "== rmat${sc}x $p" >> $OUT/scale_$TAG.log
    timeout ${PT:-150} python scripts/one_count.py rmat${sc}x $p 1 >> $OUT/scale_$TAG.log 2>&1 || echo "timeout/fail" >> $OUT/scale_$TAG.log
  done
done
for p in clique4 diamond; do
  echo "== rmat22 $p" >> $OUT/scale_$TAG.log
  timeout 600 python scripts/one_count.py rmat22 $p 1 >> $OUT/scale_$TAG.log 2>&1 || echo "timeout/fail" >> $OUT/scale_$TAG.log
done
cat $OUT/scale_$TAG.log
