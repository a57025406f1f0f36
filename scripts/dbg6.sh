#!/bin/bash
mkdir -p gpurun_out
for sc in 20 22; do
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/l6_$sc.csv python scripts/one_count.py rmat${sc}x 1-tailed-triangle 2 > /dev/null 2>&1
python - <<PY
import csv
rows=[r for r in csv.DictReader(open('gpurun_out/l6_$sc.csv')) if r.get('Metric Name')=='gpu__time_duration.sum']
agg={}
for r in rows:
    k=r['Kernel Name'][:70]; agg.setdefault(k,[]).append(float(r['Metric Value']))
for k,v in sorted(agg.items(), key=lambda kv:-sum(kv[1]))[:8]: print($sc, k, len(v), '%.1f us'%(sum(v)/len(v)/1e3))
PY
done
