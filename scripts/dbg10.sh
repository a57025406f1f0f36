#!/bin/bash
mkdir -p gpurun_out
for sc in 22; do
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/l10_$sc.csv python scripts/one_count.py rmat${sc}x 1-tailed-triangle 2 > /dev/null 2>&1
python scripts/launch_agg.py gpurun_out/l10_$sc.csv 4
done
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_q10.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_q10.log
for wl in internet rmat22; do
timeout 600 python bench.py --workload $wl --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_q10_$wl.json 2> gpurun_out/bench_q10_$wl.err; echo "$wl rc=$?"; tail -2 gpurun_out/bench_q10_$wl.err
python -c "
import json;d=json.load(open('gpurun_out/bench_q10_$wl.json'))
print('ms/step',d['ms_per_step'],'value',d['value'], 'e2e', d['e2e']['ms_per_step'])
for r in [d['roofline']]+d['roofline_other_kernels']: print(' ',r['kernel'][:50],'%.4f ms'%r['kernel_ms'],'frac %.3f'%r['frac'], r['algorithmic_bytes_per_launch'])
"
done
