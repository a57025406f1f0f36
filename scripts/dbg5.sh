#!/bin/bash
mkdir -p gpurun_out
timeout 300 python scripts/debug_support.py 16 16 > gpurun_out/dbg5_sup16.txt 2>&1; echo "sup16 rc=$?"; cat gpurun_out/dbg5_sup16.txt
timeout 300 python scripts/debug_support.py 20 16 > gpurun_out/dbg5_sup20.txt 2>&1; echo "sup20 rc=$?"; tail -3 gpurun_out/dbg5_sup20.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_q5.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_q5.log
for wl in internet rmat22; do
timeout 600 python bench.py --workload $wl --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_q5_$wl.json 2> gpurun_out/bench_q5_$wl.err; echo "$wl rc=$?"; tail -2 gpurun_out/bench_q5_$wl.err
python -c "
import json;d=json.load(open('gpurun_out/bench_q5_$wl.json'))
print('ms/step',d['ms_per_step'],'value',d['value'], 'e2e', d['e2e']['ms_per_step'])
for r in [d['roofline']]+d['roofline_other_kernels']: print(' ',r['kernel'][:50],'%.4f ms'%r['kernel_ms'],'frac %.3f'%r['frac'])
"
done
FSGC_SUP_MERGE_ONLY=1 timeout 600 python bench.py --workload rmat22 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_q5m.json 2>&1; python -c "
import json;d=json.load(open('gpurun_out/bench_q5m.json'))
print('merge-only ms/step',d['ms_per_step'])"
