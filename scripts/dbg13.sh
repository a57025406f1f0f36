#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_q13.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_q13.log
for wl in pl10m rmat16; do
timeout 900 python bench.py --workload $wl --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_q13_$wl.json 2> gpurun_out/bench_q13_$wl.err; echo "$wl rc=$?"; tail -2 gpurun_out/bench_q13_$wl.err
python -c "
import json;d=json.load(open('gpurun_out/bench_q13_$wl.json'))
print('ms/step',d['ms_per_step'],'value',d['value'])
for r in [d['roofline']]+d['roofline_other_kernels']: print(' ',r['kernel'][:50],'%.4f ms'%r['kernel_ms'],'frac %.3f'%r['frac'], r['algorithmic_bytes_per_launch'])
"
done
