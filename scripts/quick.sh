#!/bin/bash
# Fast GPU iteration: the edge/triangle-core parity tests + the default bench.
#   gpurun --timeout 900 -- 'bash scripts/quick.sh TAG [pytest -k expr]'
TAG=${1:-q}
K=${2:-"fig2 or small_patterns or pl2k or internet or beyond_64 or overflow or degenerate or batch"}
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_$TAG.log
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
python -c "
import json;d=json.load(open('gpurun_out/bench_$TAG.json'))
print('ms/step',d['ms_per_step'],'value',d['value'],'e2e',d['e2e']['ms_per_step'])
for r in [d['roofline']]+d['roofline_other_kernels']: print(' ',r['kernel'][:40],'%.4f ms'%r['kernel_ms'],'frac %.3f'%r['frac'])
" 2>&1 | tail -5
