#!/bin/bash
P=tricore+3f,fig4,k4core+2f
for v in "" "FSGC_NO_VENN_TERMS=1"; do env $v timeout 120 python scripts/debug_variants.py pl2k $P 2; done
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_q4.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_q4.log
timeout 600 python bench.py --workload pl10m --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_q4_pl10m.json 2> gpurun_out/bench_q4_pl10m.err; echo "pl10m rc=$?"; head -c 300 gpurun_out/bench_q4_pl10m.json; tail -3 gpurun_out/bench_q4_pl10m.err
python -c "
import json;d=json.load(open('gpurun_out/bench_q4_pl10m.json'))
print('ms/step',d['ms_per_step'],'value',d['value'])
for r in [d['roofline']]+d['roofline_other_kernels']: print(' ',r['kernel'][:50],'%.4f ms'%r['kernel_ms'],'frac %.3f'%r['frac'])
"
