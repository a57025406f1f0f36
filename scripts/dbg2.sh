#!/bin/bash
mkdir -p gpurun_out
timeout 300 python scripts/debug_support.py 16 16 > gpurun_out/dbg_sup16.txt 2>&1; echo "sup16 rc=$?"; cat gpurun_out/dbg_sup16.txt
timeout 300 python scripts/debug_support.py 14 16 > gpurun_out/dbg_sup14.txt 2>&1; echo "sup14 rc=$?"; tail -3 gpurun_out/dbg_sup14.txt
timeout 900 python -m pytest tests -m gpu -x -q -k "venn or pl2k or fig2 or small_patterns or hub or symmetry" > gpurun_out/pytest_q2.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_q2.log
timeout 600 python bench.py --workload pl10m --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_q2_pl10m.json 2> gpurun_out/bench_q2_pl10m.err; echo "pl10m rc=$?"; head -c 600 gpurun_out/bench_q2_pl10m.json; tail -3 gpurun_out/bench_q2_pl10m.err
