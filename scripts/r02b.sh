#!/bin/bash
OUT=gpurun_out
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
timeout 900 python scripts/one_count.py rmat26 $P26 2 > $OUT/probe_r02b.log 2>&1; echo "rmat26 rc=$?" >> $OUT/probe_r02b.log
cat $OUT/probe_r02b.log
timeout 1200 python bench.py --no-per-config --steps 3 --warmup 1 --e2e-steps 1 > $OUT/bench_r02b.json 2> $OUT/bench_r02b.err; echo "bench rc=$?"
tail -30 $OUT/bench_r02b.err
