#!/bin/bash
OUT=gpurun_out
TAG=${1:-r02o}
P26=$(python -c "from inputs.patterns import CONFIG_PATTERNS as C; print(','.join(C['rmat26']))")
timeout 900 python -m pytest tests -m gpu -x -q -k "triangle or tri or venn or rmat_hubs or pl2k or small_patterns or z_tiers" > $OUT/pytest_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_$TAG.log
timeout 300 python scripts/one_count.py rmat20x $P26 3 > $OUT/probe_$TAG.log 2>&1
timeout 600 python scripts/one_count.py rmat26 $P26 1 >> $OUT/probe_$TAG.log 2>&1
timeout 600 python scripts/one_count.py rmat26 triangle/tricore 1 >> $OUT/probe_$TAG.log 2>&1
cut -c1-300 $OUT/probe_$TAG.log
timeout 900 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,launch__occupancy_limit_shared_mem,launch__occupancy_limit_registers --clock-control none -k regex:list_ --csv --log-file $OUT/ncum_${TAG}_rmat26.csv python scripts/one_count.py rmat26 $P26 1 > /dev/null 2>&1; echo "ncu rc=$?"
