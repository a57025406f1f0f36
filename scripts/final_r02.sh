#!/bin/bash
# Round-2 measurement of the committed build, one gpurun call:
#   1. ncu metrics of the listing kernels on the configs[4] workload (RMAT-26,
#      the bench's pattern set) -> profiles/ncu_r02_summary.json (the bench's
#      traffic and issue-rate roofline read it)
#   2. ncu launch list of the bench command (per-launch durations)
#   3. the GPU test suite, smoke(), the default bench line
OUT=gpurun_out
TAG=${1:-r02z}
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $OUT/gpu_$TAG.txt
if [ "${SKIP_NCU:-0}" != "1" ]; then
timeout 1200 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,launch__occupancy_limit_shared_mem,launch__occupancy_limit_registers,launch__registers_per_thread,launch__grid_size,launch__block_size --clock-control none -k regex:list_ --csv --log-file $OUT/ncum_${TAG}_rmat26.csv python scripts/one_count.py rmat26 triangle/tricore,tricore+1f,tricore+2f,2-tailed-triangle/tricore,3-tailed-triangle/tricore,4-tailed-triangle/tricore,diamond/tricore 1 > $OUT/ncum_${TAG}.log 2>&1; echo "ncu metrics rc=$?"
python scripts/ncu_r02_summary.py $TAG rmat26 $OUT/ncum_${TAG}_rmat26.csv > /dev/null && cp profiles/ncu_r02_summary.json $OUT/ncu_r02_summary.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_${TAG}_rmat26.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config > $OUT/launches_${TAG}.log 2>&1; echo "ncu launches rc=$?"
fi
if [ "${SKIP_TESTS:-0}" != "1" ]; then
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu_$TAG.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke_$TAG.log
fi
timeout 2400 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
tail -25 $OUT/bench_$TAG.err
