#!/bin/bash
# triangle-core kernel: t only when the Venn needs it; GPU suite + timings + ncu
OUT=gpurun_out; mkdir -p $OUT
TAG=r01o
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu.py::test_rmat26_full_size_wedge_hash_equals_merge > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log; tail -3 $OUT/pytest_gpu_$TAG.log
timeout 240 python scripts/rmat26_probe.py 20 "tricore+1f;tricore+2f;tricore+3f" > $OUT/probe20_$TAG.log 2>&1; echo "probe20 rc=$?"; tail -8 $OUT/probe20_$TAG.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'tri_core_kernel' -c 1 \
  -o $OUT/prof_${TAG}_rmat18 -f python scripts/one_count.py rmat18x tricore+3f 1 > $OUT/ncu_full_${TAG}_rmat18.log 2>&1; echo "ncu full rc=$?"
for r in $OUT/prof_${TAG}_*.ncu-rep; do
  ncu -i $r --page raw --csv > ${r%.ncu-rep}_raw.csv 2>/dev/null
  ncu -i $r --page source --csv > ${r%.ncu-rep}_source.csv 2>/dev/null
  rm -f $r
done
