#!/bin/bash
# end-of-round measurement: GPU tests, default bench, launch list + full ncu
# capture of the default workload, bench lines of the other configs, full ncu
# captures of the big-graph kernels.  Reports are exported to CSV on the box
# and deleted (gpurun copies back at most 64 MiB).
TAG=${1:-r01k}
OUT=gpurun_out
bash scripts/gpu_check.sh $TAG internet
bash scripts/bench_configs.sh $TAG "pl2k rmat22 pl10m rmat16"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'support_hash_kernel|edge_fc_kernel' -s 3 -c 3 \
  -o $OUT/prof_${TAG}_rmat22 -f python scripts/one_count.py rmat22 1-tailed-triangle,2-tailed-triangle,3-tailed-triangle,4-tailed-triangle,triangle,diamond 2 > $OUT/ncu_full_${TAG}_rmat22.log 2>&1; echo "ncu rmat22 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'tri_core_kernel|support_hash' -c 3 \
  -o $OUT/prof_${TAG}_pl10m -f python scripts/one_count.py pl10m fig4 1 > $OUT/ncu_full_${TAG}_pl10m.log 2>&1; echo "ncu pl10m rc=$?"
for r in $OUT/prof_${TAG}_*.ncu-rep; do
  ncu -i $r --page raw --csv > ${r%.ncu-rep}_raw.csv 2>/dev/null
  ncu -i $r --page details --csv > ${r%.ncu-rep}_details.csv 2>/dev/null
  rm -f $r
done
du -sh $OUT
