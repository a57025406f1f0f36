#!/bin/bash
# ncu full capture of the listing kernels; only CSV extracts come back
# usage: [SKIP=n] ncu_r02.sh TAG WORKLOAD PATTERNS [KERNEL_REGEX] [COUNT]
TAG=$1; WL=$2; PATS=$3; KRE=${4:-list_}; CNT=${5:-4}
OUT=gpurun_out
TMP=/tmp/ncu_$TAG
mkdir -p $TMP $OUT
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:$KRE -s ${SKIP:-0} -c $CNT \
  -o $TMP/prof -f python scripts/one_count.py $WL $PATS 1 > $OUT/ncu_${TAG}_${WL}.log 2>&1
echo "ncu rc=$?"
ncu -i $TMP/prof.ncu-rep --page raw --csv > $OUT/prof_${TAG}_${WL}_raw.csv 2>/dev/null
for k in list_block_kernel list_warp_kernel core_kernel edge_fc_kernel; do
  ncu -i $TMP/prof.ncu-rep --page source --csv --print-source sass --kernel-name regex:$k > $TMP/src_$k.csv 2>/dev/null
  python scripts/src_hot.py $TMP/src_$k.csv 60 $OUT/prof_${TAG}_${WL}_offs_$k.csv > $OUT/prof_${TAG}_${WL}_hot_$k.txt 2>&1
  ncu -i $TMP/prof.ncu-rep --page source --csv --print-source cuda --kernel-name regex:$k > $TMP/cu_$k.csv 2>/dev/null
  python scripts/src_hot.py $TMP/cu_$k.csv 80 > $OUT/prof_${TAG}_${WL}_cuhot_$k.txt 2>&1; head -c 3000 $TMP/cu_$k.csv > $OUT/prof_${TAG}_${WL}_cuhead_$k.txt
done
ls -la $OUT | grep $TAG
