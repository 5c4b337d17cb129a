#!/bin/bash
# one warm-cache (--cache-control none) full capture of the kernels matching $2
TAG=${1:-x}
KRE=${2:-"bsort_|combine_kernel|partition_kernel"}
CNT=${3:-8}
OUT=gpurun_out/ncuw_$TAG
mkdir -p $OUT
ncu --set full --cache-control none --clock-control none --import-source on -k "regex:$KRE" -s ${SKIP:-10} -c $CNT -o $OUT/full \
  python tools/ab.py --reps 1 --steps 12 X=1 > $OUT/log.txt 2>&1
python tools/ncu_summary.py $OUT/full.ncu-rep > $OUT/summary.txt 2>&1
cat $OUT/summary.txt
