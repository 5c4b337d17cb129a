#!/bin/bash
# Profiling recipe (B200_PROFILING.md): launch list + one full capture per hot kernel.
# usage: bash tools_profile.sh <tag> [kernel-regex]
TAG=${1:-r1}
KRE=${2:-"group_kernel|query_kernel|update_kernel|bsort_|result_long|finalize"}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
BENCH="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv $BENCH > $OUT/launches_bench.log 2>&1
python tools/launches.py $OUT/launches.csv 2 > $OUT/launches_summary.txt
ncu --set full --clock-control none --import-source on -k "regex:$KRE" -s 40 -c 12 -o $OUT/full $BENCH > $OUT/full.log 2>&1
ls -la $OUT
