#!/bin/bash
# Profiling recipe (B200_PROFILING.md): launch list + one full capture per hot kernel.
# usage: bash tools_profile.sh <tag>
set -x
TAG=${1:-r1}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
BENCH="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv $BENCH > $OUT/launches_bench.log 2>&1
for K in sort_pass_kernel update_kernel query_kernel combine_kernel; do
  ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 -o $OUT/$K $BENCH > $OUT/$K.log 2>&1
done
ls -la $OUT
