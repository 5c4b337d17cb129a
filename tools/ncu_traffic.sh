#!/bin/bash
# DRAM traffic of the dominant kernel for bench.py's roofline "traffic" field:
# one ncu --set full capture per kernel launch of the bench workload, caches
# NOT flushed between replays' originals (--cache-control none: steady state,
# inner levels L2-resident as in the timed run), clocks unlocked.
TAG=${1:-r1}
K=${2:-query_kernel}
OUT=gpurun_out/traffic_$TAG
mkdir -p $OUT
ncu --set full --cache-control none --clock-control none --import-source on -k "regex:$K" -s 6 -c 3 -o $OUT/full \
  python bench.py --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/log.txt 2>&1
python tools/ncu_summary.py $OUT/full.ncu-rep > $OUT/summary.txt 2>&1
cat $OUT/summary.txt
