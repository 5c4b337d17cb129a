#!/bin/bash
# warm-cache full capture of the range kernel on the range workload (cfg6)
TAG=${1:-r}
OUT=gpurun_out/ncu_range_$TAG
mkdir -p $OUT
ncu --set full --cache-control none --clock-control none --import-source on -k "regex:range_kernel" -s 6 -c 2 -o $OUT/full \
  python bench.py --config 6 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/log.txt 2>&1
python tools/ncu_summary.py $OUT/full.ncu-rep > $OUT/summary.txt 2>&1
cat $OUT/summary.txt
