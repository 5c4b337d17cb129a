#!/bin/bash
OUT=gpurun_out/grp_${1:-x}
mkdir -p $OUT
EIRENE_GROUP_PROF=1 timeout 600 python bench.py --config 3 --steps 1 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/cfg3.log 2>&1
grep "group prof" $OUT/cfg3.log | sort -t' ' -k13 -g -r | head -5; grep -c "group prof" $OUT/cfg3.log
EIRENE_GROUP_PROF=1 timeout 600 python bench.py --config 5 --tree 16777216 --steps 1 --warmup 1 --e2e-steps 0 --cpu-batches 0 > $OUT/cfg5s.log 2>&1
grep -c "group prof" $OUT/cfg5s.log; grep "group prof" $OUT/cfg5s.log | awk '{print $7, $8, $9, $10, $11, $12, $13, $14, $15, $16}' | sort | uniq -c | sort -rn | head -3
grep "group prof" $OUT/cfg5s.log | sort -k11 -g -r | head -8
grep "group prof" $OUT/cfg5s.log | sort -k13 -g -r | head -8
