#!/bin/bash
# update-kernel phase times (EIRENE_UPDATE_PROF) and one full ncu capture of it, cfg1 / cfg4
OUT=gpurun_out/upd_${1:-x}
mkdir -p $OUT
for c in 4 1; do
  EIRENE_UPDATE_PROF=1 timeout 600 python bench.py --config $c --steps 4 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/prof_cfg$c.log 2>&1
  grep "upd prof" $OUT/prof_cfg$c.log | tail -4
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel -s 3 -c 1 -o $OUT/upd_cfg4 python bench.py --config 4 --steps 1 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/ncu_cfg4.log 2>&1
ls -la $OUT
# group kernel under Zipf hot keys: cfg3 and a cfg5-sized batch (2^24 requests) on a 2^24-key tree
timeout 600 ncu --set full --clock-control none --import-source on -k regex:group_kernel -s 3 -c 1 -o $OUT/grp_cfg3 python bench.py --config 3 --steps 1 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/ncu_grp3.log 2>&1
timeout 600 python bench.py --config 5 --tree 16777216 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/cfg5s.log 2>&1
tail -1 $OUT/cfg5s.log | cut -c1-900
timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -s 3 -c 1 -o $OUT/grp_cfg5s python bench.py --config 5 --tree 16777216 --steps 1 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/ncu_grp5.log 2>&1
ls -la $OUT
