#!/bin/bash
# update-kernel phase times under split storms (EIRENE_UPDATE_PROF) for cfg1 / cfg4; launch lists
OUT=gpurun_out/r2y; mkdir -p $OUT
for c in 1 4; do
  EIRENE_UPDATE_PROF=1 timeout 600 python bench.py --config $c --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/uprof_cfg$c.log 2>&1
  grep "upd prof" $OUT/uprof_cfg$c.log | tail -4
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/l$c.csv python bench.py --config $c --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > /dev/null 2>&1
  python tools/launches.py $OUT/l$c.csv 2 2>/dev/null | head -6
done
