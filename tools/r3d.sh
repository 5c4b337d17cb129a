#!/bin/bash
# update kernel: one-round-trip update_needed / publish (A/B vs HEAD on cfg2); split-storm phase times (cfg1, cfg4)
OUT=gpurun_out/r3d; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab_libs.sh r3d2 2 $P/libeirene_head.so $P/libeirene.so
for c in 1 4; do
  EIRENE_UPDATE_PROF=1 timeout 600 python bench.py --config $c --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/uprof$c.log 2>&1
  echo "== cfg$c"; grep "upd prof" $OUT/uprof$c.log | tail -3
done
