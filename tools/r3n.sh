#!/bin/bash
# update kernel: register budget A/B (6 / 7 / 8 resident CTAs per SM) on cfg4, cfg1; cost of the cooperative launch
# of a no-op update kernel on cfg2 (EIRENE_NO_LSYNC=1: plain launch)
OUT=gpurun_out/r3n; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab2.sh r3n4 4 10 1 $P/libeirene.so $P/libeirene_minb7.so $P/libeirene_minb8.so
bash tools/ab2.sh r3n1 1 20 1 $P/libeirene.so $P/libeirene_minb7.so $P/libeirene_minb8.so
for v in 0 1; do
  if [ $v = 1 ]; then export EIRENE_NO_LSYNC=1; fi
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/nolsync_$v.log 2>&1
  tail -1 $OUT/nolsync_$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('no_lsync=$v', round(d['value'],3), round(d['batch_ms']['mean']*1e3,1), {k: round(x*1e3,1) for k,x in d['stage_ms'].items()})"
done
