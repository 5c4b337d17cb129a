#!/bin/bash
# split storms: leaf runs of a chunk applied together (UPD_BATCH) -- GPU parity suite, A/B cfg1 / cfg4, phase times
OUT=gpurun_out/r3f; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -3 $OUT/gpu_tests.log
bash tools/ab_libs.sh r3f4 4 $P/libeirene_nobatch.so $P/libeirene.so
bash tools/ab_libs.sh r3f1 1 $P/libeirene_nobatch.so $P/libeirene.so
for c in 1 4; do
  EIRENE_UPDATE_PROF=1 timeout 600 python bench.py --config $c --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/uprof$c.log 2>&1
  echo "== cfg$c"; grep "upd prof" $OUT/uprof$c.log | tail -2; tail -1 $OUT/uprof$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['parity'])"
done
