#!/bin/bash
# skew-adaptive group count (twice the groups when a bin holds > 1/4 of a base group): GPU suite, A/B cfg3 / cfg2
OUT=gpurun_out/r3m; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab2.sh r3m3 3 20 2 $P/libeirene_head.so $P/libeirene.so
bash tools/ab2.sh r3m2 2 20 2 $P/libeirene_head.so $P/libeirene.so
for m in A B; do
  timeout 900 python bench.py --config 5 --mix $m --steps 4 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/c5$m.log 2>&1
  tail -1 $OUT/c5$m.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg5$m', round(d['value'],3), {k: round(x*1e3,1) for k,x in d['stage_ms'].items()}, d['parity']['mismatches'])"
done
