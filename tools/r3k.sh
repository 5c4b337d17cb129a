#!/bin/bash
# deferred hot keys: bitmap bits set by every CTA of the query kernel (payloads compacted by the group CTA)
OUT=gpurun_out/r3k; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab2.sh r3k3 3 20 2 $P/libeirene_head.so $P/libeirene.so
for L in libeirene_head.so libeirene.so; do
  EIRENE_LIB=$P/$L timeout 900 python bench.py --config 5 --mix B --steps 4 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/c5B_$L.log 2>&1
  tail -1 $OUT/c5B_$L.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg5B $L', round(d['value'],3), {k: round(x*1e3,1) for k,x in d['stage_ms'].items()}, d['parity'])"
done
