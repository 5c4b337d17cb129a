#!/bin/bash
# pipelined batches (EIRENE_F_PIPELINE) A/B on cfg2 / cfg3, GPU suite
TAG=${1:-r2g}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
for c in 2 3; do for p in 0 1; do
  EIRENE_BENCH_VERBOSE=1 timeout 300 python bench.py --config $c --pipeline $p --steps 30 --warmup 5 --e2e-steps 11 --cpu-batches 2 --ra-probe 0 > $OUT/bench${c}_p$p.log 2>&1
done; done
tail -3 $OUT/gpu_tests.log
for c in 2 3; do for p in 0 1; do tail -1 $OUT/bench${c}_p$p.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], 'pipe $p value', round(d['value'],3), 'ms/step', round(d['ms_per_step']*1e3,1), 'dev batch', round(d['batch_ms']['mean']*1e3,1), 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3), 'e2e', round(d['e2e']['value'],3), 'parity', d['parity']['mismatches'])"; done; done
