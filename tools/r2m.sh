#!/bin/bash
TAG=${1:-r2m}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
for c in 2 3 7; do timeout 300 python bench.py --config $c --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench_c$c.log 2>&1; done
tail -3 $OUT/gpu_tests.log
for c in 2 3 7; do tail -1 $OUT/bench_c$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], 'value', round(d['value'],3), 'ms/step', round(d['ms_per_step']*1e3,1), 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'parity', d['parity']['mismatches'])"; done
