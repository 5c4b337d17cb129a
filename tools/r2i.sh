#!/bin/bash
# 32-bit key build (NEXT(4)): GPU suite incl. tests/test_gpu_key32.py, cfg7 bench line, cfg2 line
TAG=${1:-r2i}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
timeout 600 python bench.py --config 7 --steps 20 --warmup 5 > $OUT/bench7.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --ra-probe 0 > $OUT/bench2.log 2>&1
tail -5 $OUT/gpu_tests.log
for c in 7 2; do tail -1 $OUT/bench$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], d['dtype'], 'value', round(d['value'],3), 'ms/step', round(d['ms_per_step']*1e3,1), 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'parity', d['parity'], 'e2e', d['e2e'] and round(d['e2e']['value'],3), 'roof', d['roofline'] and round(d['roofline']['frac'],3))"; done
tail -3 $OUT/bench7.log | cut -c1-300
