#!/bin/bash
# quick GPU check: parity suites + short cfg2 / cfg6 bench lines (diagnostic)
OUT=gpurun_out/quick_${1:-x}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_range.py -x -q > $OUT/tests.log 2>&1; echo "rc=$?" >> $OUT/tests.log
for c in 2 6; do
  timeout 300 python bench.py --config $c --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 > $OUT/bench$c.log 2>&1
done
tail -2 $OUT/tests.log
for c in 2 6; do tail -1 $OUT/bench$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], 'value', round(d['value'],3), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'frac', round(d['roofline']['frac'],3), 'parity', d['parity']['mismatches'], 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3))"; done
