#!/bin/bash
# one bench line per config (diagnostic sweep; the default run is cfg2)
OUT=gpurun_out/allcfg_${1:-x}
mkdir -p $OUT
for c in ${CFGS:-1 2 3 4 6}; do
  timeout 600 python bench.py --config $c ${BENCH_ARGS} > $OUT/cfg$c.log 2>&1
  tail -1 $OUT/cfg$c.log | python -c "
import json,sys
try:
    d=json.loads(sys.stdin.read())
    print('cfg $c', round(d['value'],3), d['unit'], {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3), 'parity', (d['parity'] or {}).get('mismatches'), 'roof', d['roofline'] and (d['roofline']['kernel'], round(d['roofline']['frac'],3)), 'e2e', d['e2e'] and d['e2e']['value'])
except Exception as e: print('cfg $c FAILED', e)"
done
