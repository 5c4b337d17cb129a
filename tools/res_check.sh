#!/bin/bash
OUT=gpurun_out/res_${1:-x}
mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/tests.log 2>&1; echo "rc=$?" >> $OUT/tests.log
tail -2 $OUT/tests.log
for c in 3 2; do
  timeout 600 python bench.py --config $c --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 2 --ra-probe 0 > $OUT/cfg$c.log 2>&1
  tail -1 $OUT/cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], round(d['value'],3), {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, d['parity']['mismatches'])"
done
