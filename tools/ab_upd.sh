#!/bin/bash
OUT=gpurun_out/abupd_${1:-x}
mkdir -p $OUT
for v in default minb6 minb4; do
  if [ $v = default ]; then L=""; else L=variants/libeirene_$v.so; fi
  for c in 4 1; do
    EIRENE_LIB=$L timeout 600 python bench.py --config $c --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/$v.cfg$c.log 2>&1
    tail -1 $OUT/$v.cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v cfg', d['config']['cfg'], round(d['value'],3), {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, d['parity']['mismatches'])"
  done
done
