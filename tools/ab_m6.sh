#!/bin/bash
OUT=gpurun_out/abm6
mkdir -p $OUT
for v in default minb6; do
  if [ $v = default ]; then L=""; else L=variants/libeirene_$v.so; fi
  for c in 1 4 2; do
    EIRENE_LIB=$L timeout 600 python bench.py --config $c --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/$v.cfg$c.log 2>&1
    tail -1 $OUT/$v.cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v cfg', d['config']['cfg'], round(d['value'],3), round(d['stage_ms']['update']*1e3,1), d['parity']['mismatches'])"
  done
done
