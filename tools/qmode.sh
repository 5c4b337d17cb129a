#!/bin/bash
# diagnostic: query-kernel variants (EIRENE_QMODE / EIRENE_QCAP) on cfg2
for m in "0 8" "0 16" "0 32" "0 64" "4 32"; do
  set -- $m
  EIRENE_QMODE=$1 EIRENE_QCAP=$2 python bench.py --steps 30 --warmup 5 --cpu-batches 1 --e2e-steps 3 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('qmode $m', d['value']/1e9, d['ms_per_step'], d.get('stage_ms'))"
done
