#!/bin/bash
# A/B/.. of library builds on the same box, interleaved: bash tools/ab_libs.sh TAG CFG LIB1 LIB2 [LIB3 ...]
TAG=$1; CFG=$2; shift 2
OUT=gpurun_out/ab_$TAG
mkdir -p $OUT
for r in 1 2 3; do i=0; for L in "$@"; do i=$((i+1))
  EIRENE_LIB=$L timeout 300 python bench.py --config $CFG --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/${i}_$r.log 2>&1
  tail -1 $OUT/${i}_$r.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('$i', '$(basename $L)', '$r', round(d['value'],3), 'dev', round(d['batch_ms']['mean']*1e3,1), 'step', round(d['ms_per_step']*1e3,1), {k: round(x*1e3,1) for k,x in d['stage_ms'].items()})"
done; done
