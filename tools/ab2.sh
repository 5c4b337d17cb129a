#!/bin/bash
# lean A/B of library builds: bash tools/ab2.sh TAG CFG STEPS REPS LIB1 LIB2 [...]
TAG=$1; CFG=$2; STEPS=$3; REPS=$4; shift 4
OUT=gpurun_out/ab_$TAG
mkdir -p $OUT
for r in $(seq 1 $REPS); do i=0; for L in "$@"; do i=$((i+1))
  EIRENE_LIB=$L timeout 300 python bench.py --config $CFG --steps $STEPS --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/${i}_$r.log 2>&1
  tail -1 $OUT/${i}_$r.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('$i', '$(basename $L)', '$r', round(d['value'],3), 'dev', round(d['batch_ms']['mean']*1e3,1), 'step', round(d['ms_per_step']*1e3,1), {k: round(x*1e3,1) for k,x in d['stage_ms'].items()})"
done; done
