#!/bin/bash
# plain resident-grid launches by default (cooperative with pipelined handles / EIRENE_COOP=1): GPU suite, cfg2 / pipelined / COOP
OUT=gpurun_out/r3p; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
A="--steps 30 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0"
for v in plain coop pipeline; do
  case $v in coop) export EIRENE_COOP=1;; pipeline) unset EIRENE_COOP; X="--pipeline 1";; *) X="";; esac
  timeout 300 python bench.py $A $X > $OUT/c2_$v.log 2>&1
  tail -1 $OUT/c2_$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value'],3), round(d['batch_ms']['mean']*1e3,1), d['parity']['mismatches'])"
done
