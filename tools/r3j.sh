#!/bin/bash
# e2e: zero-copy upsert values vs copied values; cfg7 QCOOP A/B (32-bit); group phase profile cfg3
OUT=gpurun_out/r3j; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
for v in 0 1; do
  if [ $v = 1 ]; then export EIRENE_VALS_COPY=1; fi
  timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 21 --cpu-batches 0 --ra-probe 0 > $OUT/e2e_$v.log 2>&1
  tail -1 $OUT/e2e_$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('vals_copy=$v', round(d['value'],3), d['e2e'])"
done
unset EIRENE_VALS_COPY
for r in 1 2; do for L in libeirene32.so libeirene_q32.so; do
  EIRENE_LIB32=$P/$L timeout 300 python bench.py --config 7 --steps 20 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/c7_$L_$r.log 2>&1
  tail -1 $OUT/c7_$L_$r.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$L', round(d['value'],3), {k: round(x*1e3,1) for k,x in d['stage_ms'].items()})"
done; done
EIRENE_LIB=$P/libeirene_phase.so timeout 300 python tools/phase_prof.py 3 > $OUT/phase3.txt 2>&1; cat $OUT/phase3.txt
