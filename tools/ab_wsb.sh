#!/bin/bash
OUT=gpurun_out/abwsb_${1:-x}
mkdir -p $OUT
for v in ${VARIANTS:-default wsb256 wsb512}; do
  if [ $v = default ]; then L=""; else L=variants/libeirene_$v.so; fi
  EIRENE_LIB=$L timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "hot_key or mixes or dense or storm" > $OUT/$v.tests.log 2>&1; echo "$v tests rc=$?"
  EIRENE_LIB=$L timeout 600 python bench.py --config 3 --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 2 --ra-probe 0 > $OUT/$v.cfg3.log 2>&1
  tail -1 $OUT/$v.cfg3.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v cfg', d['config']['cfg'], round(d['value'],3), {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, d['parity']['mismatches'])"
done
