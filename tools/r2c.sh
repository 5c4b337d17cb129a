#!/bin/bash
# GPU suite, PDL / host-event A/B on cfg2, multi-GPU code path on one GPU (gloo, 2 ranks, parity), cfg5 N=1 mix B
TAG=${1:-r2c}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
B="python bench.py --steps 20 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0"
for v in "0 0" "1 0" "0 1" "1 1"; do set -- $v
  EIRENE_PDL=$1 EIRENE_BENCH_NO_EVENTS=$([ $2 = 1 ] && echo 1) EIRENE_BENCH_VERBOSE=1 timeout 300 $B > $OUT/bench_pdl$1_noev$2.log 2>&1
done
EIRENE_PDL=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > $OUT/gpu_tests_pdl.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests_pdl.log
EIRENE_BENCH_ONE_GPU=1 timeout 900 python bench.py --gpus 2 --backend gloo --steps 5 --warmup 3 --e2e-steps 3 > $OUT/gloo2.log 2>&1
timeout 1200 python bench.py --config 5 --mix B --steps 10 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/cfg5B.log 2>&1
tail -2 $OUT/gpu_tests.log; tail -2 $OUT/gpu_tests_pdl.log
for v in "0 0" "1 0" "0 1" "1 1"; do set -- $v; f=$OUT/bench_pdl$1_noev$2.log; echo "== pdl $1 noev $2"; grep -E "device gap" $f | cut -c1-150; tail -1 $f | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('value', round(d['value'],3), 'dev batch', round(d['batch_ms']['mean']*1e3,1), 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'parity', d['parity'])"; done
tail -1 $OUT/gloo2.log | cut -c1-400; grep -E "parity|e2e" -o $OUT/gloo2.log | head -2; tail -1 $OUT/gloo2.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('gloo2', d['n_gpus'], d['parity'], d['e2e'])"
tail -1 $OUT/cfg5B.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg5B', round(d['value'],3), {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, d['parity'], d['roofline'] and round(d['roofline']['frac'],3))"
