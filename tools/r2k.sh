#!/bin/bash
# merged update + result phase (one kernel fewer), value-line L2 prefetch A/B, GPU suite
TAG=${1:-r2k}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
python -m paper_conf_ppopp_zhangz0lzl23_b200.build --variant val3 -DEIRENE_VAL_LOAD=3 >> $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
for v in 0 3; do
  L=paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so; [ $v != 0 ] && L=paper_conf_ppopp_zhangz0lzl23_b200/libeirene_val$v.so
  EIRENE_LIB=$L timeout 300 python bench.py --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench_v$v.log 2>&1
  EIRENE_LIB=$L timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none \
    --clock-control none --csv --log-file $OUT/l$v.csv python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/l$v.log 2>&1
done
for c in 1 3 4; do timeout 300 python bench.py --config $c --steps 20 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench_c$c.log 2>&1; done
tail -3 $OUT/gpu_tests.log
for v in 0 3; do echo "== val$v"; python tools/traffic1.py $OUT/l$v.csv 3 | head -6; tail -1 $OUT/bench_v$v.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('value', round(d['value'],3), 'ms/step', round(d['ms_per_step']*1e3,1), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'parity', d['parity']['mismatches'])"; done
for c in 1 3 4; do tail -1 $OUT/bench_c$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], 'value', round(d['value'],3), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'parity', d['parity']['mismatches'])"; done
