#!/bin/bash
# value-load variants of the query kernel: steady-state DRAM bytes (single-pass ncu) and cfg2 timing
TAG=${1:-r2j}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
for v in 1 2; do python -m paper_conf_ppopp_zhangz0lzl23_b200.build --variant val$v -DEIRENE_VAL_LOAD=$v >> $OUT/build.log 2>&1; done
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
for v in 0 1 2; do
  L=paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so; [ $v != 0 ] && L=paper_conf_ppopp_zhangz0lzl23_b200/libeirene_val$v.so
  EIRENE_LIB=$L timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none \
    --clock-control none -k regex:query_kernel --csv --log-file $OUT/q$v.csv $BENCH > $OUT/q$v.log 2>&1
  EIRENE_LIB=$L timeout 300 python bench.py --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench_v$v.log 2>&1
done
for v in 0 1 2; do echo "== val$v"; python tools/traffic1.py $OUT/q$v.csv 3 | head -2; tail -1 $OUT/bench_v$v.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('value', round(d['value'],3), 'query', round(d['stage_ms']['query']*1e3,1), 'parity', d['parity']['mismatches'])"; done
