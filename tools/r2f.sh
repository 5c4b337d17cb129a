#!/bin/bash
# dist kernel atomics fix: phase profile cfg2, single-pass traffic per kernel, cfg2/3 bench, GPU suite
TAG=${1:-r2f}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
python -m paper_conf_ppopp_zhangz0lzl23_b200.build --variant phase -DEIRENE_PHASE_PROF >> $OUT/build.log 2>&1
EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/libeirene_phase.so timeout 300 python tools/phase_prof.py 2 > $OUT/phase_cfg2.txt 2>&1
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none \
  --clock-control none --csv --log-file $OUT/launches.csv $BENCH > $OUT/launches_bench.log 2>&1
python tools/traffic1.py $OUT/launches.csv 3 > $OUT/traffic1.txt 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench2.log 2>&1
timeout 300 python bench.py --config 3 --steps 20 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench3.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
head -9 $OUT/phase_cfg2.txt; head -8 $OUT/traffic1.txt; tail -2 $OUT/gpu_tests.log
for c in 2 3; do tail -1 $OUT/bench$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], 'value', round(d['value'],3), 'ms/step', round(d['ms_per_step']*1e3,1), 'dev batch', round(d['batch_ms']['mean']*1e3,1), 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'parity', d['parity']['mismatches'])"; done
