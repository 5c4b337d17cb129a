#!/bin/bash
# hot sub-bucket timestamp sort (cfg3), new random-access probes (cfg2 default bench line), GPU suite
TAG=${1:-r2h}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
python -m paper_conf_ppopp_zhangz0lzl23_b200.build --variant phase -DEIRENE_PHASE_PROF >> $OUT/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/libeirene_phase.so timeout 300 python tools/phase_prof.py 3 > $OUT/phase_cfg3.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > $OUT/bench2.log 2>&1
timeout 300 python bench.py --config 3 --steps 20 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench3.log 2>&1
tail -2 $OUT/gpu_tests.log; cat $OUT/phase_cfg3.txt | tail -6
for c in 2 3; do tail -1 $OUT/bench$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], 'value', round(d['value'],3), 'ms/step', round(d['ms_per_step']*1e3,1), 'dev batch', round(d['batch_ms']['mean']*1e3,1), 'var', round(d['batch_ms']['variance_maxmin_over_mean'],3), 'stages', {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, 'parity', d['parity']['mismatches'])
print(json.dumps(d.get('random_access_roofline'))[:900]); print(json.dumps(d.get('roofline'))[:700])"; done
