#!/bin/bash
OUT=gpurun_out/final_${1:-x}
mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/tests.log 2>&1; echo "rc=$?" >> $OUT/tests.log
tail -2 $OUT/tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench.log 2>&1
tail -1 $OUT/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['e2e']['value'], d['random_access_roofline']['frac'], d['roofline']['frac'], d['parity'], d['batch_ms']['variance_maxmin_over_mean'])"
CFGS="1 3 4 6" BENCH_ARGS="--e2e-steps 0 --cpu-batches 1 --ra-probe 0" bash tools/allcfg.sh $1 > $OUT/allcfg.txt 2>&1
cat $OUT/allcfg.txt
