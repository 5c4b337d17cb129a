#!/bin/bash
# round-2 first check: full GPU suite, smoke, cfg2 bench (verbose batch times), cfg3/1/4 lines, sanitizers
TAG=${1:-r2a}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
EIRENE_BENCH_VERBOSE=1 timeout 600 python bench.py --steps 20 --warmup 5 > $OUT/bench.log 2>&1
CFGS="1 3 4" BENCH_ARGS="--e2e-steps 0 --cpu-batches 1 --ra-probe 0" bash tools/allcfg.sh $TAG > $OUT/allcfg.txt 2>&1
timeout 1500 bash tools/sanitize.sh $TAG > $OUT/sanitize.txt 2>&1
tail -3 $OUT/gpu_tests.log; tail -1 $OUT/smoke.log; cat $OUT/allcfg.txt; cat $OUT/sanitize.txt
tail -1 $OUT/bench.log | cut -c1-1500
grep "batch ms" $OUT/bench.log
