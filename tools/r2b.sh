#!/bin/bash
# launch list + single-pass steady-state DRAM traffic per kernel (cfg2 bench), gap study, full GPU suite
TAG=${1:-r2b}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none \
  --clock-control none --csv --log-file $OUT/launches.csv $BENCH > $OUT/launches_bench.log 2>&1
python tools/traffic1.py $OUT/launches.csv 3 > $OUT/traffic1.txt 2>&1
EIRENE_BENCH_VERBOSE=1 timeout 300 python bench.py --steps 20 --warmup 5 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/bench_graph.log 2>&1
EIRENE_NO_GRAPHS=1 EIRENE_BENCH_VERBOSE=1 timeout 300 python bench.py --steps 20 --warmup 5 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/bench_nograph.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
cat $OUT/traffic1.txt; tail -3 $OUT/gpu_tests.log
for f in bench_graph bench_nograph; do echo $f; grep -E "device gap|device batch" $OUT/$f.log; tail -1 $OUT/$f.log | cut -c1-200; done
