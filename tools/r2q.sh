#!/bin/bash
# query kernel without the device graph API (ncu sees it inside graphs): GPU suite, launch list, full capture of the query kernel
OUT=gpurun_out/r2q; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv $BENCH > $OUT/launches.log 2>&1
python tools/launches.py $OUT/launches.csv 3 2>/dev/null | head -8
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:query_kernel" -s 3 -c 1 -o $OUT/q $BENCH > $OUT/q.log 2>&1
python tools/ncu_lines.py $OUT/q.ncu-rep query_kernel 30 > $OUT/q_lines.txt 2>&1; head -20 $OUT/q_lines.txt
