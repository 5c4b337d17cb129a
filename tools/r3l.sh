#!/bin/bash
# cfg3 slow groups: phases inside l2_sort (gprof build)
OUT=gpurun_out/r3l; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
EIRENE_LIB=$P/libeirene_gprof.so EIRENE_GROUP_PROF=1 timeout 300 python bench.py --config 3 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/gprof3.log 2>&1
grep "group prof" $OUT/gprof3.log | tail -40
