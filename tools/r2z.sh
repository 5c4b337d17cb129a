#!/bin/bash
# split storms: no level_count[0] atomic, counters on their own lines, no root check below height 2
OUT=gpurun_out/r2z; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab_libs.sh r2z1 1 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
bash tools/ab_libs.sh r2z4 4 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
EIRENE_UPDATE_PROF=1 timeout 600 python bench.py --config 4 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 2>&1 | grep "upd prof" | tail -2
