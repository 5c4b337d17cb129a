#!/bin/bash
# hot-key bitmaps filled by the query kernel: GPU suite, cfg5 mixes, cfg3 / cfg2 A/B
OUT=gpurun_out/r2o; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -3 $OUT/gpu_tests.log
for m in B A; do timeout 900 python bench.py --config 5 --mix $m --steps 5 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/cfg5$m.log 2>&1; tail -1 $OUT/cfg5$m.log | cut -c1-120; grep -o '"stage_ms": {[^}]*}' $OUT/cfg5$m.log; grep -o '"mismatches": [0-9]*' $OUT/cfg5$m.log; done
bash tools/ab_libs.sh r2o3 3 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
bash tools/ab_libs.sh r2o 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
