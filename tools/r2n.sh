#!/bin/bash
# two-phase group stage: GPU suite, cfg5 mixes, cfg2/cfg3 A/B against the previous build
OUT=gpurun_out/r2n; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -3 $OUT/gpu_tests.log
for m in B U A C; do timeout 900 python bench.py --config 5 --mix $m --steps 5 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/cfg5$m.log 2>&1; tail -1 $OUT/cfg5$m.log | cut -c1-250; grep -o '"stage_ms": {[^}]*}' $OUT/cfg5$m.log; grep -o '"parity": {[^}]*}' $OUT/cfg5$m.log; done
bash tools/ab_libs.sh r2n 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
bash tools/ab_libs.sh r2n3 3 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
