#!/bin/bash
# write values gathered by the query kernel (WVAL_TS); group-kernel unroll variants (A/B)
OUT=gpurun_out/r2s; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab_libs.sh r2s 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_ru4.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_gu2.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_gu4.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_gu2ru4.so
bash tools/ab_libs.sh r2s3 3 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_gu2ru4.so
