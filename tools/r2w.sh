#!/bin/bash
OUT=gpurun_out/r2w; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
bash tools/ab_libs.sh r2w3 3 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_v0.so
bash tools/ab_libs.sh r2w 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
