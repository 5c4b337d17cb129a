#!/bin/bash
# group kernel: rank-loop sub-bucket bound FAST_SB 32 / 16 / 8 (bigger sub-buckets: bitonic / hot-run sort)
OUT=gpurun_out/r3s; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab2.sh r3s3 3 20 2 $P/libeirene.so $P/libeirene_fs16.so $P/libeirene_fs8.so
bash tools/ab2.sh r3s2 2 20 1 $P/libeirene.so $P/libeirene_fs16.so $P/libeirene_fs8.so
