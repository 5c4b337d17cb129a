#!/bin/bash
# split storms: 32-write level-0 chunks with batched runs (UPD_LSYNC_CH=32) vs 16: parity of the variant, A/B cfg4 / cfg1
OUT=gpurun_out/r3t; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
EIRENE_LIB=$P/libeirene_ch32.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $OUT/ch32_tests.log 2>&1; tail -2 $OUT/ch32_tests.log
bash tools/ab2.sh r3t4 4 10 2 $P/libeirene.so $P/libeirene_ch32.so
bash tools/ab2.sh r3t1 1 20 2 $P/libeirene.so $P/libeirene_ch32.so
