#!/bin/bash
# update kernel: one thread per CTA reads what is left (vs every thread); query kernel CTA size 256 / 768 / 1024
OUT=gpurun_out/r3x; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab2.sh r3x2 2 30 2 $P/libeirene_head.so $P/libeirene.so $P/libeirene_q768.so $P/libeirene_q1024.so
bash tools/ab2.sh r3x3 3 20 1 $P/libeirene_head.so $P/libeirene.so
bash tools/ab2.sh r3x1 1 20 1 $P/libeirene_head.so $P/libeirene.so
