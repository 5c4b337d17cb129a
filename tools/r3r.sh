#!/bin/bash
# query kernel register budget: 8 / 6 / 5 / 4 CTAs per SM
OUT=gpurun_out/r3r; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab2.sh r3r2 2 30 2 $P/libeirene.so $P/libeirene_q6.so $P/libeirene_q5.so $P/libeirene_q4.so
bash tools/ab2.sh r3r3 3 20 1 $P/libeirene.so $P/libeirene_q6.so
