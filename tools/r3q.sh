#!/bin/bash
# query kernel register budget: 6 CTAs/SM (40 regs) vs 8 (32 regs)
OUT=gpurun_out/r3q; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab2.sh r3q2 2 30 2 $P/libeirene.so $P/libeirene_q6.so
