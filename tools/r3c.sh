#!/bin/bash
# query kernel: contiguous per-thread runs (EIRENE_QRUN) A/B on cfg2, cfg3, cfg7-like (cfg2 only for 64-bit libs)
OUT=gpurun_out/r3c; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab_libs.sh r3c2 2 $P/libeirene.so $P/libeirene_qrun.so $P/libeirene_qrunpf.so
bash tools/ab_libs.sh r3c3 3 $P/libeirene.so $P/libeirene_qrun.so
