#!/bin/bash
# resident-sized grid-barrier kernels (distribution, update) launched without the cooperative attribute: A/B cfg2, cfg7-like cfg3, cfg1
OUT=gpurun_out/r3o; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab2.sh r3o2 2 30 2 $P/libeirene.so $P/libeirene_plain.so
bash tools/ab2.sh r3o3 3 20 1 $P/libeirene.so $P/libeirene_plain.so
bash tools/ab2.sh r3o1 1 20 1 $P/libeirene.so $P/libeirene_plain.so
EIRENE_LIB=$P/libeirene_plain.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "pipelin or structural or storm or cfg1" > $OUT/plain_tests.log 2>&1; tail -2 $OUT/plain_tests.log
